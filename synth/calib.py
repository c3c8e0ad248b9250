"""Synthetic calibration descriptions (the "hardware mock").

A calibration is a plain dict (JSON-serialisable) that both the oracle and
the library consume as DATA:

    n_gpus           visible GPUs (logical indices 0..n-1)
    nvl_Bps          NVLink bandwidth per direction per GPU, bytes/s (int)
    h2d_Bps[i]       solo pinned host->GPU i bandwidth, bytes/s (int)
    h2d_alpha_ps[i]  per-chunk copy-engine overhead on GPU i, picoseconds
    h2d_phi_ps[i]    first-chunk (fill) latency of the direct path into i, ps
    relay_phi_ps     extra fill latency of a relayed path (one NVLink hop), ps
    h2d_pair_Bps     n x n: concurrent H2D sum when i and j copy together
                     (diagonal = solo).  Absent => ``uplink_groups`` given.
    uplink_groups    optional explicit list of GPU groups sharing an uplink
    p2p              n x n 0/1 peer-access matrix
    device_map       optional: logical GPU -> physical CUDA ordinal.  Only
                     the library runner reads it (several logical GPUs may
                     share one physical B200 in single-GPU tests); the
                     oracle ignores it.

The numbers here are inputs, not measurements; ``calib/probe`` in the
library writes the same format from a live box.
"""
from __future__ import annotations

import json
import random

PS = 10**12  # picoseconds per second


def _pair_matrix(n, solo, groups):
    g_of = {}
    for gi, g in enumerate(groups):
        for x in g:
            g_of[x] = gi
    m = [[0] * n for _ in range(n)]
    for i in range(n):
        for j in range(n):
            if i == j:
                m[i][j] = solo[i]
            elif g_of[i] == g_of[j]:
                m[i][j] = max(solo[i], solo[j])  # shared uplink: no gain
            else:
                m[i][j] = solo[i] + solo[j]
    return m


def b200_hgx(n: int = 8, h2d_Bps: int = 55_000_000_000, shared_pairs: bool = True,
             nvl_Bps: int = 900_000_000_000) -> dict:
    """Uniform NVSwitch box; GPUs (2k, 2k+1) share one PCIe uplink if
    ``shared_pairs`` (a plausible HGX layout -- the probe decides on a real box)."""
    solo = [h2d_Bps] * n
    if shared_pairs:
        groups = [[i, i + 1] if i + 1 < n else [i] for i in range(0, n, 2)]
    else:
        groups = [[i] for i in range(n)]
    return {
        "name": f"b200_hgx{n}" + ("_pairs" if shared_pairs else "_solo"),
        "n_gpus": n,
        "nvl_Bps": nvl_Bps,
        "h2d_Bps": solo,
        "h2d_alpha_ps": [4_000_000] * n,      # 4 us per CE chunk
        "h2d_phi_ps": [10_000_000] * n,       # 10 us to first byte
        "relay_phi_ps": 20_000_000,           # forward launch + one hop
        "h2d_pair_Bps": _pair_matrix(n, solo, groups),
        "p2p": [[1] * n for _ in range(n)],
    }


def fig5a() -> dict:
    """Worked example of PAPER.md L178 / Fig. 5(a): GPU1 and GPU2 share a PCIe
    switch, routes for GPU1 are GPU3, GPU5, GPU7.  Paper numbering is 1-based;
    here GPU k of the paper is logical index k-1, switches {1,2},{3,4},{5,6},{7,8}."""
    c = b200_hgx(8, shared_pairs=True)
    c["name"] = "fig5a"
    c["uplink_groups"] = [[0, 1], [2, 3], [4, 5], [6, 7]]
    del c["h2d_pair_Bps"]
    return c


def virtual(k: int, phys: int = 0, h2d_Bps: int = 55_000_000_000) -> dict:
    """k logical GPUs on ONE physical GPU, each its own uplink group, for
    exercising striping/forwarding logic on a single B200."""
    c = b200_hgx(k, h2d_Bps=h2d_Bps, shared_pairs=False)
    c["name"] = f"virtual{k}"
    c["device_map"] = [phys] * k
    return c


def random_calib(rng: random.Random, n: int) -> dict:
    """Random integer topology for fuzzing planner parity."""
    solo = [rng.randint(8, 64) * 1_000_000_000 for _ in range(n)]
    # random grouping
    groups, cur = [], []
    for i in range(n):
        cur.append(i)
        if rng.random() < 0.5:
            groups.append(cur)
            cur = []
    if cur:
        groups.append(cur)
    c = {
        "name": f"random{n}",
        "n_gpus": n,
        "nvl_Bps": rng.choice([24, 48, 300, 900]) * 1_000_000_000,
        "h2d_Bps": solo,
        "h2d_alpha_ps": [rng.randint(0, 20) * 1_000_000 for _ in range(n)],
        "h2d_phi_ps": [rng.randint(0, 50) * 1_000_000 for _ in range(n)],
        "relay_phi_ps": rng.randint(0, 60) * 1_000_000,
        "h2d_pair_Bps": _pair_matrix(n, solo, groups),
        "p2p": [[1 if (i == j or rng.random() < 0.9) else 0 for j in range(n)] for i in range(n)],
    }
    for i in range(n):
        for j in range(n):
            c["p2p"][i][j] = c["p2p"][j][i] = max(c["p2p"][i][j], c["p2p"][j][i]) if i != j else 1
    return c


def dump(c: dict, path: str) -> None:
    with open(path, "w") as f:
        json.dump(c, f, indent=1)


def load(path: str) -> dict:
    with open(path) as f:
        return json.load(f)


# NVLink topologies for Alg. 1; capacities in B/s per direction.
NVL_LINK_Bps = 24_000_000_000        # L242 "24 GB/s or 48 GB/s per link" (V100 NVLink2)
# DGX-V100 hybrid cube-mesh, numbered so that the paper's examples hold
# (0-based index = paper "GPUk" - 1): GPU1-GPU4 has one link (half bandwidth,
# L131), GPU1-GPU5 none, and Fig. 9(b)'s GPU4->GPU6->GPU7->GPU1 path exists.
DGX_V100_LINKS = {(0, 1): 1, (0, 2): 2, (0, 3): 1, (0, 6): 2, (1, 2): 1, (1, 3): 2, (1, 4): 2,
                  (2, 3): 2, (2, 7): 1, (3, 5): 1, (4, 5): 2, (4, 6): 1, (4, 7): 1, (5, 6): 1,
                  (5, 7): 2, (6, 7): 2}


def dgx_v100_topo() -> list:
    """8x8 directed capacity matrix of the DGX-V100 NVLink mesh (Fig. 6a)."""
    t = [[0] * 8 for _ in range(8)]
    for (a, b), k in DGX_V100_LINKS.items():
        t[a][b] = t[b][a] = k * NVL_LINK_Bps
    return t


def nvswitch_topo(n: int = 8, port_Bps: int = 900_000_000_000) -> list:
    """HGX B200: n GPUs and one NVSwitch node (index n); every GPU has one
    port of port_Bps per direction to the switch fabric."""
    t = [[0] * (n + 1) for _ in range(n + 1)]
    for g in range(n):
        t[g][n] = t[n][g] = port_Bps
    return t


def random_topo(rng: random.Random, n: int) -> list:
    """Random symmetric NVLink mesh (0-3 links per pair) for fuzzing."""
    t = [[0] * n for _ in range(n)]
    for a in range(n):
        for b in range(a + 1, n):
            k = rng.choice([0, 0, 1, 2, 3])
            t[a][b] = t[b][a] = k * NVL_LINK_Bps
    return t
