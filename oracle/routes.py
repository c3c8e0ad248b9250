"""Route set R(d) and per-path cost parameters.

Paper basis:
* L178 §4.3.1 "gFn-host": data is staged over idle PCIe links of route GPUs;
  "GPUs sharing a PCIe switch (e.g., GPU2) are excluded as route GPUs, as
  they share a single PCIe link to host memory".
* L131 §3.2.2: selecting several GPUs behind one switch induces contention.
* L271 §5: PCIe paths "are fixed and can be pre-generated during GROUTER
  initialization" -- R(d) is computed once from the calibration.
* Readings R10 (lowest index represents a group; d represents its own group).
"""
from __future__ import annotations


def uplink_groups(calib: dict) -> list:
    """O7 step 1.  Explicit ``uplink_groups`` win; else GPUs i != j share an
    uplink iff their concurrent H2D sum is <= 1.15x the better solo bandwidth
    (integer test: 100*pair <= 115*max(solo_i, solo_j)); groups are the
    connected components of that relation, each sorted, listed by lowest index."""
    n = calib["n_gpus"]
    if "uplink_groups" in calib:
        gs = [sorted(g) for g in calib["uplink_groups"]]
        return sorted(gs, key=lambda g: g[0])
    solo = calib["h2d_Bps"]
    pair = calib["h2d_pair_Bps"]
    # plain connected components by repeated relabelling (n <= 8)
    label = list(range(n))
    changed = True
    while changed:
        changed = False
        for i in range(n):
            for j in range(n):
                if i != j and 100 * pair[i][j] <= 115 * max(solo[i], solo[j]):
                    m = min(label[i], label[j])
                    if label[i] != m or label[j] != m:
                        label[i] = label[j] = m
                        changed = True
    groups = {}
    for i in range(n):
        groups.setdefault(label[i], []).append(i)
    return sorted((sorted(g) for g in groups.values()), key=lambda g: g[0])


def route_set(calib: dict, d: int, multipath: bool = True) -> list:
    """O7 steps 2-5: R(d) = [d] + lowest-index GPU of every other uplink group
    (ascending by that index) that has P2P access to d."""
    if not multipath:
        return [d]
    routes = [d]
    for g in uplink_groups(calib):
        if d in g:
            continue
        r = g[0]
        if calib["p2p"][r][d]:
            routes.append(r)
    return routes


def path_params(calib: dict, d: int, r: int) -> tuple:
    """(alpha_ps, beta_Bps, phi_ps) of the path host -> r (-> d).

    Direct (r == d): the CE of d.  Relayed: CE of r, then one NVLink hop whose
    bandwidth caps the path (beta = min(PCIe_r, NVLink)) and whose fill adds
    ``relay_phi_ps``."""
    alpha = calib["h2d_alpha_ps"][r]
    if r == d:
        return alpha, calib["h2d_Bps"][d], calib["h2d_phi_ps"][d]
    beta = min(calib["h2d_Bps"][r], calib["nvl_Bps"])
    return alpha, beta, calib["h2d_phi_ps"][r] + calib["relay_phi_ps"]
