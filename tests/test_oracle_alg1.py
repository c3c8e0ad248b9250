"""Pins of oracle/alg1.py (§4.3.3, Alg. 1; readings R11,
R46) and of the synthetic NVLink topologies it runs on.

* the DGX-V100 mesh reproduces the paper's Fig. 6 statistics (28% of pairs
  at half bandwidth, 42% without a direct NVLink) and its named pairs;
* NVSwitch (HGX B200): every one of the 56 ordered pairs gets exactly the
  direct path (R11's special case);
* a hand-derived selection on the idle DGX-V100 (GPU4 -> GPU1) that contains
  both paths of Fig. 9(b);
* direct priority, balancing and its refusal conditions by hand;
* conservation invariants on random request sequences;
* L242's chunk-size example through nvl_plan."""
import random

import pytest

from oracle import alg1
from synth import calib as C

G24, G48 = 24_000_000_000, 48_000_000_000


def test_dgx_v100_statistics():
    t = C.dgx_v100_topo()
    pairs = [(a, b) for a in range(8) for b in range(a + 1, 8)]
    half = [p for p in pairs if t[p[0]][p[1]] == G24]
    none = [p for p in pairs if t[p[0]][p[1]] == 0]
    assert round(100 * len(half) / len(pairs)) == 29 and len(half) == 8     # "28% of GPU pairs"
    assert round(100 * len(none) / len(pairs)) == 43 and len(none) == 12    # "42% lack direct NVLink"
    assert t[0][3] == G24            # "GPU1-GPU4 achieve only half the expected bandwidth"
    assert t[0][4] == 0              # "GPU1-GPU5 lack direct NVLink"
    assert all(sum(1 for b in range(8) if t[a][b]) in (4,) for a in range(8))
    assert all(sum(t[a]) == 6 * G24 for a in range(8))      # 6 NVLinks per V100


def test_nvswitch_direct_only():
    t = C.nvswitch_topo(8)
    for gs in range(8):
        for gd in range(8):
            if gs == gd:
                continue
            pt = alg1.PathTable(t, 8)
            paths, moved = pt.select(1, gs, gd)
            assert paths == [([gs, 8, gd], 900_000_000_000)] and moved == []


def test_fig9b_gpu4_to_gpu1_idle():
    """Idle DGX-V100, GPU4 -> GPU1 (0-based 3 -> 0).  By hand: the direct
    link (1 x 24 GB/s); 2-edge paths 3-1-0 (b = min(48, 24) = 24) and 3-2-0
    (48); then BW_in(0) still has 6->0 and BW_out(3) has 3->1 (24 left) and
    3->5, so 3-edge paths are scanned: 3-1-2-0 is not idle (3->1 carries a
    path), 3-5-6-0 is idle (b = min(24, 24, 48) = 24).  Fig. 9(b) names
    GPU4->GPU1 and GPU4->GPU6->GPU7->GPU1 = [3, 0] and [3, 5, 6, 0]."""
    pt = alg1.PathTable(C.dgx_v100_topo(), 8)
    paths, moved = pt.select(1, 3, 0)
    assert paths == [([3, 0], G24), ([3, 1, 0], G24), ([3, 2, 0], G48), ([3, 5, 6, 0], G24)]
    assert moved == []


def test_direct_priority_reassigns_indirect_user():
    """L235: a direct path occupied by another function's indirect route is
    given back to the pair it connects."""
    t = C.dgx_v100_topo()
    pt = alg1.PathTable(t, 8)
    pt.select(7, 3, 0)                     # takes [3,1,0] among others: uses 1->0
    assert any(p == (3, 1, 0) for _, _, p in pt.table())
    paths, moved = pt.select(8, 1, 0)      # 1->0 has a direct link
    assert (7, 3, 0) in moved
    assert paths[0] == ([1, 0], G24)
    assert not any(f == 7 and p == (3, 1, 0) for f, _, p in pt.table())


def _mesh(n, links):
    t = [[0] * n for _ in range(n)]
    for (a, b), k in links.items():
        t[a][b] = t[b][a] = k * G24
    return t


def test_balancing_takes_a_busy_path_from_a_richer_function():
    """L237 by hand.  Links 0-1, 1-3, 0-2, 2-3, 4-1, 5-3 (one each).  f1
    (0 -> 3) takes [0,1,3] and [0,2,3] (48 GB/s, two paths).  f2 (4 -> 3) has
    one candidate, [4,1,3], whose 1->3 is saturated by f1; BW_out(4) = 24 and
    BW_in(3) = 24 (5->3) are unsaturated, f1 uses more (48 > 0) and keeps
    [0,2,3]: f1 gives [0,1,3] up and f2 takes [4,1,3]."""
    links = {(0, 1): 1, (1, 3): 1, (0, 2): 1, (2, 3): 1, (4, 1): 1, (5, 3): 1}
    pt = alg1.PathTable(_mesh(6, links), 6)
    assert pt.select(1, 0, 3)[0] == [([0, 1, 3], G24), ([0, 2, 3], G24)]
    paths, moved = pt.select(2, 4, 3)
    assert paths == [([4, 1, 3], G24)] and moved == [(1, 0, 3)]
    assert pt.table() == [(1, G24, (0, 2, 3)), (2, G24, (4, 1, 3))]


def test_balancing_refused_for_a_single_path_holder():
    links = {(0, 1): 1, (1, 3): 1, (4, 1): 1, (5, 3): 1}
    pt = alg1.PathTable(_mesh(6, links), 6)
    assert pt.select(1, 0, 3)[0] == [([0, 1, 3], G24)]
    assert pt.select(2, 4, 3) == ([], [])                  # f1 cannot switch


def test_balancing_refused_when_holder_is_not_richer():
    """f2 first takes the idle [4,5,3] at 48 GB/s; f1 also uses 48: not more."""
    links = {(0, 1): 1, (1, 3): 1, (0, 2): 1, (2, 3): 1, (4, 1): 1, (4, 5): 2, (5, 3): 3}
    pt = alg1.PathTable(_mesh(6, links), 6)
    pt.select(1, 0, 3)
    paths, moved = pt.select(2, 4, 3)
    assert paths == [([4, 5, 3], 2 * G24)] and moved == []


@pytest.mark.parametrize("seed", range(25))
def test_random_sequences_conserve_bandwidth(seed):
    rng = random.Random(seed)
    n = rng.choice([3, 4, 5, 6, 8])
    t = C.random_topo(rng, n) if seed % 3 else C.dgx_v100_topo()
    n = len(t)
    pt = alg1.PathTable(t, n, max_edges=rng.choice([2, 3, 4]))
    live = set()
    for step in range(30):
        if live and rng.random() < 0.3:
            f = rng.choice(sorted(live))
            pt.release(f)
            live.discard(f)
        else:
            f = step + 1
            gs, gd = rng.sample(range(n), 2)
            paths, _ = pt.select(f, gs, gd)
            live.add(f)
            for p, b in paths:
                assert p[0] == gs and p[-1] == gd and len(set(p)) == len(p) and b > 0
                assert len(p) - 1 <= pt.H
        # per edge: free + allocated == capacity, nothing negative
        used = [[0] * n for _ in range(n)]
        for f, b, p in pt.table():
            for u, v in alg1.edges(list(p)):
                used[u][v] += b
        for u in range(n):
            for v in range(n):
                assert pt.bw[u][v] >= 0 and pt.bw[u][v] + used[u][v] == t[u][v]
        # a function's own paths never share an edge (no self-contention)
        for f in live:
            es = [e for a in pt.paths_of(f) for e in alg1.edges(a[1])]
            assert len(es) == len(set(es))
    for f in sorted(live):
        pt.release(f)
    assert pt.bw == t and pt.alloc == []


def test_serve_order_least_residual_first():
    t = C.dgx_v100_topo()
    reqs = [(1, 0, 2), (2, 0, 3), (3, 0, 4), (4, 1, 3)]
    # residual direct capacity: 0-2 48, 0-3 24, 0-4 none, 1-3 48
    assert alg1.serve_order(t, reqs) == [(3, 0, 4), (2, 0, 3), (1, 0, 2), (4, 1, 3)]


def test_nvl_plan_chunk_size_proportional():
    """L242: "a 48 GB/s link receives twice the chunk size of a 24 GB/s link"."""
    paths = [([0, 2], G48), ([0, 3], G24)]
    plan = alg1.nvl_plan(paths, 64 << 20, 8, 0, 2 << 20)
    sizes = {}
    for c in plan:
        sizes.setdefault(c["path"], set()).add(c["bytes"])
    assert max(sizes[0]) == 2 << 20 and max(sizes[1]) == 1 << 20
    off = 0
    for c in sorted(plan, key=lambda c: c["offset"]):
        assert c["offset"] == off
        off += c["bytes"]
    assert off == 64 << 20
    by = {p: sum(c["bytes"] for c in plan if c["path"] == p) for p in (0, 1)}
    assert abs(by[0] - 2 * by[1]) <= 2 << 20                 # 2:1 shares
