"""Pins for the oracle's chunk splitter.

* brute force over every composition of N granules into k paths (tiny N):
  the oracle's T* must equal the true minimum makespan, and its shares the
  lexicographically-largest optimal composition (canonical fill-in-route-order);
* worked example L242 (48 vs 24 GB/s -> 2:1 chunk sizes);
* hand-evaluated cost values, closed-form balanced split, tiling invariant I1.
"""
import itertools
import random

import pytest

from oracle import splitter
from oracle.splitter import CHUNK, GRANULE
from synth import calib as C

PS = 10**12


def _compositions(N, k):
    for cuts in itertools.combinations(range(N + k - 1), k - 1):
        prev, parts = -1, []
        for c in cuts:
            parts.append(c - prev - 1)
            prev = c
        parts.append(N + k - 1 - prev - 1)
        yield parts


def _brute(N, params, Cps, g):
    def cost(m, a, b, f, cp):  # cost model of O6, evaluated independently
        if m == 0:
            return 0
        return f + ((m * g + cp - 1) // cp) * a + (m * g * PS + b - 1) // b
    best, best_s = None, None
    for s in _compositions(N, len(params)):
        ms = max(cost(m, a, b, f, cp) for m, (a, b, f), cp in zip(s, params, Cps))
        if best is None or ms < best or (ms == best and s > best_s):
            best, best_s = ms, s
    return best, best_s


@pytest.mark.parametrize("seed", range(120))
def test_split_matches_brute_force(seed):
    rng = random.Random(seed)
    k = rng.randint(1, 4)
    N = rng.randint(0, 48 if k <= 3 else 30)
    g = rng.choice([1, 4, 4096])
    params = [(rng.randint(0, 50) * 1000, rng.randint(1, 64) * 10**9 // (4096 // g),
               rng.randint(0, 200) * 1000) for _ in range(k)]
    Cps = splitter.chunk_sizes([b for _, b, _ in params], C=8 * g, g=g)
    T, s = splitter.split_shares(N, params, Cps, g)
    bT, bs = _brute(N, params, Cps, g)
    assert T == bT
    assert s == bs
    assert splitter.makespan(s, params, Cps, g) == T


def test_worked_example_l242_proportional_chunks():
    # "a 48 GB/s link receives twice the chunk size of a 24 GB/s link"
    assert splitter.chunk_sizes([48 * 10**9, 24 * 10**9]) == [2 * 2**20, 2**20]
    assert splitter.chunk_sizes([24 * 10**9, 48 * 10**9]) == [2**20, 2 * 2**20]
    # rounded down to the 4 KiB granule, never below it
    assert splitter.chunk_sizes([900 * 10**9, 55 * 10**9])[1] == (2**21 * 55 // 900) // 4096 * 4096
    assert splitter.chunk_sizes([10**12, 1])[1] == GRANULE


def test_cost_hand_values():
    # phi=10, alpha=3, beta=1e12 B/s (1 B/ps), g=4096, C_p=8192, m=3:
    # 10 + ceil(12288/8192)*3 + ceil(12288) = 10 + 6 + 12288
    assert splitter.path_time(3, 3, 10**12, 10, 8192, 4096) == 12304
    assert splitter.path_time(0, 3, 10**12, 10, 8192, 4096) == 0
    assert splitter.path_cap(12304, 100, 3, 10**12, 10, 8192, 4096) == 3
    assert splitter.path_cap(12303, 100, 3, 10**12, 10, 8192, 4096) == 2


def test_balanced_closed_form():
    # identical paths, no per-chunk or fill cost: shares = ceil(N/k) greedily
    params = [(0, 10**9, 0)] * 4
    Cps = splitter.chunk_sizes([10**9] * 4)
    for N in range(0, 40):
        _, s = splitter.split_shares(N, params, Cps)
        q = -(-N // 4)
        exp, rem = [], N
        for _ in range(4):
            exp.append(min(q, rem))
            rem -= exp[-1]
        assert s == exp


def test_small_payload_stays_on_direct_path():
    c = C.b200_hgx(8, shared_pairs=False)
    plan = splitter.plan_h2d(c, 3, 4096)
    assert [(p["offset"], p["bytes"], p["route_gpu"]) for p in plan] == [(0, 4096, 3)]


def _check_tiling(plan, n):
    off = 0
    for ch in plan:
        assert ch["offset"] == off and ch["bytes"] > 0
        off += ch["bytes"]
    assert off == n


@pytest.mark.parametrize("n", [0, 1, 4095, 4096, 4097, 2**21 - 1, 2**21, 2**21 + 1,
                               38_535_168, 1 << 30])
@pytest.mark.parametrize("topo", ["pairs", "solo", "one"])
def test_plan_tiles_payload(n, topo):
    c = {"pairs": C.b200_hgx(8), "solo": C.b200_hgx(8, shared_pairs=False),
         "one": C.b200_hgx(1)}[topo]
    plan = splitter.plan_h2d(c, 0, n)
    _check_tiling(plan, n)
    routes = sorted({p["route_gpu"] for p in plan})
    Cps = splitter.chunk_sizes([c["h2d_Bps"][0]] * 8)
    for p in plan:
        assert p["bytes"] <= Cps[0]
    if topo == "pairs" and n >= 1 << 30:
        assert routes == [0, 2, 4, 6]     # one GPU per uplink group


def test_plan_single_d2d():
    n = 38_535_168
    plan = splitter.plan_single(n, 5)
    assert len(plan) == 19 and plan[-1]["bytes"] == n - 18 * CHUNK == 786_432
    _check_tiling(plan, n)
    assert all(p["route_gpu"] == 5 and p["path"] == 0 for p in plan)
    assert len(splitter.plan_single(1 << 30, 0)) == 512
    assert splitter.plan_single(0, 0) == []


def test_layout_interleaves_rounds():
    # two paths, C_0 = 2 granules, C_1 = 1 granule, shares 5 and 2 (g = 1)
    ch = splitter.layout(7, [5, 2], [2, 1], [0, 4], g=1)
    assert [(c["offset"], c["bytes"], c["route_gpu"]) for c in ch] == \
        [(0, 2, 0), (2, 1, 4), (3, 2, 0), (5, 1, 4), (6, 1, 0)]
    # final chunk clipped to end at n when the last granule is partial (g = 4)
    ch = splitter.layout(25, [5, 2], [8, 4], [0, 4], g=4)
    assert [(c["offset"], c["bytes"], c["route_gpu"]) for c in ch] == \
        [(0, 8, 0), (8, 4, 4), (12, 8, 0), (20, 4, 4), (24, 1, 0)]
