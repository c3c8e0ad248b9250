"""Oracle: striped migration (GROUTER_STRIPED_MIGRATION, R47).

Spills leave a GPU over its route set R(src) -- the gFn-host plan of
PAPER.md L178 / Fig. 5(a) ("data from GPU1 is first routed via NVLink to peer
GPUs (GPU3, GPU5, and GPU7), which concurrently stage it to host memory ...
GPUs sharing a PCIe switch (e.g., GPU2) are excluded") -- and restores come
back over R(d) like a fetch ("parallel PCIe transfers in GROUTER mitigate the
overhead of fetching data from host memory", L366).  Pinned on the L178 worked
example (which GPUs carry bytes), on tiling and conservation, and on the
property that striping changes routes only: every decision and every byte
equals the single-path run.
"""
import random

import pytest

from oracle import model, runner
from synth import calib as C
from synth import traces as T

MiB = 1 << 20


def _spill_and_restore(calib, n, striped, dev=0):
    b = T.Builder(11)
    f = T.fn(1, 1, dev)
    o = b.put(f, n)                      # gFn put by copy: resident on `dev`, no PCIe traffic
    b.pool_limit(dev, 0)                 # spill it
    b.pool_limit(dev, 1 << 40)           # room again: proactive restore (R42)
    g = b.get(T.fn(1, 2, dev), o)
    b.release(T.fn(1, 2, dev), g)
    return runner.run(b.ops, calib, restore=True, striped_migration=striped, keep_bytes=True)


def test_fig5a_spill_uses_l178_routes():
    """L178 worked example: GPU1's data reaches the host through GPU1, GPU3,
    GPU5 and GPU7 (logical 0, 2, 4, 6); GPU2 (logical 1, same PCIe switch) and
    the even-numbered paper GPUs carry nothing."""
    n = 64 * MiB
    out = _spill_and_restore(C.fig5a(), n, striped=True)
    recs = out["records"]
    assert recs[1]["victims"] == [1] and recs[2]["restored"] == [1]
    lb = out["oracle"].link_bytes
    d2h = {g: lb.get(("d2h", g), 0) for g in range(8)}
    h2d = {g: lb.get(("h2d", g), 0) for g in range(8)}
    assert {g for g, v in d2h.items() if v} == {0, 2, 4, 6}
    assert {g for g, v in h2d.items() if v} == {0, 2, 4, 6}
    assert sum(d2h.values()) == n and sum(h2d.values()) == n
    # single path: everything on the GPU's own engines
    ref = _spill_and_restore(C.fig5a(), n, striped=False)["oracle"].link_bytes
    assert ref == {("copy", 0): n, ("d2h", 0): n, ("h2d", 0): n}     # copy: the gFn's by-copy put


def test_migration_plans_tile_the_object():
    """I1 for migration plans: chunks are disjoint and cover [0, n) exactly,
    striped or not, for sizes around the chunk boundary."""
    orc = model.Oracle(C.fig5a(), striped_migration=True)
    for n in (1, 4095, 2 * MiB - 1, 2 * MiB, 2 * MiB + 1, 38_535_168, 67_108_864 + 12345):
        for src, dst in ((0, model.HOST), (model.HOST, 0), (5, model.HOST), (model.HOST, 3)):
            plan = orc._migration_plan(src, dst, n)
            spans = sorted((c["offset"], c["offset"] + c["bytes"]) for c in plan)
            assert spans[0][0] == 0 and spans[-1][1] == n
            assert all(a[1] == b[0] for a, b in zip(spans, spans[1:])), (n, src, dst)
            assert all(c["bytes"] > 0 for c in plan)


def test_one_route_reduces_to_single_path():
    """A GPU whose route set is itself alone (one GPU, or no multipath)
    migrates exactly as R41/R42 say: one path on its own engines."""
    for calib, mp in ((C.b200_hgx(1), True), (C.b200_hgx(4), False)):
        b = T.Builder(3)
        f = T.fn(1, 1, 0)
        b.put(f, 9 * MiB)
        b.pool_limit(0, 0)
        b.pool_limit(0, 1 << 40)
        lb = runner.run(b.ops, calib, restore=True, striped_migration=True, multipath=mp)["oracle"].link_bytes
        assert lb == {("copy", 0): 9 * MiB, ("d2h", 0): 9 * MiB, ("h2d", 0): 9 * MiB}


@pytest.mark.parametrize("seed", range(10))
def test_striping_changes_routes_only(seed):
    """Random traces with spills and restores: statuses, victims, restores,
    placements, pool usage and every delivered byte equal the single-path
    run; per direction the engines move the same total (conservation)."""
    rng = random.Random(700 + seed)
    n = rng.choice([2, 3, 4])
    calib = C.b200_hgx(n, shared_pairs=False)
    ops = T.random_trace(rng, n, n_ops=150, max_n=7 * MiB, run_seed=seed)
    caps = [rng.choice([8, 16]) * MiB for _ in range(n)]
    kw = dict(host_store_bytes=1 << 30, pool_cap=caps, restore=True)
    a = runner.run(ops, calib, striped_migration=False, **kw)
    b = runner.run(ops, calib, striped_migration=True, **kw)
    for x, y in zip(a["records"], b["records"]):
        for k in ("status", "oid", "where", "victims", "restored", "used", "host_used", "digest"):
            assert x.get(k) == y.get(k), (x["i"], k)
    la, lb = a["oracle"].link_bytes, b["oracle"].link_bytes
    for kind in ("h2d", "d2h"):
        assert sum(v for (k, _), v in la.items() if k == kind) == sum(v for (k, _), v in lb.items() if k == kind)
    # (small objects may legitimately stay on the direct path: the O6 split
    # weighs each relay's fill latency; the L178 example above shows striping)
