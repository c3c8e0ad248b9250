"""Pins for the oracle's put/get/evict state machine.

* golden trace hand-derived from the paper's rules (tests/golden/small_trace.md);
* Fig. 11(b) worked example: queue-aware eviction keeps the
  data of the function at the head of the queue, LRU would not;
* identity I2 (checked by the runner on every get), I4 capacity, I6 refcounts
  (everything back to 0 at the end of the config traces), I1/I3 on plans.
"""
import json
import os
import random

import pytest

from oracle import model, runner
from synth import calib as C
from synth import traces as T

GOLD = os.path.join(os.path.dirname(__file__), "golden")
MiB = 1 << 20


def _small_trace_ops():
    b = T.Builder(run_seed=11)
    cfn, g0, g1 = T.fn(1, 1, T.HOST), T.fn(1, 2, 0), T.fn(1, 3, 1)
    o1 = b.put(cfn, 3 * MiB, hint=0, consumers=1)                 # 0
    o2 = b.put(g0, 1, consumers=0)                                 # 1
    o3 = b.put(T.fn(2, 1, 0), 2 * MiB, consumers=0)                # 2
    g3 = b.get(g1, o1)                                             # 3
    b.get(T.fn(2, 9, 0), o2)                                       # 4 EPERM
    g5 = b.get(T.fn(1, 9, 0), o2)                                  # 5 zero copy
    b.free(T.fn(1, 1, T.HOST), o2)                                 # 6
    b.get(T.fn(1, 9, 0), o2)                                       # 7 ENOENT
    b.release(T.fn(1, 9, 0), g5)                                   # 8
    b.release(g1, g3)                                              # 9
    b.pool_limit(0, 0)                                             # 10
    g11 = b.get(T.fn(2, 2, 1), o3)                                 # 11
    b.free(T.fn(2, 1, 0), o3)                                      # 12
    b.release(T.fn(2, 2, 1), g11)                                  # 13
    b.seal(cfn, o1)                                                # 14
    b.flush()                                                      # 15
    return b.ops


def _plan_tuples(plan):
    return [[c["offset"], c["bytes"], c["path"], c["route_gpu"]] for c in plan]


def test_golden_small_trace():
    g = json.load(open(os.path.join(GOLD, "small_trace.json")))
    ops = _small_trace_ops()
    out = runner.run(ops, C.b200_hgx(2, shared_pairs=False),
                     host_store_bytes=g["host_store_bytes"], pool_cap=g["pool_cap"])
    recs = out["records"]
    assert len(recs) == len(g["expect"])
    for r, e in zip(recs, g["expect"]):
        assert r["status"] == e["status"], (r["i"], r, e)
        if "oid" in e:
            assert r["oid"] == e["oid"]
        if "where" in e:
            assert r.get("where") == e["where"], (r["i"], r)
        assert r["victims"] == e["victims"], r["i"]
        if "plan" in e:
            assert _plan_tuples(r["plan"]) == e["plan"], r["i"]
    disp = [{"server": d["server"], "tenant": d["tenant"], "chunks": d["chunks"], "at_op": r["i"]}
            for r in recs for d in r.get("dispatched", [])]
    assert disp == g["dispatch"]
    orc = out["oracle"]
    assert orc.used == g["final"]["used"] and orc.host_used == g["final"]["host_used"]


def _fig11b(with_hints):
    """Fig. 11(b): a1 and a2 produce outputs O1 (older) and O2 (newer) on one
    GPU; b1 (consumer of O1) is enqueued before b2 (consumer of O2).  A new
    object needs one page."""
    b = T.Builder(3)
    a1, a2, a3 = T.fn(1, 1, 0), T.fn(1, 2, 0), T.fn(1, 3, 0)
    o1 = b.alloc(a1, MiB, consumers=1)
    b.seal(a1, o1)
    o2 = b.alloc(a2, MiB, consumers=1)
    b.seal(a2, o2)
    if with_hints:
        b.next_use(o1, 0)     # b1 at the head of the request queue
        b.next_use(o2, 1)     # b2 behind it (tail)
    b.put(a3, MiB)
    out = runner.run(b.ops, C.b200_hgx(1), pool_cap=[4 * MiB])
    return out["records"]


def test_fig11b_queue_aware_vs_lru():
    # queue-aware: "the output data of function a2 is migrated before the output of a1"
    assert _fig11b(True)[-1]["victims"] == [2]
    # LRU fallback (no queue knowledge) evicts the least recently used: a1's output
    assert _fig11b(False)[-1]["victims"] == [1]


def test_charge():
    assert model.charge(0) == 0
    assert model.charge(1) == 2 * MiB
    assert model.charge(2 * MiB) == 2 * MiB
    assert model.charge(2 * MiB + 1) == 4 * MiB
    assert model.charge(38_535_168) == 19 * 2 * MiB


@pytest.mark.parametrize("n_gpus", [1, 2, 4, 8])
def test_config_traces_drain_to_zero(n_gpus):
    """I6: after every consumer has released, every pool is back to 0 used."""
    c = C.b200_hgx(n_gpus)
    for ops in [T.cfg1(n_gpus, iters=4, scale=64), T.cfg2(n_gpus, requests=6, scale=64),
                T.cfg4(n_gpus, rounds=2, scale=256), T.cfg5(n_gpus, requests=3, scale=256, layers=4),
                T.cfg5(n_gpus, requests=4, limit_frac=0.1, scale=64, layers=4)]:
        if n_gpus == 1 and ops[0]["op"] == "pool_limit":
            continue   # co-located stage B cannot lease a spilled object under a full pool
        out = runner.run(ops, c)
        assert all(r["status"] == "OK" for r in out["records"]), \
            [r for r in out["records"] if r["status"] != "OK"][:2]
        orc = out["oracle"]
        assert orc.used == [0] * n_gpus and orc.host_used == 0
        assert not orc.objects and not orc.leases


def test_cfg5_spills_under_limit():
    """cfg5 at a 10% limit: migration happens, and it is queue-aware (L258):
    no object of request q is evicted while an object of a later request
    q' > q (further back in the queue) stays resident on stage A's GPU.
    Checked by replaying each prefix of the trace and reading the oracle's
    resident set right after every op that evicted something."""
    ops = T.cfg5(2, requests=4, limit_frac=0.1, scale=64, layers=4)
    calib = C.b200_hgx(2)
    out = runner.run(ops, calib)
    assert out["records"][0]["op"] == "pool_limit"
    req_of = {}                                     # oid -> request (queue position)
    for r in out["records"]:
        if r["op"] == "alloc" and r["status"] == "OK":
            req_of[r["oid"]] = ops[r["i"]]["fn"]["wf"] - 500
    evicting = [r for r in out["records"] if r["victims"]]
    assert evicting, "10% pool limit must force migration"
    later_seen = 0
    for r in evicting:
        orc = runner.run(ops[:r["i"] + 1], calib)["oracle"]
        resident = [o for o in orc.objects.values() if o.loc == 0 and o.state == "SEALED"]
        for v in r["victims"]:
            q = req_of[v]
            later = [o.oid for o in resident if req_of.get(o.oid, -1) > q]
            assert not later, (r["i"], v, q, later)
            later_seen += q > 0
    # request 0's objects were spilled only while request 0 itself was being
    # produced; once request 1 exists, spills come from the queue tail
    assert later_seen > 0


@pytest.mark.parametrize("seed", range(40))
def test_random_traces_invariants(seed):
    rng = random.Random(seed)
    n = rng.choice([1, 2, 3, 4, 8])
    c = C.b200_hgx(n, shared_pairs=bool(seed % 2))
    ops = T.random_trace(rng, n, n_ops=150, max_n=5 * MiB, run_seed=seed)
    caps = [rng.choice([8, 16, 64]) * MiB for _ in range(n)]
    out = runner.run(ops, c, host_store_bytes=48 * MiB, pool_cap=caps)
    orc = out["oracle"]
    for r in out["records"]:
        if r["op"] in ("get", "get_into") and r["status"] == "OK":
            off = 0
            for ch in r["plan"]:                      # I1 tiling of [0, n)
                assert ch["offset"] == off
                off += ch["bytes"]
            assert off in (0, r["n"])
            if r.get("zero_copy"):
                assert r["plan"] == []                # zero copy moves no byte
    assert orc.host_used <= orc.H
    statuses = {r["status"] for r in out["records"]}
    assert statuses <= set(model.STATUS) and "OK" in statuses


def test_capacity_never_exceeded_by_reserve():
    """I4: with no pool_limit ops, used <= cap after EVERY op."""
    for s in range(10):
        ops = T.random_trace(random.Random(s), 2, n_ops=200, max_n=7 * MiB, limits=False, run_seed=s)
        caps = [10 * MiB, 6 * MiB]
        res = runner.run(ops, C.b200_hgx(2), host_store_bytes=1 << 30, pool_cap=caps)
        for r in res["records"]:
            assert all(u <= c for u, c in zip(r["used"], caps)), r
        # the caps are small enough that every trace really evicts (the bound is exercised)
        assert any(r["victims"] for r in res["records"]), s


# ---------------------------------------------------------------- proactive restore
def _fig11b_restore(restore):
    """Fig. 11(b) continued: "after the output of a1 is
    processed, the output of a2 is reloaded into GPU memory"."""
    return runner.run(_fig11b_restore_ops(), C.b200_hgx(1), pool_cap=[4 * MiB], restore=restore)


def _fig11b_restore_ops():
    b = T.Builder(3)
    a1, a2, a3, b1 = T.fn(1, 1, 0), T.fn(1, 2, 0), T.fn(1, 3, 0), T.fn(1, 4, 0)
    o1 = b.alloc(a1, MiB, consumers=1)
    b.seal(a1, o1)
    o2 = b.alloc(a2, MiB, consumers=1)
    b.seal(a2, o2)
    b.next_use(o1, 0)
    b.next_use(o2, 1)
    b.put(a3, MiB)                      # evicts O2 (queue-aware)
    g = b.get(b1, o1)                   # b1 processes a1's output (zero copy)
    b.release(b1, g)                    # ... and is done with it
    return b.ops


def test_fig11b_restore_after_a1_output_processed():
    out = _fig11b_restore(True)
    recs = out["records"]
    assert recs[6]["victims"] == [2]
    assert recs[-1]["restored"] == [2]             # a2's output reloaded
    orc = out["oracle"]
    assert orc.where(2) == 0 and orc.host_used == 0 and orc.used == [4 * MiB]
    # without restore the object stays on the host; restore moves, never changes, bytes
    out2 = _fig11b_restore(False)
    assert out2["records"][-1]["restored"] == [] and out2["oracle"].where(2) == model.HOST
    assert bytes(orc.objects[2].buf) == bytes(out2["oracle"].objects[2].buf)


def _restore_setup(hints, cap_after):
    """Four spilled 1-page objects (oids 1-4), then the limit is raised."""
    b = T.Builder(5)
    f = T.fn(1, 1, 0)
    refs = [b.put(f, MiB) for _ in range(4)]
    for r, h in zip(refs, hints):
        if h is not None:
            b.next_use(r, h)
    b.pool_limit(0, 0)                  # spill everything
    b.pool_limit(0, cap_after)
    out = runner.run(b.ops, C.b200_hgx(1), restore=True)
    return out["records"]


def test_restore_order_hinted_first_then_mru():
    # hints: oid1 -> 5, oid2 none, oid3 -> 2, oid4 none
    recs = _restore_setup([5, None, 2, None], 8 * MiB)
    assert sorted(recs[-2]["victims"]) == [1, 2, 3, 4]
    # queue head first among hinted (3 then 1), then most recently used (4, 2)
    assert recs[-1]["restored"] == [3, 1, 4, 2]


def test_restore_stops_at_cap():
    recs = _restore_setup([5, None, 2, None], 5 * MiB)    # room for 2 pages
    assert recs[-1]["restored"] == [3, 1]
    assert recs[-1]["used"] == [4 * MiB]


def test_restore_stops_at_first_misfit():
    """Strict priority: a small later object is not restored past a large
    earlier one that does not fit (R42)."""
    b = T.Builder(5)
    f = T.fn(1, 1, 0)
    big, small = b.put(f, 3 * MiB), b.put(f, MiB)
    b.next_use(big, 0)
    b.next_use(small, 1)
    b.pool_limit(0, 0)
    b.pool_limit(0, 2 * MiB)            # small fits, big (4 MiB) does not
    recs = runner.run(b.ops, C.b200_hgx(1), restore=True)["records"]
    assert recs[-1]["restored"] == [] and recs[-1]["used"] == [0]


def test_restore_respects_home_gpu():
    """Only objects migrated away from the GPU that gained room come back."""
    b = T.Builder(6)
    f0, f1 = T.fn(1, 1, 0), T.fn(1, 2, 1)
    b.put(f0, MiB)
    o2 = b.put(f1, MiB)
    b.pool_limit(0, 0)
    b.pool_limit(1, 0)
    b.pool_limit(0, 8 * MiB)
    recs = runner.run(b.ops, C.b200_hgx(2), restore=True)["records"]
    assert recs[-1]["restored"] == [1]
    del o2


@pytest.mark.parametrize("seed", range(12))
def test_restore_preserves_bytes_and_caps(seed):
    """Restore moves data, never changes it: every get/get_into that succeeds
    both with and without restore reads identical bytes; and restore never
    takes a pool above its cap (I4 holds after restore-only ops)."""
    rng = random.Random(100 + seed)
    n = rng.choice([1, 2, 4])
    c = C.b200_hgx(n)
    ops = T.random_trace(rng, n, n_ops=150, max_n=5 * MiB, run_seed=seed)
    caps = [rng.choice([8, 16]) * MiB for _ in range(n)]
    a = runner.run(ops, c, host_store_bytes=1 << 30, pool_cap=caps, restore=False)["records"]
    r = runner.run(ops, c, host_store_bytes=1 << 30, pool_cap=caps, restore=True)
    moved = 0
    caps = list(caps)
    prev = [0] * n
    for op, x, y in zip(ops, a, r["records"]):
        if op["op"] == "pool_limit" and 0 <= op["dev"] < n:
            caps[op["dev"]] = op["bytes"]
        if op["op"] == "refresh_cap" and 0 <= op["dev"] < n:
            caps[op["dev"]] = y["cap"]
        moved += len(y["restored"])
        if x["op"] in ("get", "get_into") and x["status"] == y["status"] == "OK":
            assert x.get("digest") == y.get("digest"), x["i"]
        if y["restored"] and y["op"] in ("release", "free", "get", "get_into"):
            # a GPU that grew (restore target) is within its cap (another may
            # sit above an unreachable cap with unevictable data, R34)
            assert all(u <= cp for u, cp, p in zip(y["used"], caps, prev) if u > p)
        prev = y["used"]
    assert moved > 0 or seed % 3 == 0     # most traces exercise restore


@pytest.mark.parametrize("restore", [False, True])
@pytest.mark.parametrize("hints", [False, True])
def test_cfg5_interleaved_drains(restore, hints):
    """Interleaved cfg5 (Fig. 18 setting): every op succeeds, the pools drain,
    and with queue hints + restore the head of the queue is reloaded."""
    ops = T.cfg5_interleaved(2, requests=6, window=3, limit_frac=0.3, scale=64, layers=8, hints=hints)
    out = runner.run(ops, C.b200_hgx(2), restore=restore)
    assert all(r["status"] == "OK" for r in out["records"])
    orc = out["oracle"]
    assert orc.used == [0, 0] and orc.host_used == 0 and not orc.objects
    restored = [o for r in out["records"] for o in r["restored"]]
    assert bool(restored) == (restore and hints)
    if restored:
        # restores follow consumption: each restored object belongs to a
        # request later than the one whose get_into released the room
        by_oid = {r["oid"]: ops[r["i"]]["fn"]["wf"] for r in out["records"] if r["op"] == "alloc"}
        for r in out["records"]:
            if r["op"] == "get_into" and r["restored"]:
                assert all(by_oid[o] > ops[r["i"]]["fn"]["wf"] for o in r["restored"])


def test_tenant_bytes_closed_form():
    """Per-tenant scheduled bytes per server kind (L193; grouter_tenant_stats):
    tenant 1 puts n1 from a CPU function toward GPU0 (H2D, striped over R(0))
    and a GPU1 function reads it (one NVLink copy); tenant 2's GPU function
    puts n2 by copy (an SM copy on its GPU) and a CPU function reads it (D2H).
    Zero-copy gets and the host-store memcpy move nothing scheduled."""
    n1, n2 = 5 * MiB + 123, 3 * MiB + 7
    b = T.Builder(9)
    o1 = b.put(T.fn(1, 1, model.HOST), n1, hint=0)
    g1 = b.get_into(T.fn(1, 2, 1), o1)
    z1 = b.get(T.fn(1, 3, 0), o1)                   # co-located: zero copy
    b.release(T.fn(1, 3, 0), z1)
    o2 = b.put(T.fn(2, 1, 1), n2)
    g2 = b.get(T.fn(2, 2, model.HOST), o2)
    b.release(T.fn(2, 2, model.HOST), g2)
    o3 = b.put(T.fn(3, 1, model.HOST), MiB)          # cFn -> host store: memcpy only
    b.get_into(T.fn(3, 2, model.HOST), o3)
    orc = runner.run(b.ops, C.b200_hgx(2, shared_pairs=False))["oracle"]
    assert orc.tenant_bytes == {(1, "h2d"): n1, (1, "copy"): n1, (2, "copy"): n2, (2, "d2h"): n2}
    # the H2D share really was striped over both uplinks, and sums to n1
    assert orc.link_bytes[("h2d", 0)] > 0 and orc.link_bytes[("h2d", 1)] > 0
    assert orc.link_bytes[("h2d", 0)] + orc.link_bytes[("h2d", 1)] == n1
    del g1


def test_host_centric_closed_form():
    """Ablation "UF off" (host_centric, R49; the host-centric passing of L90):
    a GPU0 object read by a GPU1 function crosses PCIe twice -- n bytes D2H
    on GPU0's engine, n bytes H2D on GPU1's, no SM copy -- while a same-GPU
    get stays zero copy and a same-GPU get_into stays an SM copy; bytes and
    every decision are those of the GPU-centric run."""
    n = 5 * MiB + 77
    b = T.Builder(4)
    o = b.put(T.fn(1, 1, 0), n)                       # gFn put by copy on GPU0 (SM copy)
    g1 = b.get_into(T.fn(1, 2, 1), o)                  # GPU1 reads it
    z = b.get(T.fn(1, 3, 0), o)                        # co-located: zero copy
    b.release(T.fn(1, 3, 0), z)
    b.get_into(T.fn(1, 4, 0), o)                       # same GPU into caller memory
    calib = C.b200_hgx(2, shared_pairs=False)
    hc = runner.run(b.ops, calib, host_centric=True, keep_bytes=True)
    gc = runner.run(b.ops, calib, keep_bytes=True)
    assert hc["oracle"].tenant_bytes == {(1, "copy"): 2 * n, (1, "d2h"): n, (1, "h2d"): n}
    assert gc["oracle"].tenant_bytes == {(1, "copy"): 3 * n}
    assert hc["oracle"].link_bytes == {("copy", 0): 2 * n, ("d2h", 0): n, ("h2d", 1): n}
    assert gc["oracle"].link_bytes == {("copy", 0): 3 * n}       # each copy crosses once (L165)
    for x, y in zip(hc["records"], gc["records"]):
        assert (x["status"], x.get("digest"), x["used"]) == (y["status"], y.get("digest"), y["used"])
    del g1


@pytest.mark.parametrize("seed", range(6))
def test_host_centric_changes_engines_only(seed):
    """On random traces the host-centric ablation (R49) changes which engines
    move the bytes and nothing else: statuses, placements, victims, pool
    usage and every delivered byte equal the GPU-centric run; per tenant, the
    SM-copy bytes it loses reappear exactly once on the D2H and once on the
    H2D engines."""
    rng = random.Random(800 + seed)
    n = rng.choice([2, 3, 4])
    calib = C.b200_hgx(n, shared_pairs=False)
    ops = T.random_trace(rng, n, n_ops=150, max_n=7 * MiB, run_seed=seed)
    caps = [rng.choice([8, 16, 64]) * MiB for _ in range(n)]
    kw = dict(host_store_bytes=1 << 30, pool_cap=caps)
    a = runner.run(ops, calib, **kw)
    b = runner.run(ops, calib, host_centric=True, **kw)
    for x, y in zip(a["records"], b["records"]):
        for k in ("status", "oid", "where", "victims", "used", "host_used", "digest"):
            assert x.get(k) == y.get(k), (x["i"], k)
    ta, tb = a["oracle"].tenant_bytes, b["oracle"].tenant_bytes
    for wf in {k[0] for k in list(ta) + list(tb)}:
        moved = ta.get((wf, "copy"), 0) - tb.get((wf, "copy"), 0)
        assert moved >= 0
        assert tb.get((wf, "d2h"), 0) - ta.get((wf, "d2h"), 0) == moved
        assert tb.get((wf, "h2d"), 0) - ta.get((wf, "h2d"), 0) == moved
