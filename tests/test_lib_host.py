"""Host-side (no GPU) tests of libgrouter.so: exported ABI, and parity of the
C++ planner and stride scheduler against the oracle (SURVEY §7 step 1:
replay-mode parity on synthetic calibrations for 1/2/4/8 GPUs).

These call only GPU-free entry points (GROUTER_PLAN_ONLY contexts and the
standalone scheduler)."""
import os
import random
import re

import pytest

from oracle import routes as oroutes
from oracle import splitter as osplit
from oracle import stride as ostride
from paper_conf_eurosys_wulywdyfwwj26_b200 import _build
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G
from synth import calib as C

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module", autouse=True)
def built():
    _build.build()
    G.load()


def _declared():
    names = set()
    for h in ("grouter.h", "grouter_testing.h"):
        txt = open(os.path.join(ROOT, "include", h)).read()
        txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
        names |= set(re.findall(r"\b(grouter_[a-z0-9_]+)\s*\(", txt))
    return names


def test_every_declared_symbol_is_exported():
    lib = G.load()
    declared = _declared()
    assert len(declared) >= 30
    for name in declared:
        assert hasattr(lib, name), name
        assert name in G.SIGNATURES, f"binding lacks {name}"
    # nothing but the ABI leaks out of the library (static cudart is hidden)
    out = os.popen(f"nm -D --defined-only {G.LIB_PATH}").read().split()
    exported = {w for w in out if w.startswith("grouter_") or w.startswith("cuda")}
    assert exported == declared


def _plan_ctx(calib, **kw):
    return G.Ctx(G.config_from_calib(calib, flags=G.PLAN_ONLY | kw.pop("flags", 0), **kw))


def _oracle_plan(calib, src, dst, n, multipath=True):
    if n == 0 or (src == -1 and dst == -1):
        return []
    if src == -1:
        p = osplit.plan_h2d(calib, dst, n, multipath)
    else:
        p = osplit.plan_single(n, src)
    return [(c["offset"], c["bytes"], c["path"], c["route_gpu"]) for c in p]


SIZES = [0, 1, 15, 16, 17, 4095, 4096, 4097, 2**21 - 1, 2**21, 2**21 + 1, 38_535_168,
         39_321_600, 602_112, 33_554_432, 67_108_864, 1 << 30]


@pytest.mark.parametrize("topo", ["pairs8", "solo8", "solo4", "solo2", "one", "fig5a"])
def test_plan_parity_config_topologies(topo):
    calib = {"pairs8": C.b200_hgx(8), "solo8": C.b200_hgx(8, shared_pairs=False),
             "solo4": C.b200_hgx(4, shared_pairs=False), "solo2": C.b200_hgx(2, shared_pairs=False),
             "one": C.b200_hgx(1), "fig5a": C.fig5a()}[topo]
    with _plan_ctx(calib) as ctx:
        n = calib["n_gpus"]
        for d in range(n):
            assert ctx.route_set(d)[1] == oroutes.route_set(calib, d)
        for src in [-1] + list(range(n)):
            for dst in [-1] + list(range(n)):
                for size in SIZES:
                    st, got = ctx.plan(src, dst, size)
                    assert st == G.OK
                    assert got == _oracle_plan(calib, src, dst, size), (src, dst, size)


@pytest.mark.parametrize("seed", range(60))
def test_plan_parity_random_calibrations(seed):
    rng = random.Random(seed)
    n = rng.choice([1, 2, 3, 4, 5, 8])
    calib = C.random_calib(rng, n)
    chunk = rng.choice([1 << 20, 2 << 20, 4 << 20])
    with _plan_ctx(calib, chunk_bytes=chunk) as ctx:
        for d in range(n):
            assert ctx.route_set(d)[1] == oroutes.route_set(calib, d)
            for _ in range(6):
                size = rng.choice([rng.randint(0, 1 << 22), rng.randint(0, 1 << 31), rng.choice(SIZES)])
                st, got = ctx.plan(-1, d, size)
                exp = osplit.plan_h2d(calib, d, size, C=chunk)
                assert got == [(c["offset"], c["bytes"], c["path"], c["route_gpu"]) for c in exp]


def test_no_multipath_flag():
    calib = C.b200_hgx(8, shared_pairs=False)
    with _plan_ctx(calib, flags=G.NO_MULTIPATH) as ctx:
        assert ctx.route_set(3)[1] == [3]
        st, got = ctx.plan(-1, 3, 1 << 30)
        assert got == _oracle_plan(calib, -1, 3, 1 << 30, multipath=False)


def test_plan_bad_arguments():
    with _plan_ctx(C.b200_hgx(2)) as ctx:
        assert ctx.plan(-1, 2, 10)[0] == G.EINVAL
        assert ctx.plan(-3, 0, 10)[0] == G.EINVAL
        assert ctx.route_set(5)[0] == G.EINVAL
        # data-path calls are refused by a planner-only context (no CPU fallback)
        st, _ = ctx.put(G.fn(1, 1, -1), 0, 0)
        assert st == G.EINVAL


@pytest.mark.parametrize("seed", range(25))
def test_sched_parity_with_oracle(seed):
    rng = random.Random(seed)
    w = {t: rng.choice([1, 2, 3, 4, 8]) for t in range(1, rng.randint(2, 7))}
    lib, orc = G.Sched(5), ostride.StrideServer()
    for t, x in w.items():
        lib.set_weight(t, x)
    cid = 0
    for step in range(300):
        if rng.random() < 0.55:
            for _ in range(rng.randint(1, 8)):
                t = rng.choice(list(w))
                nb = rng.randint(1, 4 << 20)
                lib.enqueue(t, cid, nb)
                orc.enqueue(t, cid, nb)
                cid += 1
        else:
            a = lib.dispatch()
            b = orc.dispatch(w.get)
            if b is None:
                assert a is None
            else:
                assert a is not None
                assert (a[0], a[1], a[2]) == (b[0], b[1], b[2])
                assert a[3] == orc.pass_[b[0]]


@pytest.mark.parametrize("seed", range(25))
def test_sched_account_solo_equals_queued_dispatch(seed):
    """The fast paths (an idle server's direct launch / copy, engine.cpp
    fast_direct, fast_ce) skip the queues but apply Stride::account_solo:
    the same passes and virtual time as the oracle's stride scheduler
    dispatching that tenant's chunks alone.  Checked by what it decides:
    after a solo transfer by one tenant (queued and dispatched in the
    oracle, accounted in the library), a contended workload of several
    tenants dispatches identically, with identical passes."""
    rng = random.Random(700 + seed)
    w = {t: rng.choice([1, 2, 3, 4, 8]) for t in range(1, rng.randint(2, 6))}
    C_ = rng.choice([2 << 20, 1 << 20, 4096 * rng.randint(1, 512)])
    lib, orc = G.Sched(5), ostride.StrideServer()
    for t, x in w.items():
        lib.set_weight(t, x)
    cid = 0
    for rep in range(rng.randint(1, 4)):              # solo transfers, possibly by several tenants in turn
        t = rng.choice(list(w))
        n = rng.randint(1, 40 << 20)
        full, last = divmod(n, C_)
        for b in [C_] * full + ([last] if last else []):
            orc.enqueue(t, cid, b)
            cid += 1
        while orc.dispatch(w.get) is not None:
            pass
        assert lib.account_solo(t, n, C_) == G.OK
    for t in w:                                        # then contention
        for _ in range(rng.randint(1, 12)):
            nb = rng.randint(1, C_)
            lib.enqueue(t, cid, nb)
            orc.enqueue(t, cid, nb)
            cid += 1
    while True:
        a, b = lib.dispatch(), orc.dispatch(w.get)
        if b is None:
            assert a is None
            break
        assert (a[0], a[1], a[2]) == (b[0], b[1], b[2])
        assert a[3] == orc.pass_[b[0]]


@pytest.mark.parametrize("seed", range(30))
def test_slo_weights_parity_with_oracle(seed):
    """grouter_slo_weights (C) == oracle/slo.weights on random SLO sets,
    including oversubscribed ones and 64-bit-overflowing data sizes."""
    import random
    from oracle import slo as oslo
    rng = random.Random(seed)
    s = {}
    for _ in range(rng.randint(1, 8)):
        wf = rng.randint(1, 50)
        slo_ns = rng.choice([1, 7, 10 ** 6, 5 * 10 ** 7, 10 ** 9, 3 * 10 ** 10])
        infer = rng.randint(0, slo_ns - 1)
        data = rng.choice([1, 4096, 38_535_168, rng.randint(1, 1 << 40), (1 << 63) + rng.randint(0, 1 << 20)])
        s[wf] = (data, slo_ns, infer)
    bw = rng.choice([0, 55 * 10 ** 9, 8 * 55 * 10 ** 9, 1 << 62])
    assert G.slo_weights(s, bw) == oslo.weights(s, bw)


def test_slo_weights_rejects_infeasible():
    with pytest.raises(RuntimeError):
        G.slo_weights({1: (10, 5, 5)}, 10 ** 9)


@pytest.mark.parametrize("topo", ["pairs8", "solo4", "fig5a", "one"])
@pytest.mark.parametrize("multipath", [True, False])
def test_d2h_striped_plan_parity(topo, multipath):
    """GROUTER_D2H_MULTIPATH (L178 gFn-host, R45): GPU -> host plans equal
    oracle.splitter.plan_d2h; other directions are unchanged."""
    calib = {"pairs8": C.b200_hgx(8), "solo4": C.b200_hgx(4, shared_pairs=False),
             "fig5a": C.fig5a(), "one": C.b200_hgx(1)}[topo]
    flags = G.D2H_MULTIPATH | (0 if multipath else G.NO_MULTIPATH)
    with _plan_ctx(calib, flags=flags) as ctx:
        for src in range(calib["n_gpus"]):
            for size in SIZES:
                st, got = ctx.plan(src, -1, size)
                exp = osplit.plan_d2h(calib, src, size, multipath)
                assert got == [(c["offset"], c["bytes"], c["path"], c["route_gpu"]) for c in exp]
                assert ctx.plan(-1, src, size)[1] == _oracle_plan(calib, -1, src, size, multipath=multipath)


def test_fig5a_gfn_host_routes():
    """Fig. 5(a) (L178): "data from GPU1 is first routed via NVLink to peer
    GPUs (GPU3, GPU5, and GPU7), which concurrently stage it to host memory";
    GPU2 shares GPU1's PCIe switch and is excluded (0-based: GPU0 -> 2, 4, 6)."""
    calib = C.fig5a()
    p = osplit.plan_d2h(calib, 0, 1 << 30)
    assert sorted({c["route_gpu"] for c in p}) == [0, 2, 4, 6]


# ------------------------------------------------------------------ Alg. 1 planner parity
def _alg1_ops(rng, n_gpus, steps=40):
    ops, live, nxt = [], [], 1
    for _ in range(steps):
        if live and rng.random() < 0.3:
            f = live.pop(rng.randrange(len(live)))
            ops.append(("release", f))
        else:
            gs, gd = rng.sample(range(n_gpus), 2)
            ops.append(("select", nxt, gs, gd))
            live.append(nxt)
            nxt += 1
    return ops


@pytest.mark.parametrize("seed", range(40))
def test_alg1_planner_parity(seed):
    """grouter_paths_* (C++) == oracle.alg1.PathTable op by op: each selected
    path list, the full allocation table after every op, and the NVLink chunk
    plan of every live function."""
    import random
    from oracle import alg1
    rng = random.Random(seed)
    kind = seed % 4
    if kind == 0:
        topo, ng = C.dgx_v100_topo(), 8
    elif kind == 1:
        topo, ng = C.nvswitch_topo(8), 8
    else:
        ng = rng.choice([3, 4, 5, 6, 8])
        topo = C.random_topo(rng, ng)
    H = rng.choice([2, 3, 4])
    orc, lib = alg1.PathTable(topo, ng, max_edges=H), G.Paths(topo, ng, max_edges=H)
    try:
        for op in _alg1_ops(rng, ng):
            if op[0] == "release":
                orc.release(op[1])
                assert lib.release(op[1]) == G.OK
            else:
                _, f, gs, gd = op
                exp, _ = orc.select(f, gs, gd)
                st, got = lib.select(f, gs, gd)
                assert st == G.OK and got == exp, (op, got, exp)
            assert lib.table() == orc.table()
            for f in sorted({a[0] for a in orc.alloc}):
                n = rng.choice([1, 4096, 38_535_168, 1 << 30])
                exp = alg1.nvl_plan([(a[1], a[2]) for a in orc.paths_of(f)], n, ng, 20_000_000, 2 << 20)
                got = lib.plan(f, n, 2 << 20, 20_000_000)
                assert got == [(c["offset"], c["bytes"], c["path"], c["route_gpu"]) for c in exp]
    finally:
        lib.close()


def test_alg1_planner_bad_arguments():
    t = C.dgx_v100_topo()
    p = G.Paths(t, 8)
    try:
        assert p.select(1, 0, 0)[0] == G.EINVAL
        assert p.select(1, 0, 9)[0] == G.EINVAL
        assert p.select(1, 0, 3)[0] == G.OK
        assert p.select(1, 0, 2)[0] == G.ESTATE        # release first
        assert p.release(1) == G.OK and p.table() == []
    finally:
        p.close()
    with pytest.raises(G.GrouterError):
        G.Paths([[0] * 40 for _ in range(40)], 8)


def test_tenant_rate_monitor_host():
    """grouter_tenant_rate (L197) on a planner-only context: no dispatch yet,
    so rates are 0; Rate_least follows the closed form of L195 (R43) once an
    SLO is declared (same arithmetic as the oracle's slo.rate_least);
    windows outside [1 ms, 10 s] are rejected."""
    from oracle import slo as oslo
    ctx = G.Ctx(G.config_from_calib(C.b200_hgx(2), flags=G.PLAN_ONLY))
    try:
        assert ctx.tenant_rate(7, 10_000_000) == (0, 0, False)
        G.check(ctx.set_tenant_slo(7, 38_535_168, 50_000_000, 0), "slo")
        r, least, bl = ctx.tenant_rate(7, 10_000_000)
        assert (r, bl) == (0, False)
        assert least == oslo.rate_least(38_535_168, 50_000_000, 0) == 770_703_360
        G.check(ctx.set_tenant_slo(8, 1000, 3_000_000_000, 1), "slo")
        assert ctx.tenant_rate(8, 10_000_000)[1] == oslo.rate_least(1000, 3_000_000_000, 1) == 334
        for bad in (999_999, 10_000_000_001):
            with pytest.raises(G.GrouterError):
                ctx.tenant_rate(7, bad)
    finally:
        ctx.close()


@pytest.mark.parametrize("topo", ["pairs8", "fig5a"])
def test_no_topology_flag(topo):
    """Ablation "TA off" (GROUTER_NO_TOPOLOGY, Fig. 16; reading R48): the
    library's route sets and plans equal the oracle's on the same calibration
    with every GPU its own uplink group -- so on the L178 example GPU2 (the
    switch partner of GPU1) becomes a route of GPU1, which TA excludes."""
    calib = {"pairs8": C.b200_hgx(8), "fig5a": C.fig5a()}[topo]
    n = calib["n_gpus"]
    flat = dict(calib, uplink_groups=[[i] for i in range(n)])
    with _plan_ctx(calib, flags=G.NO_TOPOLOGY) as ctx:
        for d in range(n):
            assert ctx.route_set(d)[1] == oroutes.route_set(flat, d) == list(range(n)[d:d + 1]) + \
                [r for r in range(n) if r != d]
            for size in (2**21 + 1, 38_535_168, 1 << 30):
                assert ctx.plan(-1, d, size)[1] == _oracle_plan(flat, -1, d, size)
    with _plan_ctx(calib) as ctx:                      # TA on: the switch partner is excluded
        assert 1 not in ctx.route_set(0)[1]
