"""Pins of oracle/slo.py (reading R43).

Hand-computed values (arithmetic written out in the comments) and the
property the allocation exists for: when sum Rate_least <= BW_all, stride
scheduling with the derived weights gives every backlogged tenant at least
its Rate_least share of the link (up to one batch)."""
import pytest

from oracle import model, runner, slo
from oracle.stride import StrideServer
from synth import calib as C
from synth import traces as T

MiB = 1 << 20


def test_rate_least_closed_form():
    # 38,535,168 B within (100 ms - 50 ms): 38,535,168 / 0.05 s = 770,703,360 B/s exactly
    assert slo.rate_least(38_535_168, 100_000_000, 50_000_000) == 770_703_360
    # 100 MB within 0.5 s = 200,000,000 B/s
    assert slo.rate_least(100_000_000, 1_000_000_000, 500_000_000) == 200_000_000
    # rounds up: 1 B within 3 ns = 333,333,333.33 B/s -> 333,333,334
    assert slo.rate_least(1, 3, 0) == 333_333_334
    with pytest.raises(ValueError):
        slo.rate_least(1, 5, 5)


def test_worked_allocation():
    s = {7: (38_535_168, 100_000_000, 50_000_000), 9: (100_000_000, 1_000_000_000, 500_000_000)}
    # Rate_idle = 2,000,000,000 - (770,703,360 + 200,000,000) = 1,029,296,640
    assert slo.rate_idle(2_000_000_000, [770_703_360, 200_000_000]) == 1_029_296_640
    # tightest SLO is tenant 7 (100 ms): 770,703,360 + 1,029,296,640 = 1,800,000,000
    assert slo.allocate(s, 2_000_000_000) == {7: 1_800_000_000, 9: 200_000_000}
    # weights in MiB/s, rounded up: 1.8e9 / 1,048,576 = 1716.61 -> 1717; 2e8 / 1,048,576 = 190.73 -> 191
    assert slo.weights(s, 2_000_000_000) == {7: 1717, 9: 191}


def test_oversubscribed_no_idle():
    s = {1: (10 * MiB, 10_000_000, 0), 2: (20 * MiB, 10_000_000, 0)}
    # Rate_least: 10 MiB / 10 ms = 1,048,576,000 B/s; 20 MiB -> 2,097,152,000; sum 3.1e9 > 1e9
    assert slo.rate_idle(1_000_000_000, [1_048_576_000, 2_097_152_000]) == 0
    assert slo.weights(s, 1_000_000_000) == {1: 1000, 2: 2000}


def test_tightest_tie_goes_to_lower_id():
    s = {5: (MiB, 10_000_000, 0), 3: (MiB, 10_000_000, 0)}
    a = slo.allocate(s, 10 ** 9)
    assert a[3] > a[5] and a[5] == slo.rate_least(MiB, 10_000_000, 0)


@pytest.mark.parametrize("seed", range(6))
def test_weights_meet_rate_least(seed):
    """Drain a backlog of equal chunks from every tenant with the derived
    weights; over any prefix where all stay backlogged, tenant t's byte share
    times BW_all >= Rate_least_t minus one batch (the stride bound)."""
    import random
    rng = random.Random(seed)
    bw_all = 55 * 10 ** 9
    s = {}
    for wf in range(1, rng.randint(2, 6) + 1):
        slo_ns = rng.choice([50, 100, 200, 400]) * 10 ** 6
        infer = slo_ns // rng.choice([2, 3, 4])
        s[wf] = (rng.randint(1, 400) * MiB, slo_ns, infer)
    least = {wf: slo.rate_least(*v) for wf, v in s.items()}
    if sum(least.values()) > bw_all:
        pytest.skip("oversubscribed draw")
    w = slo.weights(s, bw_all)
    srv = StrideServer()
    chunk = 2 * MiB
    n = 2000
    for wf in s:
        for i in range(n):
            srv.enqueue(wf, i, chunk)
    got = {wf: 0 for wf in s}
    total = 0
    for _ in range(n // 5):
        t, ids, nb = srv.dispatch(lambda x: w[x])
        got[t] += nb
        total += nb
    for wf in s:
        # share * BW_all >= Rate_least - slack of one batch per tenant
        slack = 5 * chunk * len(s) * bw_all // total
        assert got[wf] * bw_all // total + slack >= least[wf], (wf, got, least)
    t = slo.tightest(s)
    assert all(got[t] >= got[x] * least[t] // least[x] for x in s if x != t)


def test_model_set_slo_reweights_everyone():
    calib = C.b200_hgx(2)
    bw = sum(calib["h2d_Bps"][:2])
    o = model.Oracle(calib)
    assert o.set_slo(1, 38_535_168, 100_000_000, 50_000_000)[0] == model.OK
    assert o.weight_of(1) == slo.weights({1: (38_535_168, 100_000_000, 50_000_000)}, bw)[1]
    assert o.set_slo(2, 100_000_000, 1_000_000_000, 500_000_000)[0] == model.OK
    exp = slo.weights({1: (38_535_168, 100_000_000, 50_000_000), 2: (100_000_000, 1_000_000_000, 500_000_000)}, bw)
    assert (o.weight_of(1), o.weight_of(2)) == (exp[1], exp[2])
    assert o.set_slo(3, 1, 5, 5)[0] == model.EINVAL
    assert o.set_weight(1, 4)[0] == model.OK and o.weight_of(1) == 4 and 1 not in o.slos
    assert o.set_slo(2, 0, 0, 0)[0] == model.OK and o.weight_of(2) == 1


def test_slo_trace_runs():
    b = T.Builder(11)
    b.slo(1, 38_535_168, 100_000_000, 50_000_000)
    b.slo(2, 100_000_000, 1_000_000_000, 500_000_000)
    for wf in (1, 2):
        b.put(T.fn(wf, 1, model.HOST), 5 * MiB, hint=0)
    recs = runner.run(b.ops, C.b200_hgx(1))["records"]
    assert [r["status"] for r in recs] == ["OK"] * 4


def test_cfg4_slo_trace_weights():
    """cfg4 with SLO tenants: weights follow R43, are recomputed when tenant
    100 drops its SLO, and an explicit weight replaces tenant 101's SLO."""
    ops = T.cfg4(2, rounds=2, scale=64, slos=T.CFG4_SLOS)
    out = runner.run(ops, C.b200_hgx(2))
    assert all(r["status"] == "OK" for r in out["records"])
    orc = out["oracle"]
    bw = sum(C.b200_hgx(2)["h2d_Bps"][:2])
    rest = {100 + t: v for t, v in enumerate(T.CFG4_SLOS) if t >= 2}
    exp = slo.weights(rest, bw)
    assert {wf: orc.weight_of(wf) for wf in rest} == exp
    assert orc.weight_of(100) == 1 and orc.weight_of(101) == 3
    # tightest remaining SLO is tenant 102 (30 ms): it holds the idle bandwidth
    assert max(exp, key=exp.get) == 102
