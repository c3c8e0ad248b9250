"""Pins of oracle/poolsize.py and its use in the model (PAPER.md L250-L256,
Fig. 11a; reading R44): nearest-rank p99 by hand, a worked trace whose
reservation, window expiry and floor are computed in the comments, the
sliding history's rank boundary, and per-GPU / per-function separation."""
from oracle import model, poolsize, runner
from synth import calib as C
from synth import traces as T

MiB = 1 << 20
MS = 10 ** 6


def test_p99_nearest_rank():
    assert poolsize.p99([]) == 0
    assert poolsize.p99([7]) == 7
    assert poolsize.p99([3, 1, 2]) == 3                  # ceil(2.97) = 3rd smallest
    assert poolsize.p99(list(range(1, 101))) == 99       # ceil(99.0) = 99th
    assert poolsize.p99(list(range(1, 201))) == 198      # ceil(198.0) = 198th
    assert poolsize.p99(list(range(1, 102))) == 100     # ceil(99.99) = 100th


def _worked(floor=MiB):
    b = T.Builder(1)
    f = T.fn(1, 1, 0)
    for i in range(4):
        b.tick(i * 10 * MS)
        b.put(f, 3 * MiB)            # charge 4 MiB each, never consumed
    return b


def test_worked_reservation_and_expiry():
    """Arrivals 0, 10, 20, 30 ms -> intervals [10, 10, 10] ms -> R_window = 10 ms.
    Sizes charge(3 MiB) = 4 MiB -> R_size = 4 MiB.  Concurrency 1, 2, 3, 4 ->
    R_con = ceil(3.96) = 4th smallest = 4.  Data_size = 16 MiB."""
    b = _worked()
    b.tick(40 * MS)                  # 30 + 10 ms: still inside the window
    b.tick(40 * MS + 1)              # past it: the reservation is reclaimed
    recs = runner.run(b.ops, C.b200_hgx(1), pool_floor=MiB, targets=True)["records"]
    # one arrival: R_window 0, active at its own time (t <= 0 + 0): 4 MiB * 1
    assert recs[1]["pool_target"] == [4 * MiB]
    assert recs[-2]["pool_target"] == [16 * MiB]
    assert recs[-1]["pool_target"] == [MiB]           # floor only
    # after the 2nd put: intervals [10 ms], R_size 4 MiB, R_con = 2 -> 8 MiB, active
    assert recs[3]["pool_target"] == [8 * MiB]


def test_floor_and_cap_clamp():
    b = _worked()
    b.tick(35 * MS)
    recs = runner.run(b.ops, C.b200_hgx(1), pool_floor=32 * MiB, targets=True)["records"]
    assert recs[-1]["pool_target"] == [32 * MiB]      # max(floor, 16 MiB)
    h = poolsize.FuncHist()
    for i, con in enumerate([1, 2, 3, 4]):
        h.observe(i * MS, 4 * MiB, con)
    assert poolsize.target({1: h}, 3 * MS, 10 * MiB, MiB) == 10 * MiB   # min(cap, 16 MiB)
    assert poolsize.target({1: h}, 3 * MS, 1 << 40, MiB) == 16 * MiB


def test_functions_and_gpus_are_separate():
    b = T.Builder(2)
    f, g, h = T.fn(1, 1, 0), T.fn(1, 2, 0), T.fn(1, 1, 1)
    for i in range(3):
        b.tick(i * MS)
        b.put(f, MiB)               # f: 2 MiB x con (1,2,3) -> 2 MiB * 3 = 6 MiB
        b.put(g, 5 * MiB)           # g: 6 MiB x con (1,2,3) -> 18 MiB
        b.put(h, MiB)               # same ids on GPU 1: its own pool
        b.put(T.fn(1, 1, model.HOST), 9 * MiB)   # host-resident: no sample
    b.tick(2 * MS)
    recs = runner.run(b.ops, C.b200_hgx(2), pool_floor=MiB, targets=True)["records"]
    assert recs[-1]["pool_target"] == [24 * MiB, 6 * MiB]


def test_consumption_lowers_concurrency_samples():
    """Concurrency counts objects still holding storage: a consumer that
    drains each output before the next put keeps R_con = 1."""
    b = T.Builder(3)
    f, c = T.fn(1, 1, 0), T.fn(1, 2, 0)
    for i in range(5):
        b.tick(i * MS)
        o = b.put(f, MiB, consumers=1)
        b.get_into(c, o)
    b.tick(4 * MS)
    recs = runner.run(b.ops, C.b200_hgx(1), pool_floor=0, targets=True)["records"]
    assert recs[-1]["pool_target"] == [2 * MiB]


def test_sliding_history_rank_boundary():
    """HIST = 1024 sizes: the p99 rank is ceil(0.99 * 1024) = 1014, so up to
    10 large samples among the last 1024 do not move R_size, 11 do."""
    h = poolsize.FuncHist()
    for i in range(2000):
        h.observe(i, 2 * MiB, 1)
    for i in range(10):
        h.observe(3000 + i, 100 * MiB, 1)
    assert h.data_size() == 2 * MiB
    h.observe(4000, 100 * MiB, 1)
    assert h.data_size() == 100 * MiB


def test_sizing_trace_targets_bounded():
    """On random sizing traces the target stays within [min(floor, cap), cap]
    and drops back to the floor after an idle gap longer than every window."""
    import random
    for seed in range(5):
        rng = random.Random(seed)
        ops = T.sizing_trace(rng, 2)
        ops.append({"op": "tick", "t_ns": 10 ** 15})
        recs = runner.run(ops, C.b200_hgx(2), pool_floor=8 * MiB, targets=True)["records"]
        for r in recs:
            assert all(8 * MiB <= x for x in r["pool_target"])
        assert recs[-1]["pool_target"] == [8 * MiB, 8 * MiB]
        assert any(x > 8 * MiB for r in recs for x in r["pool_target"])
