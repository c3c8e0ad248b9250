"""N > 1 plumbing of bench.py on CPU (world_size 2, gloo): pairing of
producer/consumer GPUs, descriptor exchange, max over ranks."""
import os
import socket

import pytest
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import bench
    descs = [bytes([rank, i]) * 8 for i in range(3)]        # stand-ins for export descriptors
    got = bench.exchange(descs, world)
    peer = bench.peer_of(rank, world)
    mx = bench.max_over_ranks(float(rank + 1), world)
    q.put((rank, peer, got[peer], mx, len(got)))
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_exchange_pairing_and_max(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(world))
    for p in ps:
        p.join(timeout=60)
    for rank, peer, peer_descs, mx, n in res:
        assert peer == (rank + 1) % world and peer != rank
        assert peer_descs == [bytes([peer, i]) * 8 for i in range(3)]
        assert mx == float(world) and n == world
    # the ring is a permutation: every GPU is a producer exactly once
    assert sorted(p for _, p, *_ in res) == list(range(world))


def test_single_rank_is_identity():
    import bench
    assert bench.exchange("x", 1) == ["x"]
    assert bench.max_over_ranks(3.5, 1) == 3.5


def test_bench_helpers():
    """bench.py's nearest-rank percentile (R26) and host description."""
    import bench
    xs = list(range(1, 101))
    assert bench.pct(xs, 50) == 50 and bench.pct(xs, 99) == 99 and bench.pct(xs, 100) == 100
    assert bench.pct([7], 99) == 7 and bench.pct([], 50) is None
    assert bench.pct([3, 1, 2], 50) == 2            # sorts its input
    cores, model = bench.host_info()
    assert cores >= 1 and (model is None or isinstance(model, str))
    assert bench.peer_of(3, 4) == 0 and bench.peer_of(0, 2) == 1
