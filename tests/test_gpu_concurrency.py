"""Concurrent callers (§8(b): "All calls are thread-safe"): several threads,
one workflow each, drive put / alloc+seal / get / get_into / release / free
at once on three logical GPUs of one B200, under pool caps small enough that
eviction, spill-on-arrival and proactive restore (striped) run concurrently
with the copies.  Placement decisions depend on the interleaving, so what is
checked is what holds under any interleaving: every successful get reads
exactly the bytes that were put (get(put(x)) == x, the O11 payload, checked
in full on the device or on the host), failures are only ENOMEM, and once
every object is gone the pools and the host store drain to zero (I6)."""
import ctypes
import random
import threading

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G  # noqa: E402
from synth import calib as C  # noqa: E402
from synth.payload import payload  # noqa: E402

MiB = 1 << 20
K = 3          # logical GPUs
THREADS = 8
OPS = int(__import__("os").environ.get("GR_STRESS_OPS", "100"))


def _consume(ctx, t, wf, item, rng, streams, dev):
    """Reads an object put earlier (FIFO per thread) and checks its bytes."""
    kind, oid, seed, n = item
    if kind == "host_put":          # gFn on a random GPU get_into's it
        d = rng.randrange(K)
        st, nn = ctx.get_into(G.fn(wf, 2, d), oid, dev.data_ptr(), n, streams[d].cuda_stream)
        G.check(st, "get_into")
        streams[d].synchronize()
        st, bad, first = G.test_verify(dev.data_ptr(), n, seed, 0, 0)
        assert st == 0 and bad == 0, (t, "put/get_into", n, bad, first)
    else:                           # a cFn reads the gFn's output into a host lease
        st, ptr, nn = ctx.get(G.fn(wf, 3, G.HOST), oid, 0)
        if st == G.ENOMEM:          # host store momentarily full
            G.check(ctx.free(G.fn(wf, 1, 0), oid), "free")
            return False
        G.check(st, "get")
        if n:
            back = np.ctypeslib.as_array((ctypes.c_uint8 * n).from_address(ptr))
            assert np.array_equal(back, payload(seed, n)), (t, "alloc/get", n)
        if ptr:                     # n = 0: no lease to release (R36)
            G.check(ctx.release(G.fn(wf, 3, G.HOST), oid, ptr, 0), "release")
    return True


def _client(ctx, t, errors, counts, rep=0):
    try:
        rng = random.Random(500 + t + 1000 * rep)
        torch.cuda.set_device(0)
        streams = [torch.cuda.Stream() for _ in range(K)]
        host = torch.empty(6 * MiB + 64, dtype=torch.uint8, pin_memory=True)
        dev = torch.empty(6 * MiB + 64, dtype=torch.uint8, device="cuda")
        wf = 100 + t
        fifo = []                   # objects put and not yet consumed (keeps pools under pressure)
        for i in range(OPS):
            n = rng.choice([0, 4096, 12345, 2 * MiB - 1, 2 * MiB + 1, rng.randint(1, 6 * MiB)])
            seed = 10_000 * t + i
            g = rng.randrange(K)
            s = streams[g]
            pat = rng.randrange(3)
            if pat == 0:            # cFn put from pinned host, hint g (striped H2D), 1 consumer
                host[:n].numpy()[:] = payload(seed, n)
                st, oid = ctx.put(G.fn(wf, 1, G.HOST), host.data_ptr(), n, g, 1)
                if st == G.ENOMEM:
                    counts["enomem"] += 1
                    continue
                G.check(st, "put")
                fifo.append(("host_put", oid, seed, n))
            elif pat == 1:          # gFn alloc + fill + seal on g, 1 consumer
                st, buf, oid = ctx.alloc(G.fn(wf, 1, g), n, G.NOHINT, 1)
                if st == G.ENOMEM:
                    counts["enomem"] += 1
                    continue
                G.check(st, "alloc")
                if n:
                    G.check(G.test_fill(buf, n, seed, 0, s.cuda_stream), "fill")
                G.check(ctx.seal(G.fn(wf, 1, g), oid, s.cuda_stream), "seal")
                fifo.append(("alloc", oid, seed, n))
            else:                   # gFn put by copy on g -> zero-copy get on g -> release -> free
                if n:
                    G.check(G.test_fill(dev.data_ptr(), n, seed, 0, s.cuda_stream), "fill")
                st, oid = ctx.put(G.fn(wf, 1, g), dev.data_ptr(), n, G.NOHINT, 0, s.cuda_stream)
                if st == G.ENOMEM:
                    counts["enomem"] += 1
                    continue
                G.check(st, "put")
                st, ptr, nn = ctx.get(G.fn(wf, 2, g), oid, s.cuda_stream)
                if st == G.ENOMEM:
                    counts["enomem"] += 1
                    G.check(ctx.free(G.fn(wf, 1, g), oid), "free")
                    continue
                G.check(st, "get")
                s.synchronize()
                if n:
                    st, bad, first = G.test_verify(ptr, n, seed, 0, 0)
                    assert st == 0 and bad == 0, (t, i, "put/get", n, bad, first)
                if ptr:
                    G.check(ctx.release(G.fn(wf, 2, g), oid, ptr, s.cuda_stream), "release")
                G.check(ctx.free(G.fn(wf, 1, g), oid), "free")
            counts["ok"] += 1
            while len(fifo) > 4:
                _consume(ctx, t, wf, fifo.pop(0), rng, streams, dev)
        while fifo:
            _consume(ctx, t, wf, fifo.pop(0), rng, streams, dev)
        for st_ in streams:
            st_.synchronize()
    except BaseException as e:  # surfaced by the main thread
        errors.append(f"thread {t}: {type(e).__name__}: {e}")


@pytest.mark.parametrize("rep", range(2))
# FORCE_REMOTE: the cross-GPU gets take a physical pair's dispatch (pulls <= 4 MiB, pushes
# from the source's copy server, R55 / R56) while other threads evict, spill and copy
@pytest.mark.parametrize("flags", [0, G.RESTORE | G.STRIPED_MIGRATION, G.D2H_MULTIPATH | G.NO_POOL,
                                   G.FORCE_REMOTE | G.RESTORE])
def test_concurrent_clients(flags, rep):
    calib = C.virtual(K)
    ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=256 * MiB, pool_cap=[24 * MiB] * K,
                                    pool_floor_bytes=16 * MiB, flags=flags))
    errors, counts = [], {"ok": 0, "enomem": 0}
    try:
        ths = [threading.Thread(target=_client, args=(ctx, t, errors, counts, rep)) for t in range(THREADS)]
        for th in ths:
            th.start()
        for th in ths:
            th.join(timeout=300)
        assert not any(th.is_alive() for th in ths), "a client thread hung"
        assert not errors, errors[:3]
        assert counts["ok"] > THREADS * OPS // 2, counts
        G.check(ctx.sync(), "sync")
        st = ctx.stats()
        assert [st.used[g] for g in range(K)] == [0] * K and st.host_used == 0, \
            ([st.used[g] for g in range(K)], st.host_used)
        assert st.spill_count > 0, "the caps should force concurrent evictions"
        if flags & G.RESTORE:
            assert st.restore_count > 0
    finally:
        ctx.close()


def test_pool_growth_without_the_lock_under_concurrency():
    """Puts that must grow the pool (a cold pool, no pre-warm floor) from
    several threads at once: their segment creation runs with the context
    lock released (pool.cpp dev_alloc), so other callers and the dispatch
    thread proceed meanwhile.  Every object reads back its own bytes, the
    mapping covers what is resident, and the pool drains to zero."""
    calib = C.b200_hgx(1)
    calib["device_map"] = [0]
    ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=64 * MiB, pool_cap=[G.UNLIMITED],
                                    pool_floor_bytes=0))
    errors = []
    sizes = [3 * MiB + 5, 17 * MiB, 70 * MiB + 1, 130 * MiB]

    def worker(t):
        try:
            torch.cuda.set_device(0)
            s = torch.cuda.Stream()
            f = G.fn(40 + t, 1, 0)
            g = G.fn(40 + t, 2, 0)
            src = torch.empty(max(sizes), dtype=torch.uint8, device="cuda")
            dst = torch.empty(max(sizes), dtype=torch.uint8, device="cuda")
            live = []
            for i in range(12):
                n = sizes[(t + i) % len(sizes)]
                seed = 7000 + 100 * t + i
                G.check(G.test_fill(src.data_ptr(), n, seed, 0, s.cuda_stream), "fill")
                st, oid = ctx.put(f, src.data_ptr(), n, G.NOHINT, 0, s.cuda_stream)
                G.check(st, "put")
                live.append((oid, n, seed))
                if len(live) > 3:
                    oid, n, seed = live.pop(0)
                    G.check(ctx.get_into(g, oid, dst.data_ptr(), n, s.cuda_stream)[0], "get_into")
                    s.synchronize()
                    st, bad, first = G.test_verify(dst.data_ptr(), n, seed, 0, 0)
                    assert st == 0 and bad == 0, (t, n, bad, first)
                    G.check(ctx.free(f, oid), "free")
            for oid, n, seed in live:
                G.check(ctx.get_into(g, oid, dst.data_ptr(), n, s.cuda_stream)[0], "get_into")
                s.synchronize()
                st, bad, first = G.test_verify(dst.data_ptr(), n, seed, 0, 0)
                assert st == 0 and bad == 0, (t, n, bad, first)
                G.check(ctx.free(f, oid), "free")
        except Exception as e:  # pragma: no cover - reported below
            errors.append(repr(e))

    try:
        ths = [threading.Thread(target=worker, args=(t,)) for t in range(6)]
        for th in ths:
            th.start()
        for th in ths:
            th.join()
        assert not errors, errors
        G.check(ctx.sync(), "sync")
        st = ctx.stats()
        assert st.used[0] == 0 and st.host_used == 0
        assert st.mapped[0] >= 130 * MiB
    finally:
        ctx.close()


def test_lease_growth_without_the_lock_under_concurrency():
    """Copy leases (a gFn on logical GPU1 gets objects of logical GPU0) that
    must grow GPU1's cold pool, from several threads at once, while other
    threads put and free on GPU0: the lease's segment creation runs with the
    context lock released, and the object is looked up again afterwards.
    Every lease reads its object's bytes; a get of an object freed meanwhile
    could only return ENOENT (each thread frees its own objects only after
    releasing their leases, so here every get succeeds); the pools drain."""
    calib = C.virtual(2)
    ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=64 * MiB, pool_cap=[G.UNLIMITED] * 2,
                                    pool_floor_bytes=0))
    errors = []
    sizes = [5 * MiB + 3, 33 * MiB, 70 * MiB + 1, 97 * MiB]

    def worker(t):
        try:
            torch.cuda.set_device(0)
            s = torch.cuda.Stream()
            f = G.fn(60 + t, 1, 0)     # producer on GPU0
            g = G.fn(60 + t, 2, 1)     # consumer on GPU1: copy leases
            src = torch.empty(max(sizes), dtype=torch.uint8, device="cuda")
            for i in range(8):
                n = sizes[(t + i) % len(sizes)]
                seed = 9000 + 100 * t + i
                G.check(G.test_fill(src.data_ptr(), n, seed, 0, s.cuda_stream), "fill")
                st, oid = ctx.put(f, src.data_ptr(), n, G.NOHINT, 0, s.cuda_stream)
                G.check(st, "put")
                st, ptr, nn = ctx.get(g, oid, s.cuda_stream)
                G.check(st, "get")
                s.synchronize()
                st, bad, first = G.test_verify(ptr, n, seed, 0, 0)
                assert st == 0 and bad == 0, (t, n, bad, first)
                G.check(ctx.release(g, oid, ptr, s.cuda_stream), "release")
                G.check(ctx.free(f, oid), "free")
        except Exception as e:  # pragma: no cover - reported below
            errors.append(repr(e))

    try:
        ths = [threading.Thread(target=worker, args=(t,)) for t in range(6)]
        for th in ths:
            th.start()
        for th in ths:
            th.join(timeout=300)
        assert not any(th.is_alive() for th in ths), "a client thread hung"
        assert not errors, errors
        G.check(ctx.sync(), "sync")
        st = ctx.stats()
        assert st.used[0] == 0 and st.used[1] == 0 and st.host_used == 0
        assert st.mapped[1] >= 97 * MiB
    finally:
        ctx.close()
