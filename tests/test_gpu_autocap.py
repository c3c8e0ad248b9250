"""Auto cap (O10; "GROUTER triggers data migration and
restoration automatically based on available GPU memory, maintaining storage
usage within a fixed threshold (50% of free memory in our experiments)";
DESIGN.md R12, R54) on the GPU.

* the measured availability (cudaMemGetInfo free + the pool's own mapped
  bytes) lies between torch's own free readings around the call, and the cap
  applied is the oracle's O10 function of it;
* the background thread follows free memory: another allocation on the GPU
  (a function's working set) makes the store migrate victims to the host in
  queue-aware order until it is within the threshold again, and releasing it
  brings them back (GROUTER_RESTORE) -- payloads intact both ways;
* an explicit set_pool_limit takes the GPU out of auto mode; refresh_cap puts
  it back.
The synthetic-availability parity (case G, random traces) is in
tests/test_gpu_parity.py.
"""
import time

import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

from oracle import model as M                                        # noqa: E402
from paper_conf_eurosys_wulywdyfwwj26_b200 import _build            # noqa: E402
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G      # noqa: E402
from synth import calib as C                                         # noqa: E402

MiB = 1 << 20


@pytest.fixture(scope="module", autouse=True)
def lib():
    _build.build()
    return G.load()


def _ctx(period_us, permille=500, flags=0, host=64 * MiB):
    calib = C.b200_hgx(1)
    calib["device_map"] = [0]
    return G.Ctx(G.config_from_calib(calib, host_store_bytes=host, pool_cap=[0], pool_floor_bytes=0,
                                     auto_cap_period_us=period_us, pool_cap_permille=permille, flags=flags))


def test_measured_availability_and_cap():
    ctx = _ctx(0)
    try:
        s0 = ctx.stats()
        assert s0.auto_mode & 1
        f_hi = torch.cuda.mem_get_info(0)[0]
        st, cap = ctx.refresh_cap(0)
        f_lo = torch.cuda.mem_get_info(0)[0]
        assert st == G.OK
        s = ctx.stats()
        avail, mapped = s.auto_avail[0], s.mapped[0]
        assert s.auto_refreshes == s0.auto_refreshes + 1
        # nothing else allocates meanwhile: the library's reading is torch's
        assert min(f_hi, f_lo) + mapped <= avail <= max(f_hi, f_lo) + mapped, (f_hi, f_lo, mapped, avail)
        assert cap == M.auto_cap(avail, 500) == s.cap[0]
        assert cap % (2 * MiB) == 0 and cap <= avail // 2
        # an explicit limit leaves auto mode; refresh_cap re-enters it
        assert ctx.set_pool_limit(0, 64 * MiB) == G.OK
        assert not ctx.stats().auto_mode & 1
        st, cap2 = ctx.refresh_cap(0, 100 * MiB + 1)
        assert st == G.OK and cap2 == M.auto_cap(100 * MiB + 1) == 50 * MiB
        s = ctx.stats()
        assert s.auto_mode & 1 and s.cap[0] == 50 * MiB and s.auto_avail[0] == 100 * MiB + 1
        assert ctx.refresh_cap(3)[0] == G.EINVAL
    finally:
        ctx.close()


def _wait(pred, timeout=10.0):
    t0 = time.time()
    while not pred():
        if time.time() - t0 > timeout:
            return False
        time.sleep(0.01)
    return True


def test_background_refresh_migrates_and_restores():
    """permille 20 (2%): on an idle B200 the cap is ~3.6 GB; eight 256 MiB
    objects (2 GiB) fit.  A 100 GB torch allocation drops the cap to ~1.6 GB:
    the background thread migrates victims -- hinted objects at the tail of
    the queue first (L258) -- until used <= cap.  Freeing it raises the cap
    and every object comes back (R42)."""
    n, k = 256 * MiB, 8
    ctx = _ctx(2000, permille=20, flags=G.RESTORE, host=4 << 30)
    big = None
    try:
        free0 = torch.cuda.mem_get_info(0)[0]
        if free0 < 120 << 30:
            pytest.skip("needs an idle 180 GB GPU")
        assert _wait(lambda: ctx.stats().cap[0] > k * n)
        f = G.fn(7, 1, 0)
        s = torch.cuda.Stream()
        src = torch.empty(n, dtype=torch.uint8, device="cuda")
        oids = []
        for i in range(k):
            G.check(G.test_fill(src.data_ptr(), n, 900 + i, 0, s.cuda_stream))
            st, oid = ctx.put(f, src.data_ptr(), n, G.NOHINT, 0, s.cuda_stream)
            G.check(st, "put")
            G.check(ctx.set_next_use(oid, i))     # request i consumes object i
            oids.append(oid)
        s.synchronize()
        assert all(ctx.where(o)[1] == 0 for o in oids)
        spills0 = ctx.stats().spill_count
        big = torch.empty(100 << 30, dtype=torch.uint8, device="cuda")
        assert _wait(lambda: ctx.stats().spill_count > spills0 and ctx.stats().used[0] <= ctx.stats().cap[0])
        st_ = ctx.stats()
        assert st_.cap[0] == M.auto_cap(st_.auto_avail[0], 20) < k * n
        where = [ctx.where(o)[1] for o in oids]
        moved = [i for i, w in enumerate(where) if w == G.HOST]
        # queue-aware: the tail of the queue (largest next_use) left first
        assert moved and moved == list(range(k - len(moved), k)), where
        assert st_.used[0] == (k - len(moved)) * n
        del big
        big = None
        torch.cuda.empty_cache()
        assert _wait(lambda: all(ctx.where(o)[1] == 0 for o in oids))
        assert ctx.stats().restore_count >= len(moved)
        dst = torch.empty(n, dtype=torch.uint8, device="cuda")
        g = G.fn(7, 2, 0)
        for i, oid in enumerate(oids):
            G.check(ctx.get_into(g, oid, dst.data_ptr(), n, s.cuda_stream)[0], "get_into")
            s.synchronize()
            st2, bad, first = G.test_verify(dst.data_ptr(), n, 900 + i, 0, 0)
            assert st2 == G.OK and bad == 0, (i, bad, first)
        for oid in oids:
            assert ctx.free(f, oid) == G.OK
    finally:
        del big
        ctx.close()
