"""Small workload for compute-sanitizer: every copy-engine variant over aligned
and misaligned chunk lists, plus a replay trace through the full library."""
import os
import sys
sys.path.insert(0, ".")
import random
import torch
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G
from synth import calib as C, traces as T
G.load()
MiB = 1 << 20
for tma in (False, True):
    for so, do in ((0, 0), (3, 3), (1, 0), (7, 13)):
        n = 1 * MiB + 12345
        src = torch.empty(n + 64, dtype=torch.uint8, device="cuda")
        dst = torch.empty(n + 64, dtype=torch.uint8, device="cuda")
        G.check(G.test_fill(src.data_ptr() + so, n, 5, 0, 0))
        cuts = sorted(random.Random(so).sample(range(1, n), 4))
        b = [0] + cuts + [n]
        G.check(G.test_copy(dst.data_ptr() + do, src.data_ptr() + so, [(x, y - x, 0, 0) for x, y in zip(b, b[1:])], tma=tma))
        torch.cuda.synchronize()
        st, bad, _ = G.test_verify(dst.data_ptr() + do, n, 5, 0, 0)
        assert bad == 0
# 16 B-aligned chunk lists (the bulk-copy engines only take these)
for seed in (1, 2):
    n = 3 * MiB + 48 * seed
    rng = random.Random(seed)
    cuts = sorted({16 * rng.randint(1, n // 16 - 1) for _ in range(5)})
    b = [0] + cuts + [n]
    src = torch.empty(n, dtype=torch.uint8, device="cuda")
    dst = torch.empty(n, dtype=torch.uint8, device="cuda")
    G.check(G.test_fill(src.data_ptr(), n, 9, 0, 0))
    G.check(G.test_copy(dst.data_ptr(), src.data_ptr(), [(x, y - x, 0, 0) for x, y in zip(b, b[1:])]))
    torch.cuda.synchronize()
    st, bad, _ = G.test_verify(dst.data_ptr(), n, 9, 0, 0)
    assert bad == 0
from tests.lib_runner import LibRunner
from oracle import runner as orun
from tests.lib_runner import compare
calib = C.virtual(2)
ops = T.cfg2(2, requests=2, scale=64) + []
r = LibRunner(calib, replay=True, keep_bytes=True)
out = r(ops)
r.close()
compare(orun.run(ops, calib, keep_bytes=True), out)
# real-time mode with proactive restore and gFn-host striping: direct
# launches (event completion, PDL), server rounds, spills, restores
rng = random.Random(7)
ops = T.random_trace(rng, 2, n_ops=60, max_n=3 * MiB, run_seed=7)
r = LibRunner(calib, replay=False, keep_bytes=True, flags=G.RESTORE | G.D2H_MULTIPATH,
              host_store_bytes=64 * MiB, pool_cap=[8 * MiB, 16 * MiB])
out = r(ops)
r.close()
compare(orun.run(ops, calib, keep_bytes=True, restore=True, d2h_multipath=True,
                 host_store_bytes=64 * MiB, pool_cap=[8 * MiB, 16 * MiB]), out, check_dispatch=False)
# back-to-back direct get_into on one stream (the bench's pattern)
c1 = dict(C.b200_hgx(1), device_map=[0])
ctx = G.Ctx(G.config_from_calib(c1, host_store_bytes=64 * MiB, pool_cap=[G.UNLIMITED], pool_floor_bytes=64 * MiB))
n = 3 * MiB + 5
src = torch.empty(n, dtype=torch.uint8, device="cuda")
G.check(G.test_fill(src.data_ptr(), n, 11, 0, 0))
torch.cuda.synchronize()
st, oid = ctx.put(G.fn(1, 1, 0), src.data_ptr(), n, G.NOHINT, 0, 0)
s = torch.cuda.Stream()
dsts = [torch.empty(n, dtype=torch.uint8, device="cuda") for _ in range(3)]
for i in range(12):
    G.check(ctx.get_into(G.fn(1, 2, 0), oid, dsts[i % 3].data_ptr(), n, s.cuda_stream)[0])
s.synchronize()
for d in dsts:
    assert G.test_verify(d.data_ptr(), n, 11, 0, 0)[1] == 0
ctx.close()
# cfg1 at full size on two logical GPUs in real time: the striped put relays
# through logical GPU1's staging ring with one forward launch per chunk
# (K4'), then a D2D get; once more with every copy on the peer branch
for flags in (0, G.FORCE_REMOTE):
    ops = T.cfg1(2, iters=2)
    r = LibRunner(calib, replay=False, keep_bytes=False, flags=flags)
    out = r(ops)
    r.close()
    orc = orun.run(ops, calib)
    for o, l in zip(orc["records"], out["records"]):
        assert o["status"] == l["status"] and o.get("digest") == l.get("digest")
    assert out["stats"].kernel_launches > 0
# blocking small puts/gets on an idle copy engine (fast_ce) and small direct copies (fast_direct)
ctx = G.Ctx(G.config_from_calib(c1, host_store_bytes=64 * MiB, pool_cap=[G.UNLIMITED], pool_floor_bytes=64 * MiB))
host = torch.empty(1 << 20, dtype=torch.uint8, pin_memory=True)
host.copy_(torch.arange(1 << 20, dtype=torch.int64).to(torch.uint8))
cf = G.fn(3, 1, G.HOST)
for i in range(6):
    n = 4096 << i
    st, oid = ctx.put(cf, host.data_ptr(), n, 0, 0)
    G.check(st, "put")
    st, ptr, nn = ctx.get(cf, oid, 0)
    G.check(st, "get")
    import ctypes
    import numpy as np
    assert bytes((ctypes.c_uint8 * n).from_address(ptr)) == host.numpy()[:n].tobytes()
    ctx.release(cf, oid, ptr, 0)
    ctx.free(cf, oid)
ctx.close()
# cross-GPU dispatch on the peer branch (R55, R56): small pulls on the
# consumer's stream and whole-transfer pushes from the source's copy server,
# back to back on one consumer stream (the third get queues behind the window)
ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=64 * MiB, pool_cap=[G.UNLIMITED] * 2,
                                pool_floor_bytes=64 * MiB, flags=G.FORCE_REMOTE))
s = torch.cuda.Stream()
for n in (64 * 1024 + 16, 4 * MiB, 12 * MiB + 4096):
    src = torch.empty(n, dtype=torch.uint8, device="cuda")
    G.check(G.test_fill(src.data_ptr(), n, 21, 0, 0))
    torch.cuda.synchronize()
    st, oid = ctx.put(G.fn(4, 1, 0), src.data_ptr(), n, G.NOHINT, 0, 0)
    G.check(st, "put")
    ctx.sync()
    dsts = [torch.empty(n, dtype=torch.uint8, device="cuda") for _ in range(3)]
    for i in range(6):
        G.check(ctx.get_into(G.fn(4, 2, 1), oid, dsts[i % 3].data_ptr(), n, s.cuda_stream)[0])
    s.synchronize()
    for d in dsts:
        assert G.test_verify(d.data_ptr(), n, 21, 0, 0)[1] == 0
    ctx.free(G.fn(4, 1, 0), oid)
ctx.close()
print("sanitize workload OK", os.environ.get("GR_COPY", "default"))
