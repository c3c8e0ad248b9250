"""Host cost of the Python binding per call (what the sweep's single-call
latencies carry on top of the GPU time): ctx.get_into (fast direct path)
vs G.test_memcpy (bare cudaMemcpyAsync through the same binding) vs a
trivial ctypes call, all on an idle stream; also the dev-timed single call
both ways.  4 KiB, 300 samples, p50 in us."""
import ctypes as C
import sys
import time

sys.path.insert(0, ".")
import torch  # noqa: E402

from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G  # noqa: E402
from synth.calib import b200_hgx  # noqa: E402

lib = G.load()
calib = b200_hgx(1)
calib["device_map"] = [0]
ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=64 << 20, pool_cap=[G.UNLIMITED]))
n = 4096
host = torch.empty(n, dtype=torch.uint8, pin_memory=True)
st, oid = ctx.put(G.fn(1, 1, G.HOST), host.data_ptr(), n, 0, 0)
d = [torch.empty(n, dtype=torch.uint8, device="cuda") for _ in range(2)]
s = torch.cuda.Stream()
ss = s.cuda_stream
g = G.fn(1, 2, 0)


def p50(xs):
    xs = sorted(xs)
    return round(xs[len(xs) // 2], 2)


def host_cost(call, reps=300):
    xs = []
    for i in range(reps):
        s.synchronize()
        t = time.perf_counter()
        call(i)
        xs.append((time.perf_counter() - t) * 1e6)
    return p50(xs)


def dev_cost(call, reps=300):
    xs = []
    for i in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        call(i)
        b.record(s)
        b.synchronize()
        xs.append(a.elapsed_time(b) * 1e3)
    return p50(xs)


gi = lambda i: ctx.get_into(g, oid, d[i & 1].data_ptr(), n, ss)
mc = lambda i: G.test_memcpy(d[i & 1].data_ptr(), d[(i + 1) & 1].data_ptr(), n, ss, False)
raw = lambda i: lib.grouter_test_memcpy(d[i & 1].data_ptr(), d[(i + 1) & 1].data_ptr(), n, ss, 0)
nop = lambda i: lib.grouter_strerror(0)
ev = torch.cuda.Event(enable_timing=True)
rec = lambda i: ev.record(s)
for name, f in (("get_into", gi), ("test_memcpy", mc), ("raw ctypes memcpy", raw), ("ctypes strerror", nop),
                ("torch event record", rec)):
    f(0)
    print(f"{name:20s} host {host_cost(f):6.2f} us   dev-timed {dev_cost(f):6.2f} us", flush=True)
ctx.close()

# blocking cFn put of 4 KiB (fast copy-engine path) vs a bare pinned H2D + wait through the binding
ctx2 = G.Ctx(G.config_from_calib(calib, host_store_bytes=64 << 20, pool_cap=[G.UNLIMITED]))
cf = G.fn(2, 1, G.HOST)


def put4k(i):
    st, o = ctx2.put(cf, host.data_ptr(), n, 0, 0)
    ctx2.free(cf, o)


def put4k_only(i):
    st, o = ctx2.put(cf, host.data_ptr(), n, 0, 0)
    frees.append(o)


frees = []
h2d = lambda i: G.test_memcpy(d[0].data_ptr(), host.data_ptr(), n, 0, True)
for name, f in (("put+free 4 KiB", put4k), ("put 4 KiB", put4k_only), ("bare H2D+wait", h2d)):
    f(0)
    print(f"{name:20s} host {host_cost(f):6.2f} us", flush=True)
    for o in frees:
        ctx2.free(cf, o)
    frees.clear()
ctx2.close()
