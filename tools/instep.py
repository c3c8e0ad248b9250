"""Diagnostic: how long does one gr_copy launch take inside the cfg1 loop?

Per-launch CUDA events (GROUTER_PROFILE, gated) for the gFn's get_into of a
freshly put 38.5 MB tensor under different concurrency:
  alone     Q=1, the consumer stream is drained after every get_into and the
            next put starts only then (kernel runs with the CE idle)
  serial    Q=1, no drain (the next put's H2D overlaps the kernel)
  q4        Q=4 client threads (the bench's closed loop)
  b2b       leg B alone back to back on resident objects
Prints the average launch duration of each and the SM clock NVML reports.
"""
import faulthandler
import sys
import threading
import time

sys.path.insert(0, ".")
import torch  # noqa: E402

from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G  # noqa: E402
from synth.calib import b200_hgx  # noqa: E402

G.load()
faulthandler.dump_traceback_later(70, exit=True)   # a hang prints every thread's stack
print("loaded", flush=True)
n = 38_535_168
calib = b200_hgx(1)
calib["device_map"] = [0]
ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=256 << 20, pool_cap=[G.UNLIMITED], flags=G.PROFILE))
cfn, gfn = G.fn(1, 1, G.HOST), G.fn(1, 2, 0)
hs = [torch.empty(n, dtype=torch.uint8, pin_memory=True) for _ in range(8)]
bind = [torch.empty(n, dtype=torch.uint8, device="cuda") for _ in range(8)]
streams = [torch.cuda.Stream() for _ in range(4)]


def kstats(fn):
    s0 = ctx.stats()
    fn()
    ctx.sync()
    torch.cuda.synchronize()
    s1 = ctx.stats()
    k = s1.timed_launches - s0.timed_launches
    kk = s1.timed_kernel_launches - s0.timed_kernel_launches
    KUS[0] = (s1.timed_kernel_ns - s0.timed_kernel_ns) / max(kk, 1) / 1e3
    return k, (s1.timed_ns - s0.timed_ns) / max(k, 1) / 1e3


KUS = [0.0]


def loop(q, total, drain):
    def client(k):
        torch.cuda.set_device(0)
        for i in range(k, total, q):
            st, oid = ctx.put(cfn, hs[i % 8].data_ptr(), n, 0, 1)
            G.check(st, "put")
            G.check(ctx.get_into(gfn, oid, bind[i % 8].data_ptr(), n, streams[k].cuda_stream)[0], "get_into")
            if drain:
                streams[k].synchronize()
    ths = [threading.Thread(target=client, args=(k,)) for k in range(q)]
    for t in ths:
        t.start()
    for t in ths:
        t.join()


MODES = (("alone", 1, True), ("serial", 1, False), ("q4", 4, False), ("alone", 1, True))
if len(sys.argv) > 1:   # one mode only, then exit (GROUTER_HOST_PROFILE percentiles of that mode)
    MODES = [m for m in MODES if m[0] == sys.argv[1]][:1]
for name, q, drain in MODES:
    loop(q, 20, drain)
    k, us = kstats(lambda: loop(q, 200, drain))
    print(f"{name:8s} launches {k}  avg {us:.2f} us  (kernel stamps {KUS[0]:.2f} us)", flush=True)

if len(sys.argv) > 1:
    ctx.close()
    sys.exit(0)
res = []
for i in range(8):
    st, oid = ctx.put(cfn, hs[i].data_ptr(), n, 0, 0)
    res.append(oid)
ctx.sync()


def b2b():
    for r in range(50):
        for i, oid in enumerate(res):
            ctx.get_into(gfn, oid, bind[i].data_ptr(), n, streams[0].cuda_stream)


k, us = kstats(b2b)
print(f"b2b      launches {k}  avg {us:.2f} us (PROFILE events between launches; kernel stamps {KUS[0]:.2f} us)",
      flush=True)


def gap(delay_us):
    def f():
        for r in range(100):
            ctx.get_into(gfn, res[r % 8], bind[r % 8].data_ptr(), n, streams[0].cuda_stream)
            streams[0].synchronize()
            t = time.perf_counter()
            while (time.perf_counter() - t) * 1e6 < delay_us:
                pass
    return f


for d in (0, 50, 200, 700, 2000):
    k, us = kstats(gap(d))
    print(f"idle gap {d:5d} us before each launch: avg {us:.2f} us  (kernel stamps {KUS[0]:.2f} us)", flush=True)
ctx.close()
