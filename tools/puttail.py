"""Diagnostic: the tail of single large cFn puts (bench sweep `put_h2d` p99).

Repeats put(hint GPU0) + free of one pinned host buffer, like the sweep, and
prints every call's host time with the pool's mapped bytes before/after and
the library's host-side phase breakdown for the slow calls.  Run with
GR_DIAG=1 to see the background thread's slow pool ticks.
  python tools/puttail.py [MiB] [reps] [sweep]
`sweep`: like bench.py's sweep row -- one object of the size stays resident
and a bare pinned H2D of the same size runs between the samples.
"""
import sys
import time

sys.path.insert(0, ".")
import torch  # noqa: E402

from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G  # noqa: E402
from synth.calib import b200_hgx  # noqa: E402

G.load()
n = int(sys.argv[1] if len(sys.argv) > 1 else 1024) << 20
reps = int(sys.argv[2] if len(sys.argv) > 2 else 30)
calib = b200_hgx(1)
calib["device_map"] = [0]
ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=n + (256 << 20), pool_cap=[G.UNLIMITED],
                                pool_floor_bytes=64 << 20))
host = torch.empty(n, dtype=torch.uint8, pin_memory=True)
cfn = G.fn(7, 1, G.HOST)
sweep = len(sys.argv) > 3 and sys.argv[3] == "sweep"
if sweep:
    st, keep = ctx.put(cfn, host.data_ptr(), n, 0, 0)
    G.check(st, "put")
    dst = torch.empty(n, dtype=torch.uint8, device="cuda")
xs = []
for i in range(reps):
    m0 = ctx.stats().mapped[0]
    t = time.perf_counter()
    st, oid = ctx.put(cfn, host.data_ptr(), n, 0, 0)
    dt = (time.perf_counter() - t) * 1e3
    G.check(st, "put")
    m1 = ctx.stats().mapped[0]
    ctx.free(cfn, oid)
    xs.append(dt)
    print(f"{i:3d} put {dt:9.2f} ms  mapped {m0 >> 20} -> {m1 >> 20} MiB", flush=True)
    if sweep:
        t = time.perf_counter()
        G.check(G.test_memcpy(dst.data_ptr(), host.data_ptr(), n, 0, True))
        print(f"      memcpy {(time.perf_counter() - t) * 1e3:9.2f} ms", flush=True)
    elif i % 7 == 6:
        time.sleep(0.3)
xs.sort()
print(f"p50 {xs[len(xs) // 2]:.2f} ms  max {xs[-1]:.2f} ms  link {n / xs[len(xs) // 2] / 1e6:.1f} GB/s")
ctx.close()
