"""Host-path latency of small blocking cFn puts / gets and device get_into on an
idle GPU, with GROUTER_HOST_PROFILE=1 stage times (printed at close)."""
import sys
import time
sys.path.insert(0, ".")
import torch
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G
from synth.calib import b200_hgx
G.load()
calib = b200_hgx(1)
calib["device_map"] = [0]
ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=256 << 20, pool_cap=[G.UNLIMITED]))
cfn, gfn = G.fn(1, 1, -1), G.fn(1, 2, 0)
s = torch.cuda.Stream()
for n in [int(a) for a in sys.argv[1:]] or (4096, 262144, 4 << 20):
    h = torch.empty(n, dtype=torch.uint8, pin_memory=True)
    ts, tg, td = [], [], []
    d = torch.empty(n, dtype=torch.uint8, device="cuda")
    for i in range(300):
        t = time.perf_counter()
        st, oid = ctx.put(cfn, h.data_ptr(), n, 0, 0)
        t1 = time.perf_counter()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        ctx.get_into(gfn, oid, d.data_ptr(), n, s.cuda_stream)
        b.record(s)
        b.synchronize()
        t2 = time.perf_counter()
        st, p, m = ctx.get(cfn, oid)
        t3 = time.perf_counter()
        ctx.release(cfn, oid, p)
        ctx.free(cfn, oid)
        ts.append((t1 - t) * 1e6)
        tg.append(a.elapsed_time(b) * 1e3)
        td.append((t3 - t2) * 1e6)
    for name, xs in (("put H2D blocking", ts), ("get_into device events", tg), ("get D2H blocking", td)):
        xs.sort()
        print(f"n={n} {name}: p50 {xs[150]:.2f} us p10 {xs[30]:.2f} us", flush=True)
    t = time.perf_counter()
    for i in range(1000):
        torch.cuda.synchronize()
    print("torch.cuda.synchronize idle us", round((time.perf_counter() - t) * 1e3, 2))
ctx.close()
