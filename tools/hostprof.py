"""Host-side cost of one get_into through the C ABI (no GPU wait), split
into the ctypes call and the library; run under gpurun."""
import sys, time
sys.path.insert(0, ".")
import torch
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G
from synth.calib import b200_hgx
G.load()
n = 38_535_168
calib = b200_hgx(1); calib["device_map"] = [0]
for flags in (0, G.PROFILE):
    ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=256 << 20, pool_cap=[G.UNLIMITED], flags=flags))
    h = torch.empty(n, dtype=torch.uint8, pin_memory=True)
    st, oid = ctx.put(G.fn(1, 1, -1), h.data_ptr(), n, 0, 0)
    s = torch.cuda.Stream()
    bs = [torch.empty(n, dtype=torch.uint8, device="cuda") for _ in range(4)]
    f = G.fn(1, 2, 0)
    for rep in range(3):
        t = time.perf_counter()
        for i in range(200):
            ctx.get_into(f, oid, bs[i % 4].data_ptr(), n, s.cuda_stream)
        t1 = time.perf_counter()
        s.synchronize()
        t2 = time.perf_counter()
        print("flags", flags, "host us/call", round((t1 - t) * 1e6 / 200, 2), "total us/call", round((t2 - t) * 1e6 / 200, 2), flush=True)
    # pure ctypes overhead of a cheap call
    t = time.perf_counter()
    for i in range(2000):
        ctx.where(oid)
    print("ctypes where() us/call", round((time.perf_counter() - t) * 1e6 / 2000, 2))
    ctx.close()

# latency mode: one get_into at a time on an idle GPU (host time of the call only)
ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=256 << 20, pool_cap=[G.UNLIMITED]))
h = torch.empty(n, dtype=torch.uint8, pin_memory=True)
st, oid = ctx.put(G.fn(1, 1, -1), h.data_ptr(), n, 0, 0)
s = torch.cuda.Stream()
b = torch.empty(n, dtype=torch.uint8, device="cuda")
f = G.fn(1, 2, 0)
ts = []
for i in range(300):
    s.synchronize()
    t = time.perf_counter()
    ctx.get_into(f, oid, b.data_ptr(), n, s.cuda_stream)
    ts.append((time.perf_counter() - t) * 1e6)
ts.sort()
print("latency mode: host us/call p50", round(ts[150], 2), "p10", round(ts[30], 2), flush=True)
# raw ctypes call of the same entry point (no Python wrapper)
fnp = G.grouter_fn(1, 2, 0) if hasattr(G, "grouter_fn") else None
ctx.close()
