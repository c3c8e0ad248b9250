"""Diagnostic: host cost of a small pinned H2D copy issued by torch in this
process before and after a GROUTER context exists, and of a blocking cFn put
of the same bytes (4 KiB).  Run under gpurun."""
import sys
import time
sys.path.insert(0, ".")
import torch
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G
from synth.calib import b200_hgx

n = 4096
h = torch.empty(n, dtype=torch.uint8, pin_memory=True)
d = torch.empty(n, dtype=torch.uint8, device="cuda")
s = torch.cuda.Stream()


def torch_copy(tag):
    call, tot = [], []
    for i in range(400):
        s.synchronize()
        t0 = time.perf_counter()
        with torch.cuda.stream(s):
            d.copy_(h, non_blocking=True)
        t1 = time.perf_counter()
        s.synchronize()
        call.append((t1 - t0) * 1e6)
        tot.append((time.perf_counter() - t0) * 1e6)
    call.sort()
    tot.sort()
    print(f"{tag}: torch copy_ call p50 {call[200]:.2f} us, with sync p50 {tot[200]:.2f} us", flush=True)


torch_copy("before ctx")
G.load()
calib = b200_hgx(1)
calib["device_map"] = [0]
ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=256 << 20, pool_cap=[G.UNLIMITED]))
torch_copy("after ctx")
cfn = G.fn(1, 1, -1)
for tag, src in (("torch pinned src", h.data_ptr()),):
    ts = []
    for i in range(400):
        t = time.perf_counter()
        st, oid = ctx.put(cfn, src, n, 0, 0)
        ts.append((time.perf_counter() - t) * 1e6)
        ctx.free(cfn, oid)
    ts.sort()
    print(f"put {tag}: p50 {ts[200]:.2f} us p10 {ts[40]:.2f}", flush=True)
# a host-store source (cudaHostAlloc'ed by the library)
st, buf, oid0 = ctx.alloc(cfn, n, G.NOHINT, 0)
ctx.seal(cfn, oid0)
ts = []
for i in range(400):
    t = time.perf_counter()
    st, oid = ctx.put(cfn, buf, n, 0, 0)
    ts.append((time.perf_counter() - t) * 1e6)
    ctx.free(cfn, oid)
ts.sort()
print(f"put host-store src: p50 {ts[200]:.2f} us p10 {ts[40]:.2f}", flush=True)
ts = []
for i in range(400):
    t = time.perf_counter()
    ctx.where(oid0)
    ts.append((time.perf_counter() - t) * 1e6)
ts.sort()
print(f"ctypes where(): p50 {ts[200]:.2f} us", flush=True)
ctx.close()
torch_copy("after close")
