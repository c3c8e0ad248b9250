"""Same-GPU get_into / by-copy put with user buffers at odd addresses
(38,535,168 B, back to back, device-timed): engine choice for misaligned
rounds.  Usage: python tools/misaligned.py"""
import sys
sys.path.insert(0, ".")
import torch
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G
from synth.calib import b200_hgx
G.load()
n = 38_535_168
calib = b200_hgx(1)
calib["device_map"] = [0]
ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=64 << 20, pool_cap=[G.UNLIMITED]))
f = G.fn(1, 2, 0)
s = torch.cuda.Stream()
objs = []
for i in range(4):
    st, buf, oid = ctx.alloc(f, n, 0, 0)
    G.check(G.test_fill(buf, n, 100 + i, 0, 0))
    G.check(ctx.seal(f, oid, 0))
    objs.append(oid)
dst = [torch.empty(n + 64, dtype=torch.uint8, device="cuda") for _ in range(4)]
for off in (0, 1, 3, 16, 17):
    for i in range(3):
        G.check(ctx.get_into(f, objs[i % 4], dst[i % 4].data_ptr() + off, n, s.cuda_stream)[0])
    s.synchronize()
    st, bad, _ = G.test_verify(dst[2].data_ptr() + off, n, 102, 0, 0)
    assert bad == 0, (off, bad)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    for i in range(40):
        ctx.get_into(f, objs[i % 4], dst[i % 4].data_ptr() + off, n, s.cuda_stream)
    b.record(s)
    b.synchronize()
    us = a.elapsed_time(b) * 1e3 / 40
    print(f"get_into dst offset {off}: {us:.2f} us per 38.5 MB ({2 * n / us / 1e6:.2f} TB/s r+w)", flush=True)
# by-copy put from a device buffer at an odd offset (stream-ordered); the
# first pass only warms the pool (cuMemCreate/Map of new pages is ~ms)
src = torch.empty(n + 64, dtype=torch.uint8, device="cuda")
for off in (0, 0, 5, 16):
    G.check(G.test_fill(src.data_ptr() + off, n, 55, 0, 0))
    oids = []
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    for i in range(20):
        st, oid = ctx.put(f, src.data_ptr() + off, n, G.NOHINT, 0, s.cuda_stream)
        G.check(st, "put")
        oids.append(oid)
    b.record(s)
    b.synchronize()
    us = a.elapsed_time(b) * 1e3 / 20
    st, p, m = ctx.get(f, oids[-1], s.cuda_stream)
    s.synchronize()
    st, bad, _ = G.test_verify(p, n, 55, 0, 0)
    assert bad == 0
    ctx.release(f, oids[-1], p)
    for o in oids:
        ctx.free(f, o)
    print(f"put src offset {off}: {us:.2f} us per 38.5 MB", flush=True)
ctx.close()
