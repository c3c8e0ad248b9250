"""A/B of the Python binding's marshalling on one box: the data-path calls
with typed POINTER argtypes + per-call out objects (the round-2 binding
before the change) vs plain addresses + per-thread out slots (grouter.py
now), on the same context, interleaved; 4 KiB get_into on an idle stream,
host time per call, p50 over 2000 calls each."""
import ctypes as C
import sys
import time

sys.path.insert(0, ".")
import torch  # noqa: E402

from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G  # noqa: E402
from synth.calib import b200_hgx  # noqa: E402

lib = G.load()
old = C.CDLL(lib._name)
f_old = old.grouter_get_into
f_old.restype = C.c_int
f_old.argtypes = [C.c_void_p, C.POINTER(G.grouter_fn), C.c_uint64, C.c_void_p, C.c_uint64, C.c_void_p,
                  C.POINTER(C.c_uint64)]
calib = b200_hgx(1)
calib["device_map"] = [0]
ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=64 << 20, pool_cap=[G.UNLIMITED]))
n = 4096
host = torch.empty(n, dtype=torch.uint8, pin_memory=True)
st, oid = ctx.put(G.fn(1, 1, G.HOST), host.data_ptr(), n, 0, 0)
d = torch.empty(n, dtype=torch.uint8, device="cuda")
s = torch.cuda.Stream()
ss = s.cuda_stream
g = G.fn(1, 2, 0)


def old_call():
    nn = C.c_uint64(0)
    st = f_old(ctx.h, C.byref(g), oid, d.data_ptr() or None, n, ss or None, C.byref(nn))
    return st, nn.value


def new_call():
    return ctx.get_into(g, oid, d.data_ptr(), n, ss)


xs = {"typed POINTER args": [], "address args": []}
for i in range(4000):
    name, f = (("typed POINTER args", old_call), ("address args", new_call))[i & 1]
    s.synchronize()
    t = time.perf_counter()
    st, _ = f()
    xs[name].append((time.perf_counter() - t) * 1e6)
    assert st == 0
for k, v in xs.items():
    v.sort()
    print(f"{k:20s} get_into 4 KiB host p50 {v[len(v) // 2]:.2f} us  p10 {v[len(v) // 10]:.2f} us", flush=True)
ctx.close()
