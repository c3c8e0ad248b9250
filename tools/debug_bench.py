import sys
sys.path.insert(0, ".")
import torch
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G
from synth.calib import b200_hgx
from synth.payload import payload
import numpy as np
from tests.lib_runner import read_device
G.load()
n = 38_535_168
calib = b200_hgx(1); calib["device_map"] = [0]
for flags in [0, G.PROFILE]:
    ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=256 << 20, pool_cap=[G.UNLIMITED], flags=flags))
    tmp = torch.empty(n, dtype=torch.uint8, device="cuda")
    G.check(G.test_fill(tmp.data_ptr(), n, 1000, 0, 0))
    h = torch.empty(n, dtype=torch.uint8, pin_memory=True)
    h.copy_(tmp)
    print("host src ok:", np.array_equal(h.numpy()[:1 << 20], payload(1000, 1 << 20)), flush=True)
    st, oid = ctx.put(G.fn(1, 1, -1), h.data_ptr(), n, 0, 0)
    print("put", st, oid, flush=True)
    st, ptr, nn = ctx.get(G.fn(1, 2, 0), oid, 0)
    print("zero-copy get", st, hex(ptr), nn, flush=True)
    got = read_device(ptr, 1 << 20, 0)
    print("object ok:", np.array_equal(got, payload(1000, 1 << 20)), got[:8], payload(1000, 8), flush=True)
    st, bad, first = G.test_verify(ptr, n, 1000, 0, 0)
    print("object verify", st, bad, first, flush=True)
    s = torch.cuda.Stream()
    b = torch.empty(n, dtype=torch.uint8, device="cuda")
    st, nn = ctx.get_into(G.fn(1, 2, 0), oid, b.data_ptr(), n, s.cuda_stream)
    s.synchronize()
    st2, bad, first = G.test_verify(b.data_ptr(), n, 1000, 0, 0)
    print("get_into", st, "verify", st2, bad, first, flush=True)
    print(ctx.dump()[:600])
    ctx.release(G.fn(1, 2, 0), oid, ptr, 0)
    ctx.close()
