"""ncu target (diagnostic): back-to-back same-GPU get_into of 256 MiB objects
through the C ABI -- the default engine there is tmas4 (static TMA ring).
usage: ncu --set full -k regex:gr_copy_tmas -s 2 -c 2 python tools/ncu_tmas.py"""
import sys
sys.path.insert(0, ".")
import torch  # noqa: E402
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G  # noqa: E402
from synth.calib import b200_hgx  # noqa: E402

G.load()
n = 256 << 20
calib = b200_hgx(1)
calib["device_map"] = [0]
ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=64 << 20, pool_cap=[G.UNLIMITED]))
f = G.fn(1, 2, 0)
s = torch.cuda.Stream()
objs = []
for i in range(3):
    st, buf, oid = ctx.alloc(f, n, 0, 0)
    G.check(st, "alloc")
    G.check(G.test_fill(buf, n, 3 + i, 0, 0), "fill")
    G.check(ctx.seal(f, oid, 0), "seal")
    objs.append(oid)
dsts = [torch.empty(n, dtype=torch.uint8, device="cuda") for _ in range(2)]
for i in range(6):
    G.check(ctx.get_into(f, objs[i % 3], dsts[i % 2].data_ptr(), n, s.cuda_stream)[0], "get_into")
s.synchronize()
st, bad, _ = G.test_verify(dsts[1].data_ptr(), n, 3 + 5 % 3, 0, 0)
assert bad == 0
ctx.close()
print("ok")
