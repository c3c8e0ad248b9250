"""ncu range target (diagnostic): one blocking cFn put of 256 MiB from pinned
host (hint GPU0: the H2D engine) and one cFn get of it back (D2H engine),
each inside its own cudaProfilerStart/Stop range.
usage: ncu --replay-mode range --metrics pcie__read_bytes.sum,pcie__write_bytes.sum,gpu__time_duration.sum \
           python tools/ncu_pcie.py"""
import sys
sys.path.insert(0, ".")
import torch  # noqa: E402
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G  # noqa: E402
from synth.calib import b200_hgx  # noqa: E402

G.load()
n = 256 << 20
calib = b200_hgx(1)
calib["device_map"] = [0]
ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=512 << 20, pool_cap=[G.UNLIMITED]))
host = torch.empty(n, dtype=torch.uint8, pin_memory=True)
cfn = G.fn(1, 1, G.HOST)
torch.cuda.synchronize()
torch.cuda.profiler.start()
st, oid = ctx.put(cfn, host.data_ptr(), n, 0, 0)
G.check(st, "put")
torch.cuda.synchronize()
torch.cuda.profiler.stop()
torch.cuda.profiler.start()
st, ptr, nn = ctx.get(cfn, oid, 0)
G.check(st, "get")
torch.cuda.synchronize()
torch.cuda.profiler.stop()
ctx.release(cfn, oid, ptr, 0)
ctx.free(cfn, oid)
ctx.close()
print("ok")
