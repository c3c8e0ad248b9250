"""Diagnostic (not product code): host cost of the dispatch thread per
copy-engine round of a striped host->GPU put (the relay path of L178) on one
B200 with k virtual route GPUs.  Run with GROUTER_HOST_PROFILE=1: the library
prints the host microseconds per dispatch round at finalize.  A physical box
with k route GPUs needs k rounds per ~190 us (one 10 MiB batch per link), so
k x (us per round) must stay well below 190 us for one dispatch thread to keep
k links busy.  argv: k [ce_relay]"""
import sys
import time

sys.path.insert(0, ".")
import torch  # noqa: E402

from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G  # noqa: E402
from synth import calib as C  # noqa: E402

G.load()
k = int(sys.argv[1])
flags = G.CE_RELAY if len(sys.argv) > 2 and sys.argv[2] == "ce_relay" else 0
ctx = G.Ctx(G.config_from_calib(C.virtual(k), host_store_bytes=64 << 20, pool_cap=[G.UNLIMITED] * k,
                                flags=flags, pool_floor_bytes=64 << 20))
n = 256 << 20
host = torch.empty(n, dtype=torch.uint8, pin_memory=True)
st, plan = ctx.plan(G.HOST, 0, n)
f = G.fn(1, 1, G.HOST)
ts = []
for r in range(6):
    t = time.perf_counter()
    st, oid = ctx.put(f, host.data_ptr(), n, 0, 0)
    G.check(st, "put")
    ts.append(time.perf_counter() - t)
    ctx.free(f, oid)
print(f"k={k} flags={flags:#x} routes={sorted({c[3] for c in plan})} put 256 MiB best {min(ts[1:]) * 1e6:.0f} us "
      f"({n / min(ts[1:]) / 1e9:.1f} GB/s)", flush=True)
ctx.close()
