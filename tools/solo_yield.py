"""Diagnostic (not product code): a tenant arriving while a 1 GiB GPU -> other-GPU
transfer moves on the forced peer branch (R55 solo rounds): device and host timelines of both
calls.  Run beside GR_NO_SOLO=1 (one batch per round)."""
import sys, time, threading
sys.path.insert(0, ".")
import torch
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G
from synth import calib as C
G.load()
MiB = 1 << 20
ctx = G.Ctx(G.config_from_calib(C.virtual(2), host_store_bytes=64 * MiB, pool_cap=[G.UNLIMITED] * 2,
                                pool_floor_bytes=64 * MiB, flags=G.FORCE_REMOTE))
big, small = 1 << 30, 4096
src = torch.empty(big, dtype=torch.uint8, device="cuda")
G.check(G.test_fill(src.data_ptr(), big, 616, 0, 0)); torch.cuda.synchronize()
st, oa = ctx.put(G.fn(1, 1, 0), src.data_ptr(), big, G.NOHINT, 0, 0)
st, ob = ctx.put(G.fn(2, 1, 0), src.data_ptr(), small, G.NOHINT, 0, 0)
ctx.sync()
sa, sb = torch.cuda.Stream(), torch.cuda.Stream()
da = torch.empty(big, dtype=torch.uint8, device="cuda"); db = torch.empty(small, dtype=torch.uint8, device="cuda")
for rep in range(4):
    e0, ea, eb = (torch.cuda.Event(enable_timing=True) for _ in range(3))
    e0.record(sa); sb.wait_event(e0)
    hs = {}
    def big_get():
        t = time.perf_counter(); ctx.get_into(G.fn(1, 2, 1), oa, da.data_ptr(), big, sa.cuda_stream); hs['a'] = (t, time.perf_counter()); ea.record(sa)
    th = threading.Thread(target=big_get); t0 = time.perf_counter(); th.start(); time.sleep(100e-6)
    t1 = time.perf_counter(); ctx.get_into(G.fn(2, 2, 1), ob, db.data_ptr(), small, sb.cuda_stream); t2 = time.perf_counter(); eb.record(sb)
    th.join(); ea.synchronize(); eb.synchronize()
    print(f"rep {rep}: t_big {e0.elapsed_time(ea):.3f} ms t_small {e0.elapsed_time(eb):.3f} ms | host: A call {1e6*(hs['a'][0]-t0):.0f}->{1e6*(hs['a'][1]-t0):.0f} us, B call {1e6*(t1-t0):.0f}->{1e6*(t2-t0):.0f} us", flush=True)
st = ctx.stats(); print("launches", st.kernel_launches, "rounds", st.rounds)
