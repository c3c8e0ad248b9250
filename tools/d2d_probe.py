"""Single-process GPU0 -> GPU1 pushes for NVLink evidence (needs 2 GPUs; run
under ncu by tools/ncu_nvlink.sh): a gFn on GPU1 get_into's objects resident
on GPU0 -- GPU0's copy server pushes them with gr_copy over NVLink -- 20
times per size (5 at 1 GiB), byte-verified; then the same gets pulled by
GPU1 (GROUTER_PULL_ALL).  Also times them with CUDA events (not under ncu:
those numbers are the ones to report)."""
import json
import sys

sys.path.insert(0, ".")
import torch  # noqa: E402

from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G  # noqa: E402
from synth.calib import b200_hgx  # noqa: E402

assert torch.cuda.device_count() >= 2, "needs two GPUs"
G.load()
calib = b200_hgx(2)
calib["device_map"] = [0, 1]
res = {}
for mode, flags in (("default", 0), ("pull_all", G.PULL_ALL)):   # default: pulls <= 4 MiB, pushes above (R55, R56)
    ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=64 << 20, pool_cap=[G.UNLIMITED] * 2,
                                    pool_floor_bytes=64 << 20, flags=flags))
    s1 = torch.cuda.Stream(device=1)
    for n in (4 << 20, 38_535_168, 256 << 20, 1 << 30):
        src = torch.empty(n, dtype=torch.uint8, device="cuda:0")
        G.check(G.test_fill(src.data_ptr(), n, 99, 0, 0))
        torch.cuda.synchronize(0)
        st, oid = ctx.put(G.fn(1, 1, 0), src.data_ptr(), n, G.NOHINT, 0, 0)
        G.check(st, "put")
        ctx.sync()
        del src
        dst = torch.empty(n, dtype=torch.uint8, device="cuda:1")
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        for r in range(3):
            G.check(ctx.get_into(G.fn(1, 2, 1), oid, dst.data_ptr(), n, s1.cuda_stream)[0], "get_into")
        reps = 20 if n <= (256 << 20) else 5
        a.record(s1)
        for r in range(reps):
            G.check(ctx.get_into(G.fn(1, 2, 1), oid, dst.data_ptr(), n, s1.cuda_stream)[0], "get_into")
        b.record(s1)
        b.synchronize()
        st, bad, _ = G.test_verify(dst.data_ptr(), n, 99, 0, 0)
        assert st == 0 and bad == 0
        gbps = reps * n / (a.elapsed_time(b) / 1e3) / 1e9
        res[f"{mode}_{n}"] = {"GBps": round(gbps, 1), "frac_of_900": round(gbps / 900, 3)}
        ctx.free(G.fn(1, 1, 0), oid)
        del dst
        torch.cuda.empty_cache()
    ctx.close()
print(json.dumps(res))
