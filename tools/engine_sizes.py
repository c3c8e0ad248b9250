"""Same-GPU get_into per engine and size (SM copy kernel through the C ABI):
latency mode (one call on an idle GPU, p50 of 50, CUDA events on the
consumer stream) and throughput mode (back-to-back calls, rotating > L2
buffers).  Usage: python tools/engine_sizes.py [ENGINE ...]  (GR_COPY names)."""
import json
import os
import subprocess
import sys

sys.path.insert(0, ".")
MiB = 1 << 20
SIZES = [4 * MiB, 16 * MiB, 38_535_168, 64 * MiB, 128 * MiB, 256 * MiB, 1024 * MiB]


def child():
    import torch
    from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G
    from synth.calib import b200_hgx
    G.load()
    calib = b200_hgx(1)
    calib["device_map"] = [0]
    ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=64 << 20, pool_cap=[G.UNLIMITED]))
    f = G.fn(1, 2, 0)
    s = torch.cuda.Stream()
    out = {}
    for n in SIZES:
        k = max(2, min(8, (512 * MiB) // n + 1))
        objs = []
        for i in range(k):
            st, buf, oid = ctx.alloc(f, n, 0, 0)
            G.check(st, "alloc")
            G.check(ctx.seal(f, oid, 0), "seal")
            objs.append(oid)
        dsts = [torch.empty(n, dtype=torch.uint8, device="cuda") for _ in range(k)]
        for i in range(3):
            G.check(ctx.get_into(f, objs[i % k], dsts[i % k].data_ptr(), n, s.cuda_stream)[0])
        s.synchronize()
        lat = []
        for i in range(50):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            ctx.get_into(f, objs[i % k], dsts[(i + 1) % k].data_ptr(), n, s.cuda_stream)
            b.record(s)
            b.synchronize()
            lat.append(a.elapsed_time(b) * 1e3)
        lat.sort()
        reps = 40 if n <= 64 * MiB else 10
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        ce = os.environ.get("GR_SIZES_CE") == "1"     # baseline: cudaMemcpyAsync D2D (copy engine)
        srcs = [torch.empty(n, dtype=torch.uint8, device="cuda") for _ in range(k)] if ce else None
        if ce:
            with torch.cuda.stream(s):
                for i in range(3):
                    dsts[(i + 1) % k].copy_(srcs[i % k])
            a.record(s)
        for i in range(reps):
            if ce:
                with torch.cuda.stream(s):
                    dsts[(i + 1) % k].copy_(srcs[i % k])
            else:
                ctx.get_into(f, objs[i % k], dsts[(i + 1) % k].data_ptr(), n, s.cuda_stream)
        b.record(s)
        b.synchronize()
        us = a.elapsed_time(b) * 1e3 / reps
        out[n] = {"lat_p50_us": round(lat[25], 2), "tput_us": round(us, 2), "tput_TBps_rw": round(2 * n / us / 1e6, 3)}
        for oid in objs:
            ctx.free(f, oid)
        del dsts
        torch.cuda.empty_cache()
    ctx.close()
    print(json.dumps({"engine": "ce" if os.environ.get("GR_SIZES_CE") == "1" else os.environ.get("GR_COPY", "default"),
                      "res": out}), flush=True)


if __name__ == "__main__":
    if len(sys.argv) > 1 and sys.argv[1] == "--child":
        child()
    else:
        for e in sys.argv[1:] or ["default", "wv8", "tmas4"]:
            env = dict(os.environ)
            name, *extra = e.split(":")     # ENGINE[:ENV=VAL ...]
            env.update(kv.split("=", 1) for kv in extra)
            if name == "ce":
                env["GR_SIZES_CE"] = "1"
            elif name != "default":
                env["GR_COPY"] = name
            subprocess.run([sys.executable, __file__, "--child"], env=env, timeout=600)
