"""Cold-cache microbenchmark of the gr_copy kernel variants (same-GPU HBM
copy) vs torch copy_.  Sources and destinations rotate through > L2 bytes.
Usage: python tools/copybench.py [variants...]"""
import os
import subprocess
import sys
import json
sys.path.insert(0, ".")

SIZES = [4 << 10, 256 << 10, 2 << 20, 38_535_168, 256 << 20, 1 << 30]


def child(variant):
    import torch
    from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G
    G.load()
    out = {}
    for n in SIZES:
        nbuf = max(2, min(16, (768 << 20) // n + 1))        # > L2 worth of buffers
        bufs = [torch.empty(n, dtype=torch.uint8, device="cuda") for _ in range(nbuf)]
        C = 2 << 20
        chunks = [(o, min(C, n - o), 0, 0) for o in range(0, n, C)]
        s = torch.cuda.current_stream().cuda_stream

        def run(i):
            d, src = bufs[i % nbuf], bufs[(i + 1) % nbuf]
            if variant == "torch":
                d.copy_(src)
            else:
                for k in range(0, len(chunks), 128):
                    G.check(G.test_copy(d.data_ptr(), src.data_ptr(), chunks[k:k + 128], stream=s))
        reps = 10 if n >= (256 << 20) else 100
        for i in range(5):
            run(i)
        # throughput mode: back-to-back launches between two events
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for i in range(reps):
            run(i)
        b.record()
        b.synchronize()
        us = a.elapsed_time(b) * 1e3 / reps
        out[n] = {"us": round(us, 2), "TBps_rw": round(2 * n / us / 1e6, 3)}
        del bufs
        torch.cuda.empty_cache()
    print(json.dumps({"variant": variant, "res": out}), flush=True)


if __name__ == "__main__":
    if len(sys.argv) > 1 and sys.argv[1] == "--child":
        child(sys.argv[2])
    else:
        for name in (sys.argv[1:] or ["torch", "ldst8", "wv8", "tmas4"]):
            env = dict(os.environ, GR_COPY=name)
            subprocess.run([sys.executable, __file__, "--child", name], env=env, timeout=300)
