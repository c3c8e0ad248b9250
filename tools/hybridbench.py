"""Same-GPU cold copy of 38.5 MB split between the SM copy kernel (stream A)
and the copy engine (stream B) running concurrently; throughput mode."""
import sys
sys.path.insert(0, ".")
import torch
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G
G.load()
n = 38_535_168
nbuf = 24
bufs = [torch.empty(n, dtype=torch.uint8, device="cuda") for _ in range(nbuf)]
A, B = torch.cuda.Stream(), torch.cuda.Stream()
C2 = 2 << 20
for frac in (1.0, 0.0, 0.8, 0.7, 0.6, 0.5, 0.4):
    k = int(n * frac) // 4096 * 4096
    reps = 100
    def one(i):
        d, s = bufs[i % nbuf], bufs[(i + 7) % nbuf]
        if k:
            ch = [(o, min(C2, k - o), 0, 0) for o in range(0, k, C2)]
            G.check(G.test_copy(d.data_ptr(), s.data_ptr(), ch, stream=A.cuda_stream))
        if k < n:
            with torch.cuda.stream(B):
                d[k:].copy_(s[k:])
    for i in range(6):
        one(i)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(A)
    B.wait_event(a)
    for i in range(reps):
        one(i)
        ev = torch.cuda.Event()
        ev.record(B)
        A.wait_event(ev)          # next iteration starts after both halves
        ev2 = torch.cuda.Event()
        ev2.record(A)
        B.wait_event(ev2)
    b.record(A)
    b.synchronize()
    us = a.elapsed_time(b) * 1e3 / reps
    print(f"kernel share {frac:.1f}: {us:.2f} us per 38.5 MB copy, {2*n/us/1e6:.2f} TB/s rw", flush=True)
