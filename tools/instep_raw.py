"""Diagnostic: is the in-step event interval of a 38.5 MB D2D copy under 4
concurrent clients (tools/instep.py q4: ~42 us vs ~18 us alone) the
library's doing?  The same loop without the library: each client thread
does a blocking pinned H2D of 38.5 MB on its own stream, then an event-
bracketed device copy (torch copy_, or the library's kernel through
grouter_test_memcpy with GR=1) into its binding.  Q = 1 and 4.
  python tools/instep_raw.py
"""
import os
import sys
import threading

sys.path.insert(0, ".")
import torch  # noqa: E402

n = 38_535_168
hs = [torch.empty(n, dtype=torch.uint8, pin_memory=True) for _ in range(4)]
stage = [torch.empty(n, dtype=torch.uint8, device="cuda") for _ in range(4)]
bind = [torch.empty(n, dtype=torch.uint8, device="cuda") for _ in range(4)]
streams = [torch.cuda.Stream() for _ in range(4)]
h2d_streams = [torch.cuda.Stream() for _ in range(4)]


def run(q, total, out):
    def client(k):
        torch.cuda.set_device(0)
        s, hs_ = streams[k], h2d_streams[k]
        for i in range(k, total, q):
            with torch.cuda.stream(hs_):
                stage[k].copy_(hs[k], non_blocking=True)
            hs_.synchronize()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            with torch.cuda.stream(s):
                bind[k].copy_(stage[k])
            b.record(s)
            out.append((a, b))
    ths = [threading.Thread(target=client, args=(k,)) for k in range(q)]
    for t in ths:
        t.start()
    for t in ths:
        t.join()
    torch.cuda.synchronize()


for q in (1, 4, 1, 4):
    out = []
    run(q, 40, [])
    run(q, 200, out)
    us = [a.elapsed_time(b) * 1e3 for a, b in out]
    us.sort()
    print(f"Q={q}: torch D2D copy between events avg {sum(us) / len(us):.2f} us  p50 {us[len(us) // 2]:.2f}  "
          f"p90 {us[int(len(us) * 0.9)]:.2f}", flush=True)
