import sys
sys.path.insert(0, ".")
import ctypes as C
import torch
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G
lib = G.load()
s = torch.cuda.Stream()
for stream_name, st in (("torch stream", s.cuda_stream), ("legacy default", 0)):
    for kind in (0, 1, 2, 3, 4, 5, 6):
        for blocks in (592,):
            for rep in range(2):
                v = C.c_double(0)
                G.check(lib.grouter_test_launch_cost(kind, 2000, blocks, st or None, C.byref(v)))
            print(stream_name, "kind", kind, "blocks", blocks, "us/launch", round(v.value, 2), flush=True)
# torch's own launch cost for comparison
x = torch.empty(1, device="cuda")
import time
with torch.cuda.stream(s):
    for _ in range(100): x.add_(1)
    torch.cuda.synchronize()
    t = time.perf_counter()
    for _ in range(2000): x.add_(1)
    print("torch add_ us/launch", round((time.perf_counter() - t) * 1e6 / 2000, 2))
