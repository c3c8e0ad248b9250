"""One cold 38.5 MB copy with torch (cudaMemcpy D2D) and with gr_copy (GR_COPY
variant) for side-by-side ncu captures."""
import sys
sys.path.insert(0, ".")
import torch
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G
G.load()
n = 38_535_168
bufs = [torch.empty(n, dtype=torch.uint8, device="cuda") for _ in range(6)]
C = 2 << 20
chunks = [(o, min(C, n - o), 0, 0) for o in range(0, n, C)]
s = torch.cuda.current_stream().cuda_stream
for i in range(4):
    bufs[(i + 1) % 6].copy_(bufs[i % 6])
    G.check(G.test_copy(bufs[(i + 3) % 6].data_ptr(), bufs[(i + 2) % 6].data_ptr(), chunks, stream=s))
torch.cuda.synchronize()
