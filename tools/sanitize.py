"""Small workload for compute-sanitizer: every copy-engine variant over aligned
and misaligned chunk lists, plus a replay trace through the full library."""
import os
import sys
sys.path.insert(0, ".")
import random
import torch
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G
from synth import calib as C, traces as T
G.load()
MiB = 1 << 20
for tma in (False, True):
    for so, do in ((0, 0), (3, 3), (1, 0), (7, 13)):
        n = 1 * MiB + 12345
        src = torch.empty(n + 64, dtype=torch.uint8, device="cuda")
        dst = torch.empty(n + 64, dtype=torch.uint8, device="cuda")
        G.check(G.test_fill(src.data_ptr() + so, n, 5, 0, 0))
        cuts = sorted(random.Random(so).sample(range(1, n), 4))
        b = [0] + cuts + [n]
        G.check(G.test_copy(dst.data_ptr() + do, src.data_ptr() + so, [(x, y - x, 0, 0) for x, y in zip(b, b[1:])], tma=tma))
        torch.cuda.synchronize()
        st, bad, _ = G.test_verify(dst.data_ptr() + do, n, 5, 0, 0)
        assert bad == 0
from tests.lib_runner import LibRunner
from oracle import runner as orun
from tests.lib_runner import compare
calib = C.virtual(2)
ops = T.cfg2(2, requests=2, scale=64) + []
r = LibRunner(calib, replay=True, keep_bytes=True)
out = r(ops)
r.close()
compare(orun.run(ops, calib, keep_bytes=True), out)
print("sanitize workload OK", os.environ.get("GR_COPY", "default"))
