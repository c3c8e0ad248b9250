"""cfg5 (10% / 1% pool limit) repeated: stage-B latency per request (diagnostics)."""
import json
import sys
sys.path.insert(0, ".")
sys.argv = sys.argv[:1]
from tools import workflows as W  # noqa: E402
W._build.build()
W.G.load()
for rep in range(3):
    for frac, hints in ((0.1, True), (0.1, False), (0.01, True)):
        r = W.cfg5(4, frac, hints)
        print(json.dumps({k: r[k] for k in ("limit_frac", "queue_aware", "stageB_ms", "spill_count", "req_per_s")}),
              flush=True)
