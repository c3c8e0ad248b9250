"""Diagnostic (not product code): same-GPU get_into single-call latency between 256 KiB and 4 MiB
with the kernel (GR_SMALL_CE=65536, the product threshold) or the copy engine (GR_SMALL_CE=8388608)
moving the bytes; bench.py's sweep measurement at these sizes, a bare cudaMemcpyAsync beside it."""
import json
import os
import sys

sys.path.insert(0, ".")
import bench  # noqa: E402
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G  # noqa: E402

G.load()
K = 1 << 10
rows = bench.measure_sweep(G, 0, 6556.8, 55.5, sizes=[256 * K, 512 * K, 768 * K, 1024 * K, 1536 * K, 2048 * K,
                                                      3072 * K, 4096 * K], oracle=False)
print(json.dumps({"GR_SMALL_CE": os.environ.get("GR_SMALL_CE"),
                  "rows": [{"bytes": r["bytes"], "lib_p50": r["get_into"]["p50_us"],
                            "memcpy_p50": r["get_into"]["memcpy"]["p50_us"]} for r in rows]}))
