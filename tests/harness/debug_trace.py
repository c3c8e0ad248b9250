"""Step-by-step driver for one trace with per-op logging (debugging aid)."""
import faulthandler
import sys
import time

faulthandler.dump_traceback_later(90, exit=True)
sys.path.insert(0, ".")
import torch  # noqa: E402

from oracle import runner as orun  # noqa: E402
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G  # noqa: E402
from synth import calib as C  # noqa: E402
from tests.lib_runner import LibRunner, compare  # noqa: E402
from tests.test_oracle_model import _small_trace_ops  # noqa: E402

calib = C.b200_hgx(2, shared_pairs=False)
calib["device_map"] = [0, 0]
ops = _small_trace_ops()
orc = orun.run(ops, calib, host_store_bytes=64 << 20, pool_cap=[6 << 20, G.UNLIMITED], keep_bytes=True)
r = LibRunner(calib, replay=True, keep_bytes=True, host_store_bytes=64 << 20,
              pool_cap=[6 << 20, G.UNLIMITED])
try:
    out = r(ops)
    print("records", [(x["i"], x["status"], x.get("where"), x["victims"]) for x in out["records"]], flush=True)
    print("compare", compare(orc, out), flush=True)
except Exception as e:
    import traceback
    traceback.print_exc()
    print("last error:", G.last_error(), flush=True)
    print("words:", flush=True)
finally:
    r.close()
print("done", flush=True)
