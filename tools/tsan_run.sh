#!/bin/bash
# Race detection of the host library: the ThreadSanitizer build of
# the same sources (libgrouter_tsan.so, GROUTER_LIB=tsan) under the 8-thread
# concurrency stress and the real-time random-trace soak, with a positive
# control (grouter_test_race must be reported) so a silent run means no race,
# not an inactive detector.  Run under gpurun; reports land in gpurun_out/tsan/.
set -x
D=gpurun_out/tsan
mkdir -p $D
python paper_conf_eurosys_wulywdyfwwj26_b200/_build.py --tsan
python -c "from paper_conf_eurosys_wulywdyfwwj26_b200 import _build; _build.build()"
export LD_PRELOAD=$(gcc -print-file-name=libtsan.so) GROUTER_LIB=tsan
TSAN_OPTIONS="halt_on_error=0 log_path=$D/control" python - <<'PY'
import ctypes, sys
sys.path.insert(0, ".")
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G
lib = G.load()
v = ctypes.c_int64()
G.check(lib.grouter_test_race(200000, ctypes.byref(v)), "race")
maps = open("/proc/self/maps").read()
print("control done, libtsan mapped:", "libtsan" in maps, "tsan lib mapped:", "libgrouter_tsan.so" in maps)
PY
TSAN_OPTIONS="report_signal_unsafe=0 halt_on_error=0 log_path=$D/stress" GR_STRESS_OPS=300 \
  timeout 1200 python -m pytest tests/test_gpu_concurrency.py -m gpu -q -p no:cacheprovider > $D/stress_pytest.txt 2>&1
echo stress_rc=$?
TSAN_OPTIONS="report_signal_unsafe=0 halt_on_error=0 log_path=$D/soak" GR_SOAK_SEEDS=8 \
  timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_autocap.py -m gpu -q -p no:cacheprovider \
  -k "random_traces_realtime or two_batches or forced_remote or background_refresh" > $D/soak_pytest.txt 2>&1
echo soak_rc=$?
for f in $D/stress_pytest.txt $D/soak_pytest.txt; do tail -n 3 $f; done
for f in $D/control* $D/stress* $D/soak*; do echo "$f: $(grep -c 'WARNING: ThreadSanitizer' $f 2>/dev/null)"; done
