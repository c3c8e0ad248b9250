#!/bin/bash
# AddressSanitizer build of the host library under the concurrency
# stress and the real-time soak; CUDA needs protect_shadow_gap=0, leak
# checking is off (the CUDA runtime keeps allocations until exit).  The two-process
# IPC test is left out: its child process inherits the preload and cannot create
# a CUDA context under it ("device busy or unavailable").  Reports land
# in gpurun_out/asan/.
set -x
D=gpurun_out/asan
mkdir -p $D
python paper_conf_eurosys_wulywdyfwwj26_b200/_build.py --asan
# the product build too, before the preload (nvcc must not run under ASan)
python -c "from paper_conf_eurosys_wulywdyfwwj26_b200 import _build; _build.build()"
# libstdc++ preloaded too: the runtime must see it at start (the library throws C++ exceptions)
export LD_PRELOAD="$(gcc -print-file-name=libasan.so) $(gcc -print-file-name=libstdc++.so)" GROUTER_LIB=asan
export ASAN_OPTIONS="protect_shadow_gap=0:detect_leaks=0:halt_on_error=0:log_path=$D/asan"
# positive control (its own process: ASan stops it at the report)
ASAN_OPTIONS="protect_shadow_gap=0:detect_leaks=0:log_path=$D/control" python - <<'PY'
import ctypes, sys
sys.path.insert(0, ".")
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G
lib = G.load()
v = ctypes.c_int32()
lib.grouter_test_oob(ctypes.byref(v))
print("control returned (ASan inactive?)")
PY
GR_STRESS_OPS=200 timeout 1200 python -m pytest tests/test_gpu_concurrency.py -m gpu -q -p no:cacheprovider > $D/stress_pytest.txt 2>&1
echo stress_rc=$?
GR_SOAK_SEEDS=6 timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_ipc.py tests/test_gpu_autocap.py -m gpu -q -p no:cacheprovider \
  -k "random_traces_realtime or two_batches or forced_remote or ce_relay or sticky or two_contexts or stalled or background_refresh" > $D/soak_pytest.txt 2>&1
echo soak_rc=$?
tail -n 3 $D/stress_pytest.txt $D/soak_pytest.txt
ls $D
for f in $D/control* $D/asan*; do [ -e "$f" ] && echo "$f: $(grep -c 'ERROR: AddressSanitizer' $f)"; done
