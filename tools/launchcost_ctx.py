"""launch_copy cost in latency mode with and without a live grouter context
(diagnoses host-side interference from the library's threads/state)."""
import sys
import time
sys.path.insert(0, ".")
import ctypes as C
import torch
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G
from synth.calib import b200_hgx
lib = G.load()
s = torch.cuda.Stream()


def cost(kind):
    v = C.c_double(0)
    for rep in range(2):
        G.check(lib.grouter_test_launch_cost(kind, 300, 592, s.cuda_stream, C.byref(v)))
    return round(v.value, 2)


print("no ctx: idle launch_copy 38.5MB", cost(108), "PDL empty", cost(103), flush=True)
calib = b200_hgx(1)
calib["device_map"] = [0]
ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=256 << 20, pool_cap=[G.UNLIMITED]))
print("ctx alive: idle launch_copy 38.5MB", cost(108), "PDL empty", cost(103), flush=True)
h = torch.empty(4096, dtype=torch.uint8, pin_memory=True)
st, oid = ctx.put(G.fn(1, 1, -1), h.data_ptr(), 4096, 0, 0)
print("after a put: idle launch_copy 38.5MB", cost(108), "PDL empty", cost(103), flush=True)
time.sleep(0.2)
print("after 200 ms: idle launch_copy 38.5MB", cost(108), "PDL empty", cost(103), flush=True)
ctx.close()
print("ctx closed: idle launch_copy 38.5MB", cost(108), "PDL empty", cost(103), flush=True)
for k, name in ((208, "idle+50us launch_copy 38.5MB"), (203, "idle+50us PDL empty"), (204, "idle+50us empty no PDL"),
                (205, "idle+50us EventRecord"), (206, "idle+50us EventQuery")):
    print(name, cost(k), flush=True)
