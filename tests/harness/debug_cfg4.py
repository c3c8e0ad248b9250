import sys
sys.path.insert(0, ".")
import faulthandler
faulthandler.dump_traceback_later(120, exit=True)
from oracle import runner as orun
from synth import calib as C, traces as T
from tests.lib_runner import LibRunner, compare
from synth.payload import payload
import numpy as np
calib = C.virtual(2)
ops = T.cfg4(2, rounds=1, scale=64)
orc = orun.run(ops, calib, keep_bytes=True)
for replay in (True, False):
    r = LibRunner(calib, replay=replay, keep_bytes=True)
    out = r(ops)
    for x in out["records"]:
        if "buf" in x or "ptr" in x:
            print("  rec", x["i"], x["op"], ops[x["i"]]["fn"], hex(x.get("buf", 0) or x.get("ptr", 0)), flush=True)
    r.close()
    for o, l in zip(orc["records"], out["records"]):
        if o["op"] == "get" and o["status"] == "OK":
            ok = np.array_equal(o["bytes"], l["bytes"])
            if not ok:
                bad = np.nonzero(o["bytes"] != l["bytes"])[0]
                # which payload seed does the lib data match?
                src_op = ops[ops[o["i"]]["ref"]]
                print("replay", replay, "op", o["i"], ops[o["i"]]["fn"], "ref", ops[o["i"]]["ref"], src_op["op"], src_op["fn"], "nbad", bad.size, "first", bad[0], "n", o["n"], flush=True)
                for j, op2 in enumerate(ops):
                    if op2["op"] in ("put", "alloc") and op2["n"] == o["n"]:
                        if np.array_equal(payload(op2["seed"], 64), l["bytes"][:64]):
                            print("    lib bytes == payload of op", j, op2["op"], op2["fn"], flush=True)
    print("dispatch", [(d["kind"], d["dev"], d["tenant"], d["chunks"]) for d in out["dispatch"]][:40], flush=True)
    try:
        compare(orc, out, check_dispatch=replay)
        print("replay", replay, "OK")
    except AssertionError as e:
        print("replay", replay, "FAIL", str(e)[:300])
