import sys, os
sys.path.insert(0, ".")
import faulthandler
faulthandler.dump_traceback_later(200, exit=True)
from oracle import runner as orun
from synth import calib as C, traces as T
from tests.lib_runner import LibRunner, compare
import tests.lib_runner as LR
LR.wait_streams.__defaults__ = (8.0,)

def attempt(name, ops, replay=True, calib=None):
    calib = calib or C.virtual(2)
    orc = orun.run(ops, calib, keep_bytes=True)
    r = LibRunner(calib, replay=replay, keep_bytes=True)
    try:
        out = r(ops)
        compare(orc, out, check_dispatch=replay)
        print(name, "OK", out["stats"].kernel_launches, flush=True)
    except Exception as e:
        print(name, "FAIL", type(e).__name__, str(e)[:400], flush=True)
        print(r.ctx.dump()[:1500], flush=True)
    # leak the runner on failure (closing may block on parked streams)

MiB = 1 << 20
def mk(tenants, n=MiB, src_dev=1, dst_dev=0, weights=None, fill_get_order="all_alloc_first"):
    b = T.Builder(5)
    if weights:
        for t, w in zip(tenants, weights):
            b.weight(t, w)
    objs = []
    for t in tenants:
        f = T.fn(t, 1, src_dev)
        a = b.alloc(f, n, consumers=1); b.seal(f, a); objs.append(a)
    gs = [b.get(T.fn(t, 2, dst_dev), a) for t, a in zip(tenants, objs)]
    b.flush()
    for t, g in zip(tenants, gs):
        b.release(T.fn(t, 2, dst_dev), g)
    b.flush()
    return b.ops

which = sys.argv[1:] or ["a", "b", "c", "d", "e", "f"]
if "a" in which: attempt("a: 1 tenant d2d", mk([1]))
if "b" in which: attempt("b: 2 tenants d2d", mk([1, 2]))
if "c" in which: attempt("c: 2 tenants same-dev", mk([1, 2], src_dev=0, dst_dev=0), calib=dict(C.b200_hgx(1), device_map=[0]))
if "d" in which: attempt("d: 4 tenants weighted", mk([1, 2, 3, 4], weights=[1, 2, 4, 8]))
if "e" in which: attempt("e: cfg4 realtime", T.cfg4(2, rounds=1, scale=64), replay=False)
if "f" in which: attempt("f: 2 tenants d2d realtime", mk([1, 2]), replay=False)
print("end", flush=True)
os._exit(0)
