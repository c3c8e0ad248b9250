"""Diagnoses intermittent stage-B stalls in cfg5 under a 10% pool limit:
per get_into host time, the object's location before the call, and the
time the caller then waits on its stream."""
import sys
import time
sys.path.insert(0, ".")
import torch
from paper_conf_eurosys_wulywdyfwwj26_b200 import _build
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G
from synth.calib import b200_hgx
MiB = 1 << 20
_build.build()
G.load()
KV, HID, layers, requests = 33_554_432, 67_108_864, 32, 4
page = 2 * MiB
charge = lambda x: -(-x // page) * page
ws = requests * (layers * charge(KV) + charge(HID))
for it in range(6):
    c = b200_hgx(1)
    c["device_map"] = [0]
    ctx = G.Ctx(G.config_from_calib(c, host_store_bytes=ws + 512 * MiB, pool_cap=[G.UNLIMITED],
                                    pool_floor_bytes=64 * MiB))
    G.check(ctx.set_pool_limit(0, int(ws * 0.1) // page * page), "limit")
    s = torch.cuda.Stream()
    objs = []
    ta = time.perf_counter()
    for r in range(requests):
        A = G.fn(500 + r, 1, 0)
        mine = []
        for nb in [KV] * layers + [HID]:
            st, buf, oid = ctx.alloc(A, nb, G.NOHINT, 1)
            G.check(st, "alloc")
            G.check(G.test_fill(buf, nb, oid, 0, s.cuda_stream))
            G.check(ctx.seal(A, oid, s.cuda_stream))
            ctx.set_next_use(oid, r)
            mine.append((oid, nb))
        objs.append(mine)
    tb = time.perf_counter()
    dst = torch.empty(HID, dtype=torch.uint8, device="cuda")
    slow = []
    per_req = []
    for r in range(requests):
        B = G.fn(500 + r, 2, 0)
        t0 = time.perf_counter()
        for j, (oid, nb) in enumerate(objs[r]):
            _, loc = ctx.where(oid)
            t = time.perf_counter()
            st, n = ctx.get_into(B, oid, dst.data_ptr(), nb, s.cuda_stream)
            dt = time.perf_counter() - t
            if dt > 2e-3:
                slow.append((r, j, loc, round(dt * 1e3, 1)))
        t1 = time.perf_counter()
        s.synchronize()
        per_req.append((round((t1 - t0) * 1e3, 1), round((time.perf_counter() - t1) * 1e3, 1)))
    st = ctx.stats()
    print(f"iter {it}: stageA {1e3 * (tb - ta):.0f} ms, per request (submit ms, drain ms) {per_req}, "
          f"slow calls (req, idx, loc, ms) {slow[:12]} n_slow={len(slow)} spills={st.spill_count}", flush=True)
    ctx.close()
