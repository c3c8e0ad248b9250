"""Relay tail of a striped host->GPU put (VERDICT r01 Next #6), on one B200
with virtual routes: a cFn put of n bytes with hint GPU0 over R(0) = {0, 1}
(logical GPU1 = the same physical GPU: its share goes through GPU1's staging
ring and a forward launch), blocking, host-timed; beside it the same put
with GROUTER_NO_MULTIPATH (direct link only: no relay).  The relay tail is
the striped put's latency minus what its copy-engine work alone needs,
estimated by the direct put of the same bytes (both share the one PCIe
link here).  Run twice: per-chunk forward (default) and GR_SEGMENT_FWD=1
(round 1's one forward launch per round after all its copies)."""
import json
import os
import sys
import time

sys.path.insert(0, ".")
import torch  # noqa: E402

from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G  # noqa: E402
from synth import calib as C  # noqa: E402

G.load()
out = {"mode": "segment" if os.environ.get("GR_SEGMENT_FWD") else ("per-chunk" if os.environ.get("GR_CHUNK_FWD") else "grouped")}
for k in (2, 4):
    calib = C.virtual(k)
    for name, flags in (("striped", 0), ("direct", G.NO_MULTIPATH)):
        ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=256 << 20, pool_cap=[G.UNLIMITED] * k,
                                        flags=flags, pool_floor_bytes=64 << 20))
        for n in (38_535_168, 256 << 20):
            host = torch.empty(n, dtype=torch.uint8, pin_memory=True)
            st, plan = ctx.plan(G.HOST, 0, n)
            f = G.fn(1, 1, G.HOST)
            xs = []
            for r in range(25):
                t = time.perf_counter()
                st, oid = ctx.put(f, host.data_ptr(), n, 0, 0)
                dt = time.perf_counter() - t
                G.check(st, "put")
                ctx.free(f, oid)
                if r >= 5:
                    xs.append(dt * 1e6)
            xs.sort()
            out[f"virtual{k}_{name}_{n}"] = {"p50_us": round(xs[len(xs) // 2], 1),
                                             "routes": sorted({c[3] for c in plan}),
                                             "relayed_bytes": sum(c[1] for c in plan if c[3] != 0)}
            del host
        ctx.close()
    for n in (38_535_168, 256 << 20):
        s, d = out[f"virtual{k}_striped_{n}"], out[f"virtual{k}_direct_{n}"]
        out[f"virtual{k}_tail_{n}_us"] = round(s["p50_us"] - d["p50_us"], 1)
print(json.dumps(out))
