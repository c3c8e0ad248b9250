"""cfg3 point-to-point size sweep on one B200: p50/p99 latency
and GB/s per size, through the C ABI, next to baselines on the same buffers.

patterns (1 GPU):
  get_into_same   gFn get_into of an HBM-resident object (SM copy kernel; HBM)
  zero_copy_get   gFn get of a co-located object + release (no bytes move)
  put_h2d         cFn put(hint=GPU0) from pinned host (copy engines, R(0)={0})
  get_d2h         cFn get of a GPU object into a host lease (D2H engine)
baselines: cudaMemcpyAsync D2D (torch copy_), pinned H2D / D2H (torch copy_)
Also the calibration probe of this GPU.  Writes one JSON document.
"""
import json
import statistics
import sys
import time

sys.path.insert(0, ".")

import torch  # noqa: E402

from paper_conf_eurosys_wulywdyfwwj26_b200 import _build  # noqa: E402
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G  # noqa: E402
from synth.calib import b200_hgx  # noqa: E402

MiB = 1 << 20
SIZES = [4096 * 4 ** i for i in range(10)] + [2 * MiB - 1, 2 * MiB + 1, 38_535_168]


def samples_for(n):
    return 200 if n <= 64 * MiB else (50 if n <= 256 * MiB else 30)


def pct(xs, q):
    xs = sorted(xs)
    k = max(0, min(len(xs) - 1, -(-len(xs) * q // 100) - 1))
    return xs[k]


def summarize(n, lat_us):
    p50, p99 = pct(lat_us, 50), pct(lat_us, 99)
    return {"n": n, "p50_us": round(p50, 2), "p99_us": round(p99, 2), "GBps": round(n / p50 / 1e3, 2),
            "samples": len(lat_us)}


def dev_timed(stream, fn, reps):
    out = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        fn()
        b.record(stream)
        b.synchronize()
        out.append(a.elapsed_time(b) * 1e3)
    return out


def host_timed(fn, reps):
    out = []
    for _ in range(reps):
        t = time.perf_counter()
        fn()
        out.append((time.perf_counter() - t) * 1e6)
    return out


def oracle_get_into(n, budget_s=0.4):
    """The oracle's get_into of an n-byte GPU object (np.copyto between
    simulated buffers), single-threaded, on this box's host."""
    import numpy as np
    from oracle.model import Oracle
    from synth.calib import b200_hgx as hgx
    orc = Oracle(hgx(1))
    src = np.zeros(n, np.uint8)
    st, out = orc.put({"wf": 1, "fid": 1, "dev": 0}, src, n, -2, 0)
    oid = out["oid"]
    dst = np.empty(n, np.uint8)
    f = {"wf": 1, "fid": 2, "dev": 0}
    lat = []
    t_end = time.perf_counter() + budget_s
    while len(lat) < 3 or (time.perf_counter() < t_end and len(lat) < 200):
        t = time.perf_counter()
        orc.get_into(f, oid, dst, n)
        lat.append((time.perf_counter() - t) * 1e6)
    return summarize(n, lat)


def oracle_put_h2d(n, striped, budget_s=0.4):
    """The oracle's cFn put with a GPU0 hint on the 8-GPU HGX calibration
    (R(0) = 4 uplink groups): single-threaded (`Oracle.put` as it stands:
    plan + one np.copyto), or the same O6 plan executed with one thread per
    route path (SURVEY §8(d) striped variant, T = |R(0)| capped at the cores)."""
    import os
    from concurrent.futures import ThreadPoolExecutor

    import numpy as np
    from oracle.model import Oracle
    from oracle.splitter import CHUNK, plan_h2d
    from synth.calib import b200_hgx as hgx
    calib = hgx(8)
    src = np.zeros(n, np.uint8)
    lat = []
    t_end = time.perf_counter() + budget_s
    if not striped:
        orc = Oracle(calib)
        f = {"wf": 1, "fid": 1, "dev": -1}
        while len(lat) < 3 or (time.perf_counter() < t_end and len(lat) < 200):
            t = time.perf_counter()
            st, out = orc.put(f, src, n, 0, 0)
            lat.append((time.perf_counter() - t) * 1e6)
            orc.free(f, out["oid"])
        return dict(summarize(n, lat), threads=1)
    dst = np.empty(n, np.uint8)
    by = {}
    for c in plan_h2d(calib, 0, n, True, CHUNK):
        by.setdefault(c["route_gpu"], []).append((c["offset"], c["offset"] + c["bytes"]))
    T = max(1, min(len(by), len(os.sched_getaffinity(0))))

    def work(spans):
        for a, b in spans:
            np.copyto(dst[a:b], src[a:b])
    with ThreadPoolExecutor(T) as ex:
        while len(lat) < 3 or (time.perf_counter() < t_end and len(lat) < 200):
            t = time.perf_counter()
            list(ex.map(work, by.values()))
            lat.append((time.perf_counter() - t) * 1e6)
    return dict(summarize(n, lat), threads=T)


def main():
    _build.build()
    G.load()
    import os
    res = {"gpu": torch.cuda.get_device_name(0), "patterns": {}, "host_cores": len(os.sched_getaffinity(0))}
    res["probe"] = G.probe([0], 256 * MiB)
    calib = b200_hgx(1)
    calib["device_map"] = [0]
    ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=4 << 30, pool_cap=[G.UNLIMITED]))
    s = torch.cuda.Stream()
    cfn, gfn = G.fn(1, 1, G.HOST), G.fn(1, 2, 0)
    maxn = max(SIZES)
    host = torch.empty(maxn, dtype=torch.uint8, pin_memory=True)
    dsts = [torch.empty(maxn, dtype=torch.uint8, device="cuda") for _ in range(2)]
    pats = {k: [] for k in ["get_into_same", "zero_copy_get", "put_h2d", "get_d2h",
                            "base_memcpy_d2d", "base_h2d_pinned", "base_d2h_pinned"]}
    for n in SIZES:
        reps = samples_for(n)
        # object resident on GPU0
        st, oid = ctx.put(cfn, host.data_ptr(), n, 0, 0)
        G.check(st, "put")
        i = [0]

        def gi():
            st, _ = ctx.get_into(gfn, oid, dsts[i[0] & 1].data_ptr(), n, s.cuda_stream)
            i[0] += 1
        for _ in range(5):
            gi()
        pats["get_into_same"].append(summarize(n, dev_timed(s, gi, reps)))

        def zc():
            st, ptr, nn = ctx.get(gfn, oid, s.cuda_stream)
            ctx.release(gfn, oid, ptr, s.cuda_stream)
        pats["zero_copy_get"].append(summarize(n, host_timed(zc, reps)))

        def d2h():
            st, ptr, nn = ctx.get(cfn, oid, 0)
            ctx.release(cfn, oid, ptr, 0)
        for _ in range(3):
            d2h()
        pats["get_d2h"].append(summarize(n, host_timed(d2h, reps)))

        def h2d():
            st, o2 = ctx.put(cfn, host.data_ptr(), n, 0, 0)
            ctx.free(cfn, o2)
        for _ in range(3):
            h2d()
        pats["put_h2d"].append(summarize(n, host_timed(h2d, reps)))
        ctx.free(cfn, oid)
        # baselines on the same buffers
        src = dsts[0][:n]
        dst = dsts[1][:n]
        hb = host[:n]
        with torch.cuda.stream(s):
            pats["base_memcpy_d2d"].append(summarize(n, dev_timed(s, lambda: dst.copy_(src), reps)))
            pats["base_h2d_pinned"].append(summarize(n, dev_timed(s, lambda: dst.copy_(hb, non_blocking=True), reps)))
            pats["base_d2h_pinned"].append(summarize(n, dev_timed(s, lambda: hb.copy_(dst, non_blocking=True), reps)))
        pats.setdefault("oracle_get_into", []).append(oracle_get_into(n))
        pats.setdefault("oracle_put_h2d", []).append(oracle_put_h2d(n, False))
        pats.setdefault("oracle_put_striped", []).append(oracle_put_h2d(n, True))
        print(n, {k: v[-1]["p50_us"] for k, v in pats.items()}, flush=True)
    res["patterns"] = pats
    ctx.close()
    out = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/sweep.json"
    json.dump(res, open(out, "w"), indent=1)
    print("wrote", out)


if __name__ == "__main__":
    main()
