"""Workflow-level measurements on one B200.

cfg4  8 tenants (workflows) with weights 1,1,2,2,4,4,8,8 share GPU0's
      host->GPU engine: each tenant's CPU function loops blocking puts of a
      38,535,168 B tensor (hint GPU0) for T seconds; per-tenant GB/s and the
      share error |x_t/sum x - w_t/sum w| / (w_t/sum w) (pass <= 10%), plus a
      run with all weights 1 (no partitioning) for the Fig. 17 analog: the
      w=8 tenant's put latency alone vs with the others.
cfg5  LLM pipeline (Llama-3-8B public shapes): per request stage A allocs 32
      KV objects of 33,554,432 B + 67,108,864 B hidden states on GPU0, stage
      B (same GPU) gets them into its own buffers in queue order; pool limit
      = 10% / 1% of the working set; queue-aware (next_use = queue position)
      vs LRU (no hints).  Per-request latency p50/p99, spilled bytes, req/s.
"""
import json
import sys
import threading
import time

sys.path.insert(0, ".")

import torch  # noqa: E402

from paper_conf_eurosys_wulywdyfwwj26_b200 import _build  # noqa: E402
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G  # noqa: E402
from synth.calib import b200_hgx  # noqa: E402

MiB = 1 << 20
N1 = 38_535_168


def pct(xs, q):
    xs = sorted(xs)
    return xs[max(0, min(len(xs) - 1, -(-len(xs) * q // 100) - 1))] if xs else None


def mkctx(h2d_Bps=None, **kw):
    c = b200_hgx(1)
    c["device_map"] = [0]
    if h2d_Bps:
        c["h2d_Bps"] = [h2d_Bps]
    return G.Ctx(G.config_from_calib(c, **kw))


def cfg4(seconds=3.0, weights=(1, 1, 2, 2, 4, 4, 8, 8), slos=None, h2d_Bps=None):
    ctx = mkctx(h2d_Bps=h2d_Bps, host_store_bytes=256 * MiB, pool_cap=[G.UNLIMITED])
    T = len(weights)
    for t, w in enumerate(weights):
        if slos:
            G.check(ctx.set_tenant_slo(100 + t, *slos[t]), "slo")
        else:
            ctx.set_tenant_weight(100 + t, w)
    srcs = [torch.empty(N1, dtype=torch.uint8, pin_memory=True) for _ in range(T)]
    done = [0] * T
    lat = [[] for _ in range(T)]
    stop = [False]
    start = threading.Barrier(T + 1)

    def worker(t):
        f = G.fn(100 + t, 1, G.HOST)
        start.wait()
        while not stop[0]:
            t0 = time.perf_counter()
            st, oid = ctx.put(f, srcs[t].data_ptr(), N1, 0, 0)
            lat[t].append(time.perf_counter() - t0)
            if st == G.OK:
                ctx.free(f, oid)
                done[t] += 1

    ths = [threading.Thread(target=worker, args=(t,)) for t in range(T)]
    for th in ths:
        th.start()
    start.wait()
    t0 = time.perf_counter()
    time.sleep(seconds)
    # the library's real-time rate monitor (L197) over the last second, while backlogged
    monitor = [ctx.tenant_rate(100 + t, 1_000_000_000) for t in range(T)]
    stop[0] = True
    for th in ths:
        th.join()
    dt = time.perf_counter() - t0
    gbps = [d * N1 / dt / 1e9 for d in done]
    tot, wsum = sum(gbps), sum(weights)
    err = [abs(g / tot - w / wsum) / (w / wsum) for g, w in zip(gbps, weights)] if tot else []
    ctx.close()
    return {"weights": list(weights), "seconds": dt, "puts": done, "GBps": [round(g, 2) for g in gbps],
            "aggregate_GBps": round(tot, 2), "share_error": [round(e, 3) for e in err],
            "max_share_error": round(max(err), 3) if err else None,
            "p50_ms": [round(pct(l, 50) * 1e3, 2) if l else None for l in lat],
            "p99_ms": [round(pct(l, 99) * 1e3, 2) if l else None for l in lat],
            "monitor_GBps": [round(r / 1e9, 2) for r, _, _ in monitor],
            "monitor_rate_least_GBps": [round(q / 1e9, 3) for _, q, _ in monitor],
            "monitor_at_least": [r >= q for r, q, _ in monitor]}


def cfg4_slo(seconds=3.0, bw=53e9):
    """Transfer rate control (L193-L197, L227): 8 CPU tenants loop blocking
    puts of 38,535,168 B; tenant t must finish each put within budget_t
    (SLO = 2x inference time, L193, so budget = slo - infer = infer).  With
    SLO-derived weights vs all weights 1: per-tenant p99 put latency vs budget."""
    budgets_ms = [3, 4, 6, 8, 12, 16, 24, 32]
    slos = [(N1, int(2 * b * 1e6), int(b * 1e6)) for b in budgets_ms]
    res = {"budgets_ms": budgets_ms, "bw_all_GBps": bw / 1e9,
           "rate_least_GBps": [round(N1 / (b / 1e3) / 1e9, 2) for b in budgets_ms]}
    for name, kw in (("slo", dict(slos=slos, h2d_Bps=int(bw))), ("equal", {})):
        r = cfg4(seconds, weights=(1,) * 8, **kw)
        r["met"] = [p <= b for p, b in zip(r["p99_ms"], budgets_ms)]
        res[name] = r
    return res


def cfg4_isolation(seconds=2.0):
    """Fig. 17 analog: latency of a w=8 tenant alone, then next to 7 others
    with weights (partitioned) and with all weights 1 (unpartitioned)."""
    alone = cfg4(seconds, weights=(8,))
    part = cfg4(seconds, weights=(8, 1, 1, 1, 1, 1, 1, 1))
    flat = cfg4(seconds, weights=(1, 1, 1, 1, 1, 1, 1, 1))
    return {"alone_p50_ms": alone["p50_ms"][0], "weighted_p50_ms": part["p50_ms"][0],
            "unweighted_p50_ms": flat["p50_ms"][0], "alone_GBps": alone["GBps"][0],
            "weighted_GBps": part["GBps"][0], "unweighted_GBps": flat["GBps"][0]}


def cfg2(seconds=3.0, outstanding=4):
    """Config 2 (Traffic) at N = 1, data plane only: per request
    a decode cFn puts a 39,321,600 B frame (hint GPU0, PCIe H2D), the YOLO gFn
    gets it (zero copy: co-located), allocs + seals person and vehicle crops
    (K x 602,112 B, K ~ Poisson(4) clipped to [0, 32]), the recognition gFns get
    them (zero copy) and everyone releases.  `outstanding` closed-loop client
    threads (Q = 4 N); req/s, per-request latency, and the PCIe roofline of the
    frame put (39.3 MB per request at the probed link rate)."""
    import math
    import random
    FRAME, CROP = 39_321_600, 602_112
    ctx = mkctx(host_store_bytes=256 * MiB, pool_cap=[G.UNLIMITED])
    frames = [torch.empty(FRAME, dtype=torch.uint8, pin_memory=True) for _ in range(outstanding)]
    streams = [torch.cuda.Stream() for _ in range(outstanding)]
    lat = [[] for _ in range(outstanding)]
    done = [0] * outstanding
    stop = [False]
    start = threading.Barrier(outstanding + 1)

    def poisson(rng, lam=4.0):
        L, k, p = math.exp(-lam), 0, 1.0
        while True:
            p *= rng.random()
            if p <= L:
                return min(k, 32)
            k += 1

    def worker(t):
        rng = random.Random(2000 + t)
        s = streams[t].cuda_stream
        start.wait()
        i = 0
        while not stop[0]:
            wf = 10 + t * 100000 + i
            dec, yolo, rp, rv = G.fn(wf, 1, G.HOST), G.fn(wf, 2, 0), G.fn(wf, 3, 0), G.fn(wf, 4, 0)
            t0 = time.perf_counter()
            st, o = ctx.put(dec, frames[t].data_ptr(), FRAME, 0, 1)
            G.check(st, "put")
            st, fp, _ = ctx.get(yolo, o, s)
            G.check(st, "get")
            outs = []
            for k in (poisson(rng), poisson(rng)):
                st, buf, a = ctx.alloc(yolo, k * CROP, G.NOHINT, 1)
                G.check(st, "alloc")
                G.check(ctx.seal(yolo, a, s), "seal")
                outs.append(a)
            gets = [(rp, outs[0]), (rv, outs[1])]
            ptrs = []
            for f, a in gets:
                st, ptr, _ = ctx.get(f, a, s)
                G.check(st, "get crops")
                ptrs.append(ptr)
            G.check(ctx.release(yolo, o, fp, s), "release")
            for (f, a), ptr in zip(gets, ptrs):
                if ptr:                              # K = 0: an empty object has no lease (R36)
                    G.check(ctx.release(f, a, ptr, s), "release crops")
            streams[t].synchronize()
            lat[t].append(time.perf_counter() - t0)
            done[t] += 1
            i += 1

    ths = [threading.Thread(target=worker, args=(t,)) for t in range(outstanding)]
    for th in ths:
        th.start()
    start.wait()
    t0 = time.perf_counter()
    time.sleep(seconds)
    stop[0] = True
    for th in ths:
        th.join()
    dt = time.perf_counter() - t0
    all_lat = [x for l in lat for x in l]
    probe = G.probe([0], 256 * MiB)
    link = probe["h2d_Bps"][0]
    req_s = sum(done) / dt
    ctx.close()
    # the oracle on the same request structure (1 core)
    from oracle import runner as orun
    from synth import traces as TT
    from synth.calib import b200_hgx as hgx
    ops = TT.cfg2(1, requests=8)
    t1 = time.perf_counter()
    orun.run(ops, hgx(1))
    o_req_s = 8 / (time.perf_counter() - t1)
    return {"outstanding": outstanding, "seconds": round(dt, 3), "requests": sum(done),
            "req_per_s": round(req_s, 1), "p50_ms": round(pct(all_lat, 50) * 1e3, 3),
            "p99_ms": round(pct(all_lat, 99) * 1e3, 3),
            "roofline": {"bound": "pcie", "achieved_GBps": round(req_s * FRAME / 1e9, 2),
                         "peak_GBps": round(link / 1e9, 2), "frac": round(req_s * FRAME / link, 3),
                         "peak_source": "grouter_probe solo pinned H2D of this GPU"},
            "oracle_req_per_s": round(o_req_s, 1)}


def cfg5(requests=4, limit_frac=0.1, hints=True, layers=32):
    KV, HID = 33_554_432, 67_108_864
    page = 2 * MiB
    charge = lambda x: -(-x // page) * page
    ws = requests * (layers * charge(KV) + charge(HID))
    limit = int(ws * limit_frac) // page * page if limit_frac else G.UNLIMITED
    ctx = mkctx(host_store_bytes=ws + 512 * MiB, pool_cap=[G.UNLIMITED], pool_floor_bytes=64 * MiB)
    if limit_frac:
        G.check(ctx.set_pool_limit(0, limit), "limit")
    s = torch.cuda.Stream()
    scratch = torch.empty(HID, dtype=torch.uint8, device="cuda")
    objs = []
    t_start = time.perf_counter()
    for r in range(requests):
        A = G.fn(500 + r, 1, 0)
        mine = []
        for nb in [KV] * layers + [HID]:
            st, buf, oid = ctx.alloc(A, nb, G.NOHINT, 1)
            if st == G.ENOMEM:
                # larger than the pool limit: the producer keeps its own output
                # buffer and puts it by copy -> stored in host memory (R16)
                G.check(G.test_fill(scratch.data_ptr(), nb, r * 1000 + len(mine), 0, s.cuda_stream))
                st, oid = ctx.put(A, scratch.data_ptr(), nb, G.NOHINT, 1, s.cuda_stream)
                G.check(st, "put")
            else:
                G.check(st, "alloc")
                G.check(G.test_fill(buf, nb, oid, 0, s.cuda_stream))
                G.check(ctx.seal(A, oid, s.cuda_stream))
            if hints:
                ctx.set_next_use(oid, r)
            mine.append((oid, nb))
        objs.append(mine)
    dst = torch.empty(HID, dtype=torch.uint8, device="cuda")
    lat = []
    for r in range(requests):
        B = G.fn(500 + r, 2, 0)
        t0 = time.perf_counter()
        slow = []
        for j, (oid, nb) in enumerate(objs[r]):
            tc = time.perf_counter()
            st, n = ctx.get_into(B, oid, dst.data_ptr(), nb, s.cuda_stream)
            G.check(st, "get_into")
            if time.perf_counter() - tc > 2e-3:
                slow.append((j, round((time.perf_counter() - tc) * 1e3, 1)))
        ts = time.perf_counter()
        s.synchronize()
        lat.append(time.perf_counter() - t0)
        if slow or lat[-1] > 0.1:
            print(f"[cfg5 diag] request {r}: {lat[-1] * 1e3:.1f} ms, submit {1e3 * (ts - t0):.1f} ms, "
                  f"slow get_into calls (idx, ms) {slow}", file=sys.stderr, flush=True)
    total = time.perf_counter() - t_start
    stt = ctx.stats()
    out = {"requests": requests, "limit_frac": limit_frac, "queue_aware": hints,
           "working_set_GB": round(ws / 1e9, 3), "pool_limit_GB": round(limit / 1e9, 3) if limit_frac else None,
           "stageB_p50_ms": round(pct(lat, 50) * 1e3, 2), "stageB_p99_ms": round(pct(lat, 99) * 1e3, 2),
           "stageB_ms": [round(x * 1e3, 2) for x in lat],
           "spill_count": stt.spill_count, "spill_GB": round(stt.spill_bytes / 1e9, 3),
           "req_per_s": round(requests / total, 2)}
    ctx.close()
    return out


def cfg5_interleaved(requests=12, window=3, limit_frac=0.3, hints=True, restore=True,
                     layers=32, compute_ms=30.0, of_requests=None):
    """Fig. 18 analog: `window` requests in flight; stage B of
    request r reads its 33 objects (get_into), "computes" for compute_ms
    (host sleep: the model's inference time, during which the background
    restores run), then stage A of request r + window produces.  The pool
    limit is limit_frac of the in-flight working set."""
    KV, HID = 33_554_432, 67_108_864
    page = 2 * MiB
    charge = lambda x: -(-x // page) * page
    ws = window * (layers * charge(KV) + charge(HID))
    # the limit is limit_frac of the in-flight working set, or (of_requests)
    # of the SURVEY cfg5 working set of that many requests (8: 9.13 GB)
    base = ws if not of_requests else of_requests * (layers * charge(KV) + charge(HID))
    limit = int(base * limit_frac) // page * page
    flags = G.RESTORE if restore else 0
    ctx = mkctx(host_store_bytes=ws + 512 * MiB, pool_cap=[G.UNLIMITED], pool_floor_bytes=64 * MiB,
                flags=flags)
    G.check(ctx.set_pool_limit(0, limit), "limit")
    s = torch.cuda.Stream()
    dst = torch.empty(HID, dtype=torch.uint8, device="cuda")
    objs = {}

    def produce(r):
        A = G.fn(500 + r, 1, 0)
        mine = []
        for nb in [KV] * layers + [HID]:
            st, buf, oid = ctx.alloc(A, nb, G.NOHINT, 1)
            if st == G.ENOMEM:
                # larger than what the limit can hold: the producer puts its own
                # buffer by copy -> stored in host memory (R16)
                G.check(G.test_fill(dst.data_ptr(), nb, 7, 0, s.cuda_stream))
                st, oid = ctx.put(A, dst.data_ptr(), nb, G.NOHINT, 1, s.cuda_stream)
                G.check(st, "put")
            else:
                G.check(st, "alloc")
                G.check(G.test_fill(buf, nb, oid, 0, s.cuda_stream))
                G.check(ctx.seal(A, oid, s.cuda_stream))
            if hints:
                ctx.set_next_use(oid, r)
            mine.append((oid, nb))
        objs[r] = mine

    t_start = time.perf_counter()
    for r in range(window):
        produce(r)
    s.synchronize()
    lat, from_host = [], []
    for r in range(requests):
        B = G.fn(500 + r, 2, 0)
        where = [ctx.where(oid)[1] for oid, _ in objs[r]]
        from_host.append(sum(1 for w in where if w == G.HOST))
        t0 = time.perf_counter()
        for oid, nb in objs.pop(r):
            G.check(ctx.get_into(B, oid, dst.data_ptr(), nb, s.cuda_stream)[0], "get_into")
        s.synchronize()
        lat.append(time.perf_counter() - t0)
        time.sleep(compute_ms / 1e3)          # stage-B inference
        if r + window < requests:
            produce(r + window)
    total = time.perf_counter() - t_start
    stt = ctx.stats()
    out = {"requests": requests, "window": window, "limit_frac": limit_frac, "queue_aware": hints,
           "limit_of": f"{of_requests}-request cfg5 working set" if of_requests else f"{window}-request window",
           "restore": restore, "compute_ms": compute_ms, "pool_limit_GB": round(limit / 1e9, 3),
           "stageB_p50_ms": round(pct(lat, 50) * 1e3, 2), "stageB_p99_ms": round(pct(lat, 99) * 1e3, 2),
           "stageB_mean_ms": round(sum(lat) / len(lat) * 1e3, 2),
           "objects_read_from_host": sum(from_host),
           "spill_GB": round(stt.spill_bytes / 1e9, 3), "restore_GB": round(stt.restore_bytes / 1e9, 3),
           "req_per_s": round(requests / total, 2)}
    ctx.close()
    return out


def main():
    _build.build()
    G.load()
    res = {"gpu": torch.cuda.get_device_name(0)}
    out = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/workflows.json"

    def save():
        json.dump(res, open(out, "w"), indent=1)
    if len(sys.argv) > 2 and sys.argv[2] == "cfg2":
        res["cfg2"] = cfg2(3.0)
        print("cfg2", json.dumps(res["cfg2"]), flush=True)
        save()
        return
    if len(sys.argv) > 2 and sys.argv[2] == "slo":
        res["cfg4_slo"] = cfg4_slo(3.0)
        print("cfg4_slo", json.dumps(res["cfg4_slo"]), flush=True)
        save()
        return
    if len(sys.argv) > 2 and sys.argv[2] in ("cfg5i", "cfg5i_low"):
        res["cfg5_interleaved"] = []
        # Fig. 18 reports 10% and 1% of GPU memory; here: 30% / 10% of the
        # 3-request window, and 10% / 1% of SURVEY cfg5's 8-request working set (9.13 GB)
        runs = [(0.3, None), (0.1, None), (0.1, 8), (0.01, 8)] if sys.argv[2] == "cfg5i" else [(0.1, 8), (0.01, 8)]
        cfg5_interleaved(3, 3, 0.3, True, True)   # untimed warm-up: the first run's req/s held one-time costs
        for frac, of in runs:
            for hints, restore in ((True, True), (True, False), (False, False), (False, True)):
                r = cfg5_interleaved(12, 3, frac, hints, restore, of_requests=of)
                res["cfg5_interleaved"].append(r)
                print("cfg5i", json.dumps(r), flush=True)
                save()
        return
    res["cfg4"] = cfg4(3.0)
    print("cfg4", json.dumps(res["cfg4"]), flush=True)
    save()
    res["cfg4_isolation"] = cfg4_isolation(2.0)
    print("cfg4_isolation", json.dumps(res["cfg4_isolation"]), flush=True)
    save()
    res["cfg5"] = []
    for frac in (None, 0.1, 0.01):
        for hints in ((True, False) if frac else (True,)):
            r = cfg5(4, frac, hints)
            res["cfg5"].append(r)
            print("cfg5", json.dumps(r), flush=True)
            save()


if __name__ == "__main__":
    main()
