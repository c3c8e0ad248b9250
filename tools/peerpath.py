"""Diagnostic (not product code): cost of the cross-GPU dispatch path on one
B200.  A gFn on logical GPU1 get_into's objects resident on logical GPU0 of a
virtual 2-GPU topology (both logical GPUs = device 0).  Modes:
  direct  -- flags 0: same physical device, so the copy runs as one launch
             on the consumer's stream (the same-GPU product path);
  remote  -- GROUTER_FORCE_REMOTE: the launch a physical GPU pair takes (the
             source GPU's copy server, peer-branch kernel, completion by
             words / events on the consumer stream).
Per size: back-to-back GB/s (read + write bytes over HBM, so the per-launch
overhead shows ~10x larger than it would over NVLink) and single-call p50
(CUDA events on the consumer stream, host path included).
Env: PEERPATH_MODES=direct,remote (which modes), PEERPATH_PROFILE=1 (kernel
%globaltimer spans per size via GROUTER_PROFILE), PEERPATH_LEGB=1 (only the
bench's N >= 2 leg-B pattern: 20 objects round robin into 8 bindings).
Results: profiles/r02_peerpath.txt."""
import json
import os
import sys
import time

sys.path.insert(0, ".")
import torch  # noqa: E402

from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G  # noqa: E402
from synth import calib as C  # noqa: E402

G.load()
out = {}
PROF = G.PROFILE if os.environ.get("PEERPATH_PROFILE") else 0   # kernel %globaltimer stamps per launch
modes = [m for m in [("direct", 0 | PROF), ("remote", G.FORCE_REMOTE | PROF)]
         if m[0] in os.environ.get("PEERPATH_MODES", "direct,remote").split(",")]
for name, flags in ([] if os.environ.get("PEERPATH_LEGB") else modes):
    calib = C.virtual(2)
    ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=64 << 20, pool_cap=[G.UNLIMITED] * 2,
                                    flags=flags, pool_floor_bytes=64 << 20))
    s1 = torch.cuda.Stream()
    res = {}
    for n in (4096, 65536, 1 << 20, 4 << 20, 16 << 20, 38_535_168, 256 << 20, 1 << 30):
        reps = 40 if n <= (64 << 20) else 10
        src = torch.empty(n, dtype=torch.uint8, device="cuda")
        G.check(G.test_fill(src.data_ptr(), n, 4242, 0, 0))
        torch.cuda.synchronize()
        oids = []
        for _ in range(2):
            st, oid = ctx.put(G.fn(9, 1, 0), src.data_ptr(), n, G.NOHINT, 0, 0)
            G.check(st, "put")
            oids.append(oid)
        ctx.sync()
        dst = [torch.empty(n, dtype=torch.uint8, device="cuda") for _ in range(2)]
        f1 = G.fn(9, 2, 1)
        for i in range(3):
            G.check(ctx.get_into(f1, oids[i % 2], dst[i % 2].data_ptr(), n, s1.cuda_stream)[0], "get_into")
        s1.synchronize()
        st, bad, _ = G.test_verify(dst[0].data_ptr(), n, 4242, 0, 0)
        assert st == 0 and bad == 0, f"{name} {n}: {bad} bytes differ"
        lat = []
        for i in range(reps):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s1)
            ctx.get_into(f1, oids[i % 2], dst[i % 2].data_ptr(), n, s1.cuda_stream)
            b.record(s1)
            b.synchronize()
            lat.append(a.elapsed_time(b) * 1e3)
        lat.sort()
        ctx.sync()
        k0 = ctx.stats()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s1)
        for i in range(reps):
            ctx.get_into(f1, oids[i % 2], dst[i % 2].data_ptr(), n, s1.cuda_stream)
        b.record(s1)
        b.synchronize()
        ms = a.elapsed_time(b)
        ctx.sync()
        k1 = ctx.stats()
        res[n] = {"p50_us": round(lat[len(lat) // 2], 2), "b2b_us": round(ms * 1e3 / reps, 2),
                  "b2b_GBps_rw": round(2 * n * reps / (ms / 1e3) / 1e9, 1),
                  "b2b_launches_per_get": (k1.kernel_launches - k0.kernel_launches) / reps}
        if k1.timed_kernel_launches > k0.timed_kernel_launches:   # PEERPATH_PROFILE: the kernels' own spans
            res[n]["b2b_kernel_us_per_get"] = round((k1.timed_kernel_ns - k0.timed_kernel_ns) / 1e3 / reps, 2)
        for oid in oids:
            ctx.free(G.fn(9, 1, 0), oid)
        del src, dst
    st = ctx.stats()
    res["kernel_launches"] = st.kernel_launches
    res["rounds"] = st.rounds

    out[name] = res
    ctx.close()
if out:
    print(json.dumps(out))

# bench.py's N >= 2 leg-B pattern: 20 distinct 38.5 MB objects of logical GPU0
# get_into'd by GPU1 round robin into 8 bindings on one stream, back to back
if os.environ.get("PEERPATH_LEGB"):
    for name, flags in modes:
        ctx = G.Ctx(G.config_from_calib(C.virtual(2), host_store_bytes=64 << 20, pool_cap=[G.UNLIMITED] * 2,
                                        flags=flags, pool_floor_bytes=64 << 20))
        n = 38_535_168
        src = torch.empty(n, dtype=torch.uint8, device="cuda")
        G.check(G.test_fill(src.data_ptr(), n, 77, 0, 0))
        torch.cuda.synchronize()
        oids = [ctx.put(G.fn(1, 1, 0), src.data_ptr(), n, G.NOHINT, 0, 0)[1] for _ in range(20)]
        ctx.sync()
        binds = [torch.empty(n, dtype=torch.uint8, device="cuda") for _ in range(8)]
        s1 = torch.cuda.Stream()
        f1 = G.fn(1, 2, 1)

        def legb():
            for i, oid in enumerate(oids):
                G.check(ctx.get_into(f1, oid, binds[i % 8].data_ptr(), n, s1.cuda_stream)[0], "get_into")
        legb()
        s1.synchronize()
        k0 = ctx.stats()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s1)
        t0 = time.perf_counter()
        for _ in range(20):
            legb()
        th = time.perf_counter() - t0
        b.record(s1)
        b.synchronize()
        k1 = ctx.stats()
        out[f"legb_{name}"] = {"us_per_get": round(a.elapsed_time(b) * 1e3 / 400, 2),
                               "host_us_per_call": round(th * 1e6 / 400, 2),
                               "launches_per_get": (k1.kernel_launches - k0.kernel_launches) / 400}
        st, bad, _ = G.test_verify(binds[3].data_ptr(), n, 77, 0, 0)
        assert st == 0 and bad == 0
        ctx.close()
    print(json.dumps({k: v for k, v in out.items() if k.startswith("legb")}))
