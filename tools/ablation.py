"""Ablation (Fig. 16) and GPU-memory overhead (Fig. 20c)
on one B200 with two logical GPUs (synth.calib.virtual(2)).

Configurations (flags of the same library):
  full      -- GROUTER
  -ES       -- elastic storage off: GROUTER_NO_POOL, every object / lease its
               own cudaMalloc, cudaFree after its GPU work (L248)
  -BH       -- bandwidth harvesting off: GROUTER_NO_MULTIPATH (host->GPU over
               the destination's own link only; on one B200 both logical
               routes share the one physical link, so this isolates the
               relay hop's cost, not PCIe parallelism)
  -ES-BH    -- both
  -UF       -- unified framework off: GROUTER_HOST_CENTRIC, a GPU -> other-GPU
               copy goes through pinned host memory (D2H then H2D, R49; the
               host-centric passing of L90)
  -ES-BH-UF -- all three
(TA, topology-aware scheduling, only changes route sets where GPUs share a
PCIe switch: measured by bench.py N>1 `striped_no_topology`.)

Workloads per request (full sizes of BASELINE.json configs 1 and 5):
  cfg1: cFn put of 38,535,168 B from pinned host (hint GPU0, consumers=1) ->
        gFn on GPU1 get_into its binding (D2D) -> object consumed
  cfg5: stage-A gFn on GPU0 allocs + fills + seals 32 x 33,554,432 B KV
        objects and a 67,108,864 B hidden state (consumers=1); stage-B gFn
        on GPU1 get_into's each into its binding -> objects consumed
Reported: request latency p50/p99 (host clock, request issue -> consumer
stream drained), req/s, and pool footprint: peak/mean `mapped` (physical
pool pages) against the peak demand (`used` while a request's objects are
live); -ES maps nothing (its cudaMalloc buffers are the demand itself);
and the process CPU time over wall time while requests run (Fig. 20b
analog: the caller thread spins while it waits for its bytes, so ~1 core
is the floor for a blocking client).
usage: python tools/ablation.py OUT.json"""
import json
import sys
import time

sys.path.insert(0, ".")
import torch  # noqa: E402

from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G  # noqa: E402
from synth.calib import virtual  # noqa: E402

MiB = 1 << 20
N1 = 38_535_168
KV, HS, LAYERS = 33_554_432, 67_108_864, 32


def pct(xs, q):
    xs = sorted(xs)
    return xs[max(0, min(len(xs) - 1, -(-len(xs) * q // 100) - 1))]


def run(flags, workload, reqs):
    calib = virtual(2)
    ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=512 << 20, pool_cap=[G.UNLIMITED] * 2,
                                    flags=flags))
    s = torch.cuda.Stream()
    lat, mapped = [], []
    mid = []            # demand while the request's objects are live

    def sample():
        st = ctx.stats()
        mid.append(st.used[0] + st.used[1])
    try:
        if workload == "cfg1":
            host = torch.empty(N1, dtype=torch.uint8, pin_memory=True)
            dst = torch.empty(N1, dtype=torch.uint8, device="cuda")
            cfn, gfn = G.fn(1, 1, G.HOST), G.fn(1, 2, 1)

            def request():
                st, oid = ctx.put(cfn, host.data_ptr(), N1, 0, 1)
                G.check(st, "put")
                sample()
                G.check(ctx.get_into(gfn, oid, dst.data_ptr(), N1, s.cuda_stream)[0], "get_into")
                s.synchronize()
        else:
            sizes = [KV] * LAYERS + [HS]
            dsts = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in (KV, HS)]
            fa, fb = G.fn(2, 1, 0), G.fn(2, 2, 1)

            def request():
                oids = []
                for n in sizes:
                    st, buf, oid = ctx.alloc(fa, n, G.NOHINT, 1)
                    G.check(st, "alloc")
                    G.check(G.test_fill(buf, n, 77, 0, s.cuda_stream), "fill")
                    G.check(ctx.seal(fa, oid, s.cuda_stream), "seal")
                    oids.append(oid)
                sample()
                for n, oid in zip(sizes, oids):
                    d = dsts[1] if n == HS else dsts[0]
                    G.check(ctx.get_into(fb, oid, d.data_ptr(), n, s.cuda_stream)[0], "get_into")
                s.synchronize()
        for _ in range(3):
            request()
        c0, w0 = time.process_time(), time.perf_counter()
        for _ in range(reqs):
            t = time.perf_counter()
            request()
            lat.append((time.perf_counter() - t) * 1e6)
            st = ctx.stats()
            mapped.append(st.mapped[0] + st.mapped[1])
        cpu = (time.process_time() - c0) / (time.perf_counter() - w0)
        G.check(ctx.sync(), "sync")
    finally:
        ctx.close()
    tot = sum(lat) / 1e6
    return {"p50_us": round(pct(lat, 50), 1), "p99_us": round(pct(lat, 99), 1),
            "req_s": round(reqs / tot, 1), "mapped_peak_MiB": max(mapped) >> 20,
            "mapped_mean_MiB": round(sum(mapped) / len(mapped) / MiB, 1),
            "demand_peak_MiB": max(mid) >> 20, "requests": reqs,
            "overhead_x": round(max(mapped) / max(1, max(mid)), 2),
            "cpu_cores": round(cpu, 2)}


def main():
    G.load()
    cfgs = {"full": 0, "-ES": G.NO_POOL, "-BH": G.NO_MULTIPATH, "-ES-BH": G.NO_POOL | G.NO_MULTIPATH,
            "-UF": G.HOST_CENTRIC, "-ES-BH-UF": G.NO_POOL | G.NO_MULTIPATH | G.HOST_CENTRIC}
    out = {"gpu": torch.cuda.get_device_name(0), "what": __doc__.split("\n")[0], "results": {}}
    for wl, reqs in (("cfg1", 100), ("cfg5", 12)):
        for name, fl in cfgs.items():
            r = run(fl, wl, reqs)
            out["results"].setdefault(wl, {})[name] = r
            print(wl, name, r, flush=True)
    path = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/ablation.json"
    json.dump(out, open(path, "w"), indent=1)
    print("wrote", path)


if __name__ == "__main__":
    main()
