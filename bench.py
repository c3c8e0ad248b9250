#!/usr/bin/env python
"""bench.py -- GROUTER data-passing hot path on B200 (one JSON line).

metric (BASELINE.json): "p50/p99 data-passing latency & GB/s vs size; workflow
req/s at 1/2/4/8 B200".

value = workflow req/s of cfg1 (BASELINE configs[0]; reading R24): a CPU
function (cFn) puts a 38,535,168 B fp32 tensor (64x3x224x224, R25) from its
pinned host buffer with a placement hint for the producer GPU (striped H2D over
R(d); at one GPU the direct PCIe link), and the GPU function (gFn) gets it into
its fixed input binding (get_into: the consumer's input address is fixed,
e.g. a captured CUDA graph -- reading R51; the object is consumed and freed).
20 requests per step (the config's "20 puts/gets"), closed loop with Q = 4
requests outstanding, one client thread each.  Device-timed:
CUDA events on a timing stream that every consumer stream joins before and
after the K steps.  At N GPUs (torchrun, one process per GPU) every rank runs
the same flow with its consumer on the next GPU: put host -> GPU r (its own
PCIe link: every link carries its own rank's traffic), get_into on GPU r+1
(GPU r's SM copy kernel pushes the tensor over NVLink) -- a ring of disjoint
producer -> consumer pairs, weak scaling, no collective.

Also in the line:
  e2e          the same loop host-timed (wall clock) plus an 8 B D2H read of
               each delivered tensor (the step's result)
  latency_us   p50/p99 of single cfg1 requests on an idle GPU (R22: put call
               -> the consumer's data ready)
  roofline     gr_copy (the only kernel on the path) in leg B's own timed
               region: get_into of HBM-resident objects back to back, CUDA
               events on the stream the kernels run on / launches;
               algorithmic bytes = 2n (HBM read + write) at one GPU, n over
               NVLink at N > 1.  roofline.in_step: the same kernel timed per
               launch inside the workflow's region (isolated launches).
               roofline_step: the PCIe link that bounds the workflow
               (live-measured pinned H2D)
  sweep        cfg3 (iii)/(iv) at one GPU: per size 4 KiB..1 GiB, p50/p99 and
               GB/s of same-GPU get_into, cFn put (H2D), cFn get (D2H) and
               zero-copy get, each beside a bare cudaMemcpyAsync on the same
               buffers through the same binding, plus the oracle's get_into
  cfg2         BASELINE configs[1] (traffic monitoring) at one GPU: req/s of the
               frame put + zero-copy fan-out, wall clock
  cpu_baseline the oracle (oracle/, numpy memcpy on simulated buffers) on the
               same cfg1 request, single-threaded as it stands, plus the
               striped put variant (one thread per route of the 8-GPU HGX
               calibration's R(0))
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

N_BYTES = 64 * 3 * 224 * 224 * 4          # 38,535,168 (R25)
METRIC = "p50/p99 data-passing latency & GB/s vs size; workflow req/s at 1/2/4/8 B200"
NVL_PEAK = 900.0                           # GB/s per direction per GPU (north star roofline)
MiB = 1 << 20
WORKLOAD = ("cfg1 2-function workflow (BASELINE configs[0], R24): cFn put of a 38,535,168 B fp32 tensor from "
            "pinned host memory (hint GPU0: H2D) -> gFn on GPU0 get_into its fixed input binding (R51); "
            "20 requests/step, 4 outstanding")
WORKLOAD_N = ("cfg1 2-function workflow at N GPUs (R24): on every GPU r a cFn puts the 38,535,168 B tensor "
              "from pinned host memory into GPU r (its own PCIe link) and a gFn on GPU r+1 get_into's it "
              "(GPU r's SM kernel pushes it over NVLink); ring of disjoint pairs, 20 requests/step per GPU, "
              "4 outstanding per GPU")


def pct(xs, q):
    """Nearest-rank percentile (R26): the ceil(q/100 * m)-th smallest."""
    xs = sorted(xs)
    return xs[min(len(xs) - 1, max(0, -(-len(xs) * q // 100) - 1))] if xs else None


def host_info():
    """Host cores this process may use and the CPU model."""
    cores = len(os.sched_getaffinity(0))
    model = None
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for ln in out.splitlines():
            if ln.strip().startswith("Model name"):
                model = ln.split(":", 1)[1].strip()
                break
    except Exception:
        pass
    if not model:
        try:
            for ln in open("/proc/cpuinfo"):
                if ln.startswith("model name"):
                    model = ln.split(":", 1)[1].strip()
                    break
        except Exception:
            model = None
    return cores, model


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return d.get("hbm_gbs", 6650.0), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def _live_copy_peaks(dev: int) -> dict:
    """Same-box HBM copy figures beside the driver's MEASURED_PEAKS.json one
    (measured once, possibly on another box: 6,456-6,543 GB/s seen across
    boxes).  `torch_copy_2GiB` repeats the driver's recipe (b.copy_(a) over
    1 Gi bf16 elements, read + write bytes, best of 10, CUDA events);
    `torch_copy_38MB` is torch's copy at the bench's own size, back to back
    over 8 rotating 38.5 MB pairs (like the bench's bindings).  Plumbing-side
    context only: `roofline.peak` stays the MEASURED_PEAKS.json number."""
    import torch
    out = {}
    with torch.cuda.device(dev):
        a = torch.empty(1 << 30, dtype=torch.bfloat16, device=dev)
        b = torch.empty_like(a)
        a.fill_(1)
        best = None
        for _ in range(11):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(); b.copy_(a); e1.record(); e1.synchronize()
            ms = e0.elapsed_time(e1)
            best = ms if best is None else min(best, ms)
        out["torch_copy_2GiB"] = round(2 * a.numel() * 2 / (best * 1e6), 1)
        n = 38_535_168
        src = [a.view(torch.uint8)[i * n:(i + 1) * n] for i in range(8)]
        dst = [b.view(torch.uint8)[i * n:(i + 1) * n] for i in range(8)]
        reps = 400
        for i in range(16):
            dst[i % 8].copy_(src[i % 8])
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for i in range(reps):
            dst[i % 8].copy_(src[i % 8])
        e1.record(); e1.synchronize()
        out["torch_copy_38MB"] = round(2 * n * reps / (e0.elapsed_time(e1) * 1e6), 1)
        del a, b, src, dst
        torch.cuda.empty_cache()
    out["unit"] = "GB/s (read + write)"
    return out


class ClockSampler:
    """SM clocks / throttle reasons sampled DURING the timed region.

    NVML in a background thread every 2 ms (the default timed region is
    ~55 ms: an nvidia-smi subprocess spends that starting up); the thread's
    NVML calls release the GIL.  Falls back to `nvidia-smi -lms` when NVML is
    missing."""

    Q = ("index,clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int, period_s: float = 0.002):
        self.index = index
        self.p = None
        self.period = period_s
        self.nv = None
        try:
            import pynvml as nv
            import torch
            nv.nvmlInit()
            h = None
            try:
                pr = torch.cuda.get_device_properties(index)
                bus = f"{pr.pci_domain_id:08x}:{pr.pci_bus_id:02x}:{pr.pci_device_id:02x}.0"
                h = nv.nvmlDeviceGetHandleByPciBusId(bus)
            except Exception:
                h = nv.nvmlDeviceGetHandleByIndex(index)
            self.nv, self.h = nv, h
        except Exception:
            self.nv = None

    def _poll(self):
        nv, h = self.nv, self.h
        bits = [("hw_slowdown", nv.nvmlClocksEventReasonHwSlowdown),
                ("hw_thermal_slowdown", nv.nvmlClocksEventReasonHwThermalSlowdown),
                ("sw_thermal_slowdown", nv.nvmlClocksEventReasonSwThermalSlowdown),
                ("sw_power_cap", nv.nvmlClocksEventReasonSwPowerCap)]
        while not self.halt.is_set():
            try:
                self.sm.append(float(nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)))
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
                for name, b in bits:
                    if r & b:
                        self.reasons.add(name)
            except Exception as e:
                self.reasons.add(f"nvml error: {e}"[:60])
                return
            self.halt.wait(self.period)

    def start(self):
        if self.nv is not None:
            import threading
            self.sm, self.reasons = [], set()
            self.halt = threading.Event()
            self.mx = float(self.nv.nvmlDeviceGetMaxClockInfo(self.h, self.nv.NVML_CLOCK_SM))
            self.t = threading.Thread(target=self._poll, daemon=True)
            self.t.start()
            return
        self._start_smi()

    def _start_smi(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "50"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            time.sleep(0.3)   # let nvidia-smi start before the timed region
        except Exception:
            self.p = None

    def stop(self):
        if self.nv is not None:
            self.halt.set()
            self.t.join(timeout=5)
            return {"sm_mhz": statistics.median(self.sm) if self.sm else None, "sm_max_mhz": self.mx,
                    "samples": len(self.sm), "reasons": sorted(self.reasons), "source": "nvml, 2 ms"}
        if not self.p:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.12)
        self.p.terminate()
        out, _ = self.p.communicate(timeout=5)
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in out.strip().splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) < 7:
                continue
            try:
                sm.append(float(f[1]))
                mx = float(f[2])
            except ValueError:
                continue
            for nm, v in zip(names, f[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx,
                "samples": len(sm), "reasons": sorted(reasons)}


# ------------------------------------------------------------------ multi-rank plumbing (gloo-tested)
CPU_GROUP = [None]   # gloo group for waits that must not occupy the GPUs (set in main)


def peer_of(rank: int, world: int) -> int:
    """cfg1 at N GPUs: the object produced on GPU r is consumed on GPU r+1
    (a ring of disjoint producer->consumer pairs: every GPU's NVLink egress
    and ingress carry one stream, no link is shared)."""
    return (rank + 1) % world


def exchange(obj, world: int, group=None):
    """all_gather of a picklable object (export descriptors) over the
    process group; world == 1 returns [obj]."""
    if world == 1:
        return [obj]
    import torch.distributed as dist
    out = [None] * world
    dist.all_gather_object(out, obj, group=group)
    return out


def max_over_ranks(x: float, world: int, device=None) -> float:
    """MAX of a host float over the ranks, on the CPU (gloo) group: no kernel
    is left resident on the GPUs (device is accepted for old callers)."""
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=CPU_GROUP[0])
    return float(t.item())


# ------------------------------------------------------------------ reference / oracle arm

# ------------------------------------------------------------------ reference / oracle arm
class OracleRequest:
    """The oracle as it stands on the bench's cfg1 request: a cFn put of the
    38.5 MB tensor with hint GPU0 (O1: plan + np.copyto into the simulated
    GPU0 buffer), then the gFn's get_into of it (O4: np.copyto into the
    binding; consumers = 1, so the object is consumed and freed).  State is
    built once; only the calls are timed."""

    def __init__(self):
        import numpy as np

        from oracle.model import Oracle
        from synth.calib import b200_hgx
        from synth.payload import payload

        self.np = np
        self.orc = Oracle(b200_hgx(1))
        self.src = payload(1000, N_BYTES)
        self.dst = np.empty(N_BYTES, np.uint8)
        self.c = {"wf": 1, "fid": 1, "dev": -1}
        self.g = {"wf": 1, "fid": 2, "dev": 0}

    def run(self, requests: int):
        for _ in range(requests):
            st, out = self.orc.put(self.c, self.src, N_BYTES, 0, 1)
            assert st == 0
            st, _ = self.orc.get_into(self.g, out["oid"], self.dst, N_BYTES)
            assert st == 0
        return requests

    def check(self):
        assert self.np.array_equal(self.dst[:4096], self.src[:4096]) and not self.orc.objects


def oracle_rate(budget_s: float, requests: int = 2):
    """(req/s, requests, seconds) of the oracle over >= budget_s (1 thread)."""
    leg = OracleRequest()
    done, t0 = 0, time.perf_counter()
    while True:
        done += leg.run(requests)
        dt = time.perf_counter() - t0
        if dt >= budget_s:
            break
    leg.check()
    return done / dt, done, dt


def oracle_striped_put_rate(budget_s: float):
    """SURVEY §8(d) striped variant: the cFn put's O6 plan on the 8-GPU HGX
    calibration (R(0) = one GPU per PCIe uplink group) executed with one
    thread per route (T = |R(0)|, capped at the cores), each np.copyto-ing
    its chunks.  Returns (puts/s, threads)."""
    from concurrent.futures import ThreadPoolExecutor

    import numpy as np

    from oracle.splitter import CHUNK, plan_h2d
    from synth.calib import b200_hgx
    from synth.payload import payload
    src = payload(1000, N_BYTES)
    dst = np.empty(N_BYTES, np.uint8)
    by = {}
    for c in plan_h2d(b200_hgx(8), 0, N_BYTES, True, CHUNK):
        by.setdefault(c["route_gpu"], []).append((c["offset"], c["offset"] + c["bytes"]))
    T = max(1, min(len(by), len(os.sched_getaffinity(0))))

    def work(spans):
        for a, b in spans:
            np.copyto(dst[a:b], src[a:b])
    done = 0
    with ThreadPoolExecutor(T) as ex:
        t0 = time.perf_counter()
        while True:
            list(ex.map(work, by.values()))
            done += 1
            dt = time.perf_counter() - t0
            if dt >= budget_s:
                break
    assert np.array_equal(dst, src)
    return done / dt, T


def cpu_baseline_obj(budget_s: float):
    cores, model = host_info()
    v, done, dt = oracle_rate(budget_s)
    sv, T = oracle_striped_put_rate(max(1.0, budget_s / 4))
    return {"value": v, "unit": "req/s", "cores": 1, "kind": "oracle", "host_cores": cores, "cpu_model": model,
            "sample": f"{done} oracle cfg1 requests (put hint GPU0 + get_into, {N_BYTES} B, numpy memcpy "
                      f"on simulated buffers) in {dt:.1f} s, 1 thread",
            "striped_put": {"value": sv, "unit": "puts/s", "threads": T,
                            "what": "the put's O6 plan on the 8-GPU HGX calibration, one thread per route"}}


def run_reference(args, rank):
    """--impl reference: the oracle as it stands on the bench's cfg1 request,
    on this box's host cores (rank 0 only; other ranks exit without work)."""
    if rank != 0:
        return
    reqs = max(1, min(args.requests, 4))          # bounded sample per step
    leg = OracleRequest()
    for _ in range(args.warmup):
        leg.run(reqs)
    t0 = time.perf_counter()
    done = 0
    for _ in range(args.steps):
        done += leg.run(reqs)
    dt = time.perf_counter() - t0
    leg.check()
    v = done / dt
    cores, model = host_info()
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "req/s",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": dt * 1e3 / args.steps, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u8", "data": "synthetic (SplitMix64 payload)",
            "config": {"workload": WORKLOAD, "requests_per_step": reqs, "bytes": N_BYTES,
                       "parallelism": "oracle, 1 thread"},
            "cpu_baseline": {"kind": "oracle", "value": v, "unit": "req/s", "cores": 1, "host_cores": cores,
                             "cpu_model": model,
                             "sample": f"{args.steps} steps x {reqs} oracle cfg1 requests of {N_BYTES} B"},
            "e2e": {"value": v, "unit": "req/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)




# ------------------------------------------------------------------ cfg3 size sweep (one GPU)
SWEEP_SIZES = [4096 * 4 ** i for i in range(10)] + [2 * MiB - 1, 2 * MiB + 1, N_BYTES]


def _samples(n):
    return 200 if n <= 64 * MiB else (50 if n <= 256 * MiB else 30)


def _stats(xs, n, rw=1):
    p50, p99 = pct(xs, 50), pct(xs, 99)
    return {"p50_us": round(p50, 2), "p99_us": round(p99, 2), "GBps": round(rw * n / p50 / 1e3, 2)}


def measure_sweep(G, dev, hbm_peak, h2d_peak, sizes=SWEEP_SIZES, oracle=True):
    """cfg3 (iii) and (iv) at one GPU, per size, each beside a bare
    cudaMemcpyAsync on the same buffers called through the same binding
    (grouter_test_memcpy), byte-verified:
      get_into  gFn get_into of a GPU0-resident object: single calls on an idle
                GPU (CUDA events around the call on the consumer stream, host
                path included) and back to back (GB/s read + write, fraction
                of the HBM copy peak); baseline cudaMemcpyAsync D2D
      put_h2d   cFn put(hint GPU0) from pinned host memory, blocking, host
                timed; baseline pinned H2D + wait
      get_d2h   cFn get of a GPU0 object into a host lease (+ release),
                blocking, host timed; baseline D2H + wait
      zero_copy gFn get + release of a co-located object, host timed
    Samples: 200 (<= 64 MiB), 50 (256 MiB), 30 (1 GiB); nearest-rank p50/p99."""
    import torch
    from synth.calib import b200_hgx
    calib = b200_hgx(1)
    calib["device_map"] = [dev]
    maxn = max(sizes)
    ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=maxn + (256 << 20), pool_cap=[G.UNLIMITED],
                                    pool_floor_bytes=64 << 20))
    out = []
    try:
        s = torch.cuda.Stream(device=dev)
        host = torch.empty(maxn, dtype=torch.uint8, pin_memory=True)
        tmp = torch.empty(maxn, dtype=torch.uint8, device=f"cuda:{dev}")
        G.check(G.test_fill(tmp.data_ptr(), maxn, 31337, 0, 0))
        host.copy_(tmp)
        dsts = [torch.empty(maxn, dtype=torch.uint8, device=f"cuda:{dev}") for _ in range(2)]
        del tmp
        torch.cuda.synchronize(dev)
        cfn, gfn, gfn2 = G.fn(7, 1, G.HOST), G.fn(7, 2, 0), G.fn(7, 3, 0)
        hp, ss = host.data_ptr(), s.cuda_stream

        def dev_single(call, reps):
            xs = []
            for _ in range(reps):
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(s)
                call()
                b.record(s)
                b.synchronize()
                xs.append(a.elapsed_time(b) * 1e3)
            return xs

        def dev_b2b(call, reps):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            for _ in range(reps):
                call()
            b.record(s)
            b.synchronize()
            return a.elapsed_time(b) * 1e3 / reps

        def host_single(call, reps):
            xs = []
            for _ in range(reps):
                t = time.perf_counter()
                call()
                xs.append((time.perf_counter() - t) * 1e6)
            return xs

        import gc
        gc_was = gc.isenabled()
        gc.disable()          # no collector pauses inside single-call samples
        for n in [sizes[0]] + list(sizes):   # the first size twice: its first pass is a warm-up
            reps = _samples(n)
            row = {"bytes": n}
            st, oid = ctx.put(cfn, hp, n, 0, 0)
            G.check(st, "put")
            # back to back: a working set above the 126 MB L2 where memory allows
            # (m source objects, destinations rotating over the two 1 GiB buffers)
            m = max(1, min(32, (256 * MiB) // max(n, 1)))
            srcs = [oid]
            for _ in range(m - 1):
                st, o2 = ctx.put(cfn, hp, n, 0, 0)
                G.check(st, "put")
                srcs.append(o2)
            slots = max(1, min(64, maxn // max(-(-n // 256) * 256, 1)))
            G.check(ctx.sync(), "sync")
            k = [0]

            def dst_at(j):
                return dsts[j & 1].data_ptr() + ((j >> 1) % slots) * (-(-n // 256) * 256)

            def gi():
                st, _ = ctx.get_into(gfn, srcs[k[0] % m], dst_at(k[0]), n, ss)
                k[0] += 1
                if st:
                    G.check(st, "get_into")

            def mc():
                G.check(G.test_memcpy(dst_at(k[0]), dst_at(k[0] + 1), n, ss, False))
                k[0] += 1
            for _ in range(5):
                gi()
            s.synchronize()
            st, bad, _ = G.test_verify(dst_at(4), n, 31337, 0, 0)
            assert st == 0 and bad == 0, f"sweep get_into {n}: {bad} bytes differ"
            for _ in range(3):
                mc()
            # single calls, library and baseline interleaved sample by sample (drift
            # and host noise hit both alike)
            lib1, base1 = [], []
            for _ in range(reps):
                lib1 += dev_single(gi, 1)
                base1 += dev_single(mc, 1)
            b2b = dev_b2b(gi, max(10, min(reps, 200)))
            bb2b = dev_b2b(mc, max(10, min(reps, 200)))
            row["get_into"] = dict(_stats(lib1, n, 2), b2b_us=round(b2b, 2), b2b_GBps=round(2 * n / b2b / 1e3, 1),
                                   b2b_frac_hbm=round(2 * n / b2b / 1e3 / hbm_peak, 3),
                                   memcpy=dict(_stats(base1, n, 2), b2b_us=round(bb2b, 2)))
            # cFn put (H2D) vs bare pinned H2D; the free of each put object is
            # outside the timed call
            def put_timed(reps):
                xs = []
                for _ in range(reps):
                    m0 = ctx.stats().mapped[0] if SWEEP_DEBUG else 0
                    t = time.perf_counter()
                    st, o2 = ctx.put(cfn, hp, n, 0, 0)
                    xs.append((time.perf_counter() - t) * 1e6)
                    if SWEEP_DEBUG:
                        print(f"[sweep] put {n} {xs[-1]:.0f} us mapped {m0 >> 20} -> "
                              f"{ctx.stats().mapped[0] >> 20} MiB", file=sys.stderr, flush=True)
                    if st:
                        G.check(st, "put")
                    ctx.free(cfn, o2)
                return xs

            def h2d():
                G.check(G.test_memcpy(dsts[0].data_ptr(), hp, n, 0, True))
            put_timed(3)
            for _ in range(3):
                h2d()
            lp, bp = [], []
            for _ in range(reps):
                lp += put_timed(1)
                bp += host_single(h2d, 1)
            row["put_h2d"] = dict(_stats(lp, n), frac_link=round(n / pct(lp, 50) / 1e3 / h2d_peak, 3),
                                  memcpy=_stats(bp, n))
            # cFn get (D2H into a host lease) vs bare D2H; the lease's release
            # is outside the timed call
            def get_timed(reps):
                xs = []
                for _ in range(reps):
                    t = time.perf_counter()
                    st, ptr, nn = ctx.get(cfn, oid, 0)
                    xs.append((time.perf_counter() - t) * 1e6)
                    if st:
                        G.check(st, "get")
                    ctx.release(cfn, oid, ptr, 0)
                return xs

            def d2h():
                G.check(G.test_memcpy(hp, dsts[0].data_ptr(), n, 0, True))
            get_timed(3)
            for _ in range(3):
                d2h()
            lg, bg = [], []
            for _ in range(reps):
                lg += get_timed(1)
                bg += host_single(d2h, 1)
            row["get_d2h"] = dict(_stats(lg, n), memcpy=_stats(bg, n))

            def zc_timed(reps):   # gFn zero-copy get; the release is outside the timed call
                xs = []
                for _ in range(reps):
                    t = time.perf_counter()
                    st, ptr, nn = ctx.get(gfn2, oid, ss)
                    xs.append((time.perf_counter() - t) * 1e6)
                    ctx.release(gfn2, oid, ptr, ss)
                return xs
            zc_timed(3)
            z = zc_timed(reps)
            row["zero_copy_get_us"] = {"p50": round(pct(z, 50), 2), "p99": round(pct(z, 99), 2)}
            for o2 in srcs:
                G.check(ctx.free(cfn, o2), "free")
            row["b2b_working_set"] = {"sources": m, "dst_slots": 2 * slots}
            if oracle:   # the oracle's get_into of the same size (numpy memcpy), 1 thread
                import numpy as np
                from oracle.model import Oracle
                orc = Oracle(b200_hgx(1))
                buf = np.zeros(n, np.uint8)
                st, o = orc.put({"wf": 1, "fid": 1, "dev": 0}, buf, n, -2, 0)
                d = np.empty(n, np.uint8)
                xs, t_end = [], time.perf_counter() + 0.25
                while len(xs) < 3 or (time.perf_counter() < t_end and len(xs) < 100):
                    t = time.perf_counter()
                    orc.get_into({"wf": 1, "fid": 2, "dev": 0}, o["oid"], d, n)
                    xs.append((time.perf_counter() - t) * 1e6)
                row["oracle_get_into"] = {"p50_us": round(pct(xs, 50), 2), "samples": len(xs)}
            row["samples"] = reps
            out.append(row)
        out = out[1:]                         # drop the warm-up pass
        if gc_was:
            gc.enable()
    finally:
        ctx.close()
    return out


def measure_multipath(world, G, nbytes=1 << 30, reps=3):
    """Probe every GPU (solo/pairwise H2D -> uplink groups, P2P, NVLink), then
    time a blocking cFn put of `nbytes` from pinned host into GPU0 striped over
    R(0) vs the direct link only (GROUTER_NO_MULTIPATH)."""
    import torch
    devs = [0] * world if os.environ.get("GR_BENCH_SAME_GPU") == "1" else list(range(world))
    calib = G.probe(devs, 256 << 20)
    host = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    out = {"probe_h2d_GBps": [round(b / 1e9, 2) for b in calib["h2d_Bps"]],
           "probe_nvl_GBps": round(calib["nvl_Bps"] / 1e9, 1)}
    # TA off (GROUTER_NO_TOPOLOGY, Fig. 16): GPUs behind one PCIe switch both stage (R48)
    for name, flags in (("direct", G.NO_MULTIPATH), ("striped", 0), ("striped_no_topology", G.NO_TOPOLOGY),
                        ("striped_ce_relay", G.CE_RELAY)):
        ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=256 << 20, flags=flags,
                                        pool_cap=[G.UNLIMITED] * world, pool_floor_bytes=64 << 20))
        st, routes = ctx.route_set(0)
        f = G.fn(9, 1, G.HOST)
        ts = []
        for r in range(reps + 1):
            t0 = time.perf_counter()
            st, oid = ctx.put(f, host.data_ptr(), nbytes, 0, 0)
            G.check(st, "put")
            dt = time.perf_counter() - t0
            ctx.free(f, oid)
            if r:
                ts.append(dt)
        out[name] = {"routes": routes, "GBps": round(nbytes / min(ts) / 1e9, 2)}
        # cfg3 (iii) vs size: blocking cFn put GB/s (best of 3) at 4 MiB .. 256 MiB
        sweep = {}
        for sz in (4 << 20, 38_535_168, 64 << 20, 256 << 20):
            best = None
            for r in range(4):
                t0 = time.perf_counter()
                st, oid = ctx.put(f, host.data_ptr(), sz, 0, 0)
                G.check(st, "put")
                dt = time.perf_counter() - t0
                ctx.free(f, oid)
                if r:
                    best = dt if best is None else min(best, dt)
            sweep[sz] = round(sz / best / 1e9, 2)
        out[name]["GBps_by_size"] = sweep
        ctx.close()
    out["speedup"] = round(out["striped"]["GBps"] / out["direct"]["GBps"], 2)
    out["ce_relay_speedup"] = round(out["striped_ce_relay"]["GBps"] / out["direct"]["GBps"], 2)
    out["topology_gain"] = round(out["striped"]["GBps"] / out["striped_no_topology"]["GBps"], 2)
    # gFn-host (L178, Fig. 5a): a GPU0 object read into host memory by a cFn,
    # direct D2H vs striped over R(0) (GROUTER_D2H_MULTIPATH)
    src = torch.empty(nbytes, dtype=torch.uint8, device="cuda:0")
    for name, flags in (("d2h_direct", 0), ("d2h_striped", G.D2H_MULTIPATH)):
        ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=256 << 20, flags=flags,
                                        pool_cap=[G.UNLIMITED] * world, pool_floor_bytes=64 << 20))
        g0, c0 = G.fn(9, 1, 0), G.fn(9, 2, G.HOST)
        st, oid = ctx.put(g0, src.data_ptr(), nbytes, G.NOHINT, 0, 0)
        G.check(st, "put")
        ctx.sync()
        ts = []
        for r in range(reps + 1):
            t0 = time.perf_counter()
            st, nn = ctx.get_into(c0, oid, host.data_ptr(), nbytes, 0)
            G.check(st, "get_into")
            dt = time.perf_counter() - t0
            if r:
                ts.append(dt)
        out[name] = {"GBps": round(nbytes / min(ts) / 1e9, 2)}
        ctx.free(g0, oid)
        ctx.close()
    out["d2h_speedup"] = round(out["d2h_striped"]["GBps"] / out["d2h_direct"]["GBps"], 2)
    out.update(measure_d2d_push(world, G, calib, devs))
    if len(set(devs)) < len(devs):
        out["note"] = ("GR_BENCH_SAME_GPU: every logical GPU is device 0, so 'NVLink' copies are "
                       "same-device HBM copies and the NVLink fractions do not apply")
    return out


def measure_d2d_push(world, G, calib, devs, n=N_BYTES, objs=8, reps=10):
    """cfg1 leg B at N >= 2 inside ONE GROUTER context spanning the node (the
    paper's deployment: one service per node): a gFn on GPU1 get_into's
    objects resident on GPU0 -- GPU0's copy server pushes them over NVLink
    with the SM copy kernel (K2', L167 (1)); the consumer stream waits on the
    completion words.  Then every GPU i pulls from its ring successor at once
    (cfg3 (ii), disjoint pairs): aggregate GB/s.  Device-timed with CUDA
    events on the consumer streams."""
    import torch
    ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=256 << 20, pool_cap=[G.UNLIMITED] * world,
                                    pool_floor_bytes=64 << 20))
    out = {}
    try:
        src = torch.empty(n, dtype=torch.uint8, device=f"cuda:{devs[0]}")
        resident = {}   # logical GPU -> oids
        for g in range(world):
            s0 = torch.empty(n, dtype=torch.uint8, device=f"cuda:{devs[g]}")
            for i in range(objs):
                G.check(G.test_fill(s0.data_ptr(), n, 7000 + i, 0, 0))
                torch.cuda.synchronize(devs[g])
                st, oid = ctx.put(G.fn(9, 1, g), s0.data_ptr(), n, G.NOHINT, 0, 0)
                G.check(st, "put")
                resident.setdefault(g, []).append(oid)
        del src
        ctx.sync()

        def run(pairs):
            """pairs: [(consumer logical GPU, producer logical GPU)]; returns GB/s aggregate, us/get."""
            streams = {c: torch.cuda.Stream(device=f"cuda:{devs[c]}") for c, _ in pairs}
            dst = {c: [torch.empty(n, dtype=torch.uint8, device=f"cuda:{devs[c]}") for _ in range(2)]
                   for c, _ in pairs}

            def one_pass():
                for i in range(objs):
                    for c, p in pairs:
                        st, _ = ctx.get_into(G.fn(9, 2, c), resident[p][i], dst[c][i % 2].data_ptr(), n,
                                             streams[c].cuda_stream)
                        G.check(st, "get_into")
            one_pass()
            for c, p in pairs:
                streams[c].synchronize()
                for b in range(2):   # the last object that wrote binding b
                    last = max(i for i in range(objs) if i % 2 == b)
                    st, bad, _ = G.test_verify(dst[c][b].data_ptr(), n, 7000 + last, 0, 0)
                    assert st == 0 and bad == 0, f"d2d push {p}->{c}: {bad} bytes differ"
            ev = {c: (torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
                  for c, _ in pairs}
            for c, _ in pairs:
                ev[c][0].record(streams[c])
            for _ in range(reps):
                one_pass()
            for c, _ in pairs:
                ev[c][1].record(streams[c])
            for c, _ in pairs:
                ev[c][1].synchronize()
            ms = max(ev[c][0].elapsed_time(ev[c][1]) for c, _ in pairs)
            gets = reps * objs
            return gets * len(pairs) * n / (ms / 1e3) / 1e9, ms * 1e3 / gets

        gbps, us = run([(1, 0)])
        out["d2d_push"] = {"what": "GPU1 gFn get_into of GPU0-resident 38.5 MB objects (GPU0 SM push over "
                                   "NVLink, one context)", "GBps": round(gbps, 1), "us_per_get": round(us, 2),
                           "frac": round(gbps / NVL_PEAK, 3),
                           "frac_of_770_measured_peer_copy": round(gbps / 770.0, 3)}
        # baseline on the same devices and sizes: cudaMemcpyPeerAsync (copy engine)
        a0 = torch.empty(n, dtype=torch.uint8, device=f"cuda:{devs[0]}")
        b1 = [torch.empty(n, dtype=torch.uint8, device=f"cuda:{devs[1]}") for _ in range(2)]
        sp = torch.cuda.Stream(device=f"cuda:{devs[1]}")
        with torch.cuda.stream(sp):
            for i in range(3):
                b1[i % 2].copy_(a0, non_blocking=True)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(sp)
            for i in range(reps * objs):
                b1[i % 2].copy_(a0, non_blocking=True)
            e1.record(sp)
        e1.synchronize()
        us_b = e0.elapsed_time(e1) * 1e3 / (reps * objs)
        out["d2d_memcpy_peer_baseline"] = {"GBps": round(n / us_b / 1e3, 1), "us_per_copy": round(us_b, 2)}
        ring = [(c, (c + 1) % world) for c in range(world)]
        gbps, us = run(ring)
        out["d2d_ring"] = {"what": f"all {world} GPUs get_into their ring successor's objects at once",
                           "aggregate_GBps": round(gbps, 1), "per_gpu_GBps": round(gbps / world, 1),
                           "us_per_get": round(us, 2)}
        if world >= 4:   # cfg3 (ii): the permutation i -> (i + N/2) mod N, all pairs at once
            gbps, us = run([(c, (c + world // 2) % world) for c in range(world)])
            out["d2d_perm"] = {"what": f"all {world} GPUs get_into the objects of GPU (i + {world // 2}) mod {world} "
                                       "at once (cfg3 (ii))",
                               "aggregate_GBps": round(gbps, 1), "per_gpu_GBps": round(gbps / world, 1),
                               "frac_per_gpu": round(gbps / world / NVL_PEAK, 3), "us_per_get": round(us, 2)}
    except Exception as e:  # reported, never fatal for the line
        out["d2d_error"] = f"{type(e).__name__}: {e}"[:300]
    finally:
        ctx.close()
    out["d2d_sweep"] = measure_d2d_sweep(world, G, calib, devs)
    # the same gets pulled by GPU1's SMs at every size (GROUTER_PULL_ALL; default: pulls <= 4 MiB,
    # R56): the data for the pull/push threshold on NVLink 5
    out["d2d_sweep_pull"] = measure_d2d_sweep(world, G, calib, devs, sizes=(16 << 20, 38_535_168, 256 << 20, 1 << 30),
                                              flags=G.PULL_ALL)
    return out


def measure_d2d_sweep(world, G, calib, devs, sizes=(4096, 65536, 1 << 20, 16 << 20, 38_535_168, 64 << 20,
                                                     256 << 20, 1 << 30), flags=0):
    """cfg3 (i) at N >= 2 (the metric's "latency & GB/s vs size"): a gFn on
    GPU1 get_into's an object resident on GPU0 (GPU0's SM copy pushes it over
    NVLink), per size: p50/p99 of single calls on an idle pair (CUDA events on
    the consumer stream, host path included) and back-to-back GB/s; beside it
    cudaMemcpyPeerAsync on the same buffers.  Byte-verified per size."""
    import torch
    ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=64 << 20, pool_cap=[G.UNLIMITED] * world,
                                    pool_floor_bytes=64 << 20, flags=flags))
    res = []
    try:
        s1 = torch.cuda.Stream(device=f"cuda:{devs[1]}")
        for n in sizes:
            reps = 40 if n <= (64 << 20) else 10
            src = torch.empty(n, dtype=torch.uint8, device=f"cuda:{devs[0]}")
            G.check(G.test_fill(src.data_ptr(), n, 4242, 0, 0))
            torch.cuda.synchronize(devs[0])
            oids = []
            for _ in range(2):
                st, oid = ctx.put(G.fn(9, 1, 0), src.data_ptr(), n, G.NOHINT, 0, 0)
                G.check(st, "put")
                oids.append(oid)
            ctx.sync()
            dst = [torch.empty(n, dtype=torch.uint8, device=f"cuda:{devs[1]}") for _ in range(2)]
            f1 = G.fn(9, 2, 1)
            for i in range(3):
                G.check(ctx.get_into(f1, oids[i % 2], dst[i % 2].data_ptr(), n, s1.cuda_stream)[0], "get_into")
            s1.synchronize()
            st, bad, _ = G.test_verify(dst[0].data_ptr(), n, 4242, 0, 0)
            assert st == 0 and bad == 0, f"d2d sweep {n}: {bad} bytes differ"
            lat = []
            for i in range(reps):
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(s1)
                ctx.get_into(f1, oids[i % 2], dst[i % 2].data_ptr(), n, s1.cuda_stream)
                b.record(s1)
                b.synchronize()
                lat.append(a.elapsed_time(b) * 1e3)
            lat.sort()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s1)
            for i in range(reps):
                ctx.get_into(f1, oids[i % 2], dst[i % 2].data_ptr(), n, s1.cuda_stream)
            b.record(s1)
            b.synchronize()
            tput = n * reps / (a.elapsed_time(b) / 1e3) / 1e9
            with torch.cuda.stream(s1):                    # baseline: cudaMemcpyPeerAsync (copy engine)
                a.record(s1)
                for i in range(reps):
                    dst[i % 2].copy_(src, non_blocking=True)
                b.record(s1)
            b.synchronize()
            base = n * reps / (a.elapsed_time(b) / 1e3) / 1e9
            res.append({"bytes": n, "p50_us": round(lat[len(lat) // 2], 2),
                        "p99_us": round(lat[min(len(lat) - 1, -(-len(lat) * 99 // 100) - 1)], 2),
                        "GBps": round(tput, 1), "frac": round(tput / NVL_PEAK, 3),
                        "frac_of_770_measured_peer_copy": round(tput / 770.0, 3),
                        "memcpy_peer_GBps": round(base, 1)})
            for oid in oids:
                ctx.free(G.fn(9, 1, 0), oid)
            del src, dst
            torch.cuda.empty_cache()
    except Exception as e:  # reported, never fatal for the line
        res.append({"error": f"{type(e).__name__}: {e}"[:300]})
    finally:
        ctx.close()
    return res


def nccl_ring_baseline(world, rank, dev, n, per_step, steps):
    """The library-free baseline for the same exchange: every rank receives
    n-byte tensors from rank+1 (and sends to rank-1) with NCCL send/recv,
    per_step per step; device-timed on the NCCL stream's caller stream, max
    over ranks.  GB/s per GPU received."""
    import torch
    import torch.distributed as dist
    src = torch.empty(n, dtype=torch.uint8, device=f"cuda:{dev}")
    dst = torch.empty(n, dtype=torch.uint8, device=f"cuda:{dev}")
    to, frm = (rank - 1) % world, (rank + 1) % world

    def step():
        for _ in range(per_step):
            ops = [dist.P2POp(dist.isend, src, to), dist.P2POp(dist.irecv, dst, frm)]
            for w in dist.batch_isend_irecv(ops):
                w.wait()
    for _ in range(3):
        step()
    torch.cuda.synchronize(dev)
    dist.barrier()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(steps):
        step()
    b.record()
    b.synchronize()
    ms = max_over_ranks(a.elapsed_time(b), world, f"cuda:{dev}")
    return {"what": "NCCL send/recv ring (torch.distributed batch_isend_irecv), same bytes and pairing",
            "gbps_per_gpu": round(steps * per_step * n / (ms / 1e3) / 1e9, 1),
            "us_per_transfer": round(ms * 1e3 / (steps * per_step), 2)}


# ------------------------------------------------------------------ GPU arm

# ------------------------------------------------------------------ cfg2 (BASELINE configs[1]) at one GPU
def measure_cfg2(G, dev, seconds=2.0, outstanding=4, oracle=True):
    """Traffic-monitoring workflow (BASELINE configs[1]),
    data plane only, closed loop with `outstanding` clients: a decode cFn puts a
    39,321,600 B frame (8x3x640x640 fp32) with hint GPU0 (PCIe H2D); the YOLO
    gFn gets it (zero copy, co-located), allocs + seals person and vehicle crop
    batches (K x 602,112 B, K ~ Poisson(4) clipped to [0, 32]); the two
    recognition gFns get them (zero copy at one GPU) and everyone releases.
    Wall-clock req/s and per-request latency."""
    import math
    import random
    import torch
    from synth.calib import b200_hgx
    FRAME, CROP = 39_321_600, 602_112
    calib = b200_hgx(1)
    calib["device_map"] = [dev]
    ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=256 << 20, pool_cap=[G.UNLIMITED]))
    frames = [torch.empty(FRAME, dtype=torch.uint8, pin_memory=True) for _ in range(outstanding)]
    streams = [torch.cuda.Stream(device=dev) for _ in range(outstanding)]
    lat, done, stop = [], [0] * outstanding, threading.Event()
    go = threading.Barrier(outstanding + 1)

    def poisson(rng, lam=4.0):
        L, k, p = math.exp(-lam), 0, 1.0
        while True:
            p *= rng.random()
            if p <= L:
                return min(k, 32)
            k += 1

    def worker(t):
        torch.cuda.set_device(dev)
        rng = random.Random(2000 + t)
        s = streams[t].cuda_stream
        go.wait()
        i = 0
        while not stop.is_set():
            wf = 10 + t * 100000 + i
            dec, yolo, rp, rv = G.fn(wf, 1, G.HOST), G.fn(wf, 2, 0), G.fn(wf, 3, 0), G.fn(wf, 4, 0)
            t0 = time.perf_counter()
            st, o = ctx.put(dec, frames[t].data_ptr(), FRAME, 0, 1)
            G.check(st, "put")
            st, fp, _ = ctx.get(yolo, o, s)
            G.check(st, "get")
            crops = []
            for k in (poisson(rng), poisson(rng)):
                st, buf, a = ctx.alloc(yolo, k * CROP, G.NOHINT, 1)
                G.check(st, "alloc")
                G.check(ctx.seal(yolo, a, s), "seal")
                crops.append(a)
            leases = []
            for f, a in ((rp, crops[0]), (rv, crops[1])):
                st, ptr, _ = ctx.get(f, a, s)
                G.check(st, "get crops")
                leases.append((f, a, ptr))
            G.check(ctx.release(yolo, o, fp, s), "release")
            for f, a, ptr in leases:
                if ptr:
                    G.check(ctx.release(f, a, ptr, s), "release crops")
            streams[t].synchronize()
            lat.append((time.perf_counter() - t0) * 1e6)
            done[t] += 1
            i += 1
    ths = [threading.Thread(target=worker, args=(t,)) for t in range(outstanding)]
    for th in ths:
        th.start()
    go.wait()
    t0 = time.perf_counter()
    time.sleep(seconds)
    stop.set()
    for th in ths:
        th.join()
    dt = time.perf_counter() - t0
    ctx.sync()
    used = ctx.stats().used[0]
    ctx.close()
    n = sum(done)
    out = {"what": "cfg2 traffic monitoring (BASELINE configs[1]) at one GPU, data plane: frame put + zero-copy "
                   "YOLO get + crop alloc/seal + two zero-copy recognition gets, 4 clients, wall clock",
           "req_per_s": round(n / dt, 1), "frame_GBps": round(n * FRAME / dt / 1e9, 2),
           "latency_us": {"p50": round(pct(lat, 50), 1), "p99": round(pct(lat, 99), 1)}, "requests": n,
           "pool_used_after": used}
    if oracle:   # the oracle on the same request structure (synth.traces.cfg2), one thread
        from oracle import runner as orun
        from synth import traces as TT
        ops = TT.cfg2(1, requests=8)
        t1 = time.perf_counter()
        orun.run(ops, b200_hgx(1))
        out["oracle_req_per_s"] = round(8 / (time.perf_counter() - t1), 1)
    return out


# ------------------------------------------------------------------ GPU arm
SWEEP_DEBUG = os.environ.get("GR_SWEEP_DEBUG") == "1"


def h2d_link_peak(G, dev, nbytes=256 << 20, reps=4):
    """Pinned single-link H2D GB/s on this box (bare cudaMemcpyAsync back to
    back, CUDA events): the PCIe roofline of the workflow."""
    import torch
    host = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    d = torch.empty(nbytes, dtype=torch.uint8, device=f"cuda:{dev}")
    s = torch.cuda.Stream(device=dev)
    G.check(G.test_memcpy(d.data_ptr(), host.data_ptr(), nbytes, s.cuda_stream, True))
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    for _ in range(reps):
        G.check(G.test_memcpy(d.data_ptr(), host.data_ptr(), nbytes, s.cuda_stream, False))
    b.record(s)
    b.synchronize()
    return nbytes * reps / (a.elapsed_time(b) / 1e3) / 1e9


def run_gpu(args, rank, world, local_rank):
    import torch
    import torch.distributed as dist

    from paper_conf_eurosys_wulywdyfwwj26_b200 import _build
    from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G
    from synth.calib import b200_hgx

    _build.build()
    G.load()
    same_gpu = os.environ.get("GR_BENCH_SAME_GPU") == "1"
    dev = local_rank
    torch.cuda.set_device(dev)
    n, R = N_BYTES, args.requests
    # one context per rank: the producer GPU (logical 0) and, at N > 1, the
    # consumer GPU r+1 (logical 1); each rank's puts use its own PCIe link
    cons_dev = dev if world == 1 else (dev if same_gpu else peer_of(dev, world))
    calib = b200_hgx(1 if world == 1 else 2)
    calib["device_map"] = [dev] if world == 1 else [dev, cons_dev]
    flags = G.PROFILE | (G.COPY_TMA if args.tma else 0) | (G.NO_MULTIPATH if world > 1 else 0)
    if same_gpu and os.environ.get("GR_BENCH_FORCE_REMOTE") == "1":
        flags |= G.FORCE_REMOTE   # plumbing on one GPU: the dispatch and kernel branch of a physical pair
    ctx = G.Ctx(G.config_from_calib(calib, host_store_bytes=256 << 20, pool_cap=[G.UNLIMITED] * calib["n_gpus"],
                                    flags=flags, copy_ctas_per_sm=args.ctas))
    cons_logical = 0 if world == 1 else 1
    cfn = G.fn(1, 1, G.HOST)
    gfn = G.fn(1, 2, cons_logical)

    def barrier():
        if world > 1:
            dist.barrier(group=CPU_GROUP[0])
        torch.cuda.synchronize(dev)
        if cons_dev != dev:
            torch.cuda.synchronize(cons_dev)

    # pinned host sources (the cFn's outputs) with the SplitMix payload
    host_src = []
    tmp = torch.empty(n, dtype=torch.uint8, device=f"cuda:{dev}")
    for i in range(R):
        G.check(G.test_fill(tmp.data_ptr(), n, 1000 + i, 0, 0))
        h = torch.empty(n, dtype=torch.uint8, pin_memory=True)
        h.copy_(tmp)
        host_src.append(h)
    del tmp
    B = 8                                            # rotating input bindings: 308 MB > L2
    bindings = [torch.empty(n, dtype=torch.uint8, device=f"cuda:{cons_dev}") for _ in range(B)]
    torch.cuda.synchronize(dev)
    Q = max(1, min(args.q, B, R))
    qstreams = [torch.cuda.Stream(device=cons_dev) for _ in range(Q)]
    out8 = [torch.empty(8, dtype=torch.uint8, pin_memory=True) for _ in range(Q)]

    def request(i, qs, read_result):
        """One cfg1 request: leg A (cFn put, blocking) + leg B (gFn get_into,
        stream-ordered on the client's consumer stream)."""
        st, oid = ctx.put(cfn, host_src[i % R].data_ptr(), n, 0, 1)
        if st:
            G.check(st, "put")
        st, _ = ctx.get_into(gfn, oid, bindings[i % B].data_ptr(), n, qs.cuda_stream)
        if st:
            G.check(st, "get_into")
        if read_result:                              # e2e: the step's result back to the host
            with torch.cuda.stream(qs):
                out8[i % Q].copy_(bindings[i % B][:8], non_blocking=True)

    from concurrent.futures import ThreadPoolExecutor
    pool = ThreadPoolExecutor(max_workers=Q)

    def client(k, total, read_result):
        torch.cuda.set_device(dev)
        for i in range(k, total, Q):
            request(i, qstreams[k], read_result)

    def run_requests(total, read_result=False):
        for f in [pool.submit(client, k, total, read_result) for k in range(Q)]:
            f.result()

    def verify(total, what):
        """Every binding holds the payload of the last request that wrote it
        (full compare on the device against the generator)."""
        for qs in qstreams:
            qs.synchronize()
        for b in range(min(total, B)):
            last = max(i for i in range(total) if i % B == b)
            st, bad, _ = G.test_verify(bindings[b].data_ptr(), n, 1000 + last % R, 0, 0)
            assert st == 0 and bad == 0, f"{what}: binding {b}: {bad} bytes differ from the payload"

    # warm-up (W steps) + parity spot check
    run_requests(R * args.warmup)
    verify(R * args.warmup, "warm-up")
    total = R * args.steps
    st0 = ctx.stats()
    clk = ClockSampler(dev)
    clk.start()
    ts = torch.cuda.Stream(device=cons_dev)          # timing stream: every consumer stream joins it
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    barrier()                                        # last before the region: ranks start together
    e0.record(ts)
    for qs in qstreams:
        qs.wait_event(e0)
    h0 = time.perf_counter()
    run_requests(total)
    host_s = time.perf_counter() - h0
    for qs in qstreams:
        ev = torch.cuda.Event()
        ev.record(qs)
        ts.wait_event(ev)
    e1.record(ts)
    barrier()
    clocks = clk.stop()
    ms = e0.elapsed_time(e1)
    G.check(ctx.sync(), "sync")
    ms_max = max_over_ranks(ms, world)
    st1 = ctx.stats()
    verify(total, "timed region")
    value = total * world / (ms_max / 1e3)
    launches = st1.kernel_launches - st0.kernel_launches
    tl = st1.timed_launches - st0.timed_launches
    t_ns = st1.timed_ns - st0.timed_ns
    t_bytes = st1.timed_bytes - st0.timed_bytes
    tk = st1.timed_kernel_launches - st0.timed_kernel_launches      # %globaltimer stamps
    tk_ns = st1.timed_kernel_ns - st0.timed_kernel_ns

    # ---------------------------------------------------------- e2e (host-timed, + 8 B result read)
    e2e_steps = max(1, min(args.steps, args.e2e_steps))
    run_requests(R, True)
    barrier()
    h0 = time.perf_counter()
    run_requests(R * e2e_steps, True)
    for qs in qstreams:
        qs.synchronize()
    barrier()
    e2e_s = time.perf_counter() - h0
    e2e_val = R * e2e_steps * world / max_over_ranks(e2e_s, world)

    # ---------------------------------------------------------- single-request latency (R22)
    lat, lat_a = [], []
    s0 = qstreams[0]
    for i in range(args.lat_samples):
        t0 = time.perf_counter()
        st, oid = ctx.put(cfn, host_src[i % R].data_ptr(), n, 0, 1)
        G.check(st, "put")
        ta = time.perf_counter()
        G.check(ctx.get_into(gfn, oid, bindings[i % B].data_ptr(), n, s0.cuda_stream)[0], "get_into")
        ev = torch.cuda.Event()
        ev.record(s0)
        while not ev.query():
            pass
        t1 = time.perf_counter()
        lat.append((t1 - t0) * 1e6)
        lat_a.append((ta - t0) * 1e6)

    # ---------------------------------------------------------- leg B alone, back to back (kernel speed of light)
    # a context without GROUTER_PROFILE: per-launch events would sit between
    # the launches and defeat programmatic dependent launch
    ctx_b = G.Ctx(G.config_from_calib(calib, host_store_bytes=64 << 20, pool_cap=[G.UNLIMITED] * calib["n_gpus"],
                                      flags=flags & ~G.PROFILE, copy_ctas_per_sm=args.ctas))
    resident = []
    for i in range(R):
        st, oid = ctx_b.put(cfn, host_src[i].data_ptr(), n, 0, 0)
        G.check(st, "put")
        resident.append(oid)
    G.check(ctx_b.sync(), "sync")
    sb = qstreams[0]

    def legb():
        for i, oid in enumerate(resident):
            st, _ = ctx_b.get_into(gfn, oid, bindings[i % B].data_ptr(), n, sb.cuda_stream)
            if st:
                G.check(st, "get_into")
    for _ in range(3):
        legb()
    sb.synchronize()
    k0 = ctx_b.stats()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(sb)
    b2b_steps = max(20, args.b2b_steps)
    for _ in range(b2b_steps):
        legb()
    b.record(sb)
    b.synchronize()
    G.check(ctx_b.sync(), "sync")
    k1 = ctx_b.stats()
    verify(R, "back-to-back leg B")
    b2b_l = k1.kernel_launches - k0.kernel_launches
    b2b_us = a.elapsed_time(b) * 1e3 / max(b2b_l, 1)
    for oid in resident:
        ctx_b.free(cfn, oid)
    ctx_b.close()
    pool.shutdown()

    # ---------------------------------------------------------- rooflines
    peak_hbm, peak_src = _peaks()
    link_peak = h2d_link_peak(G, dev)
    rw = 2 if world == 1 or same_gpu else 1     # HBM read + write on one GPU; NVLink carries n once
    kpeak = peak_hbm if rw == 2 else NVL_PEAK
    k_us = t_ns / max(tl, 1) / 1e3
    k_ach = rw * t_bytes / t_ns if t_ns else None   # bytes / ns == GB/s
    b2b_ach = rw * n / b2b_us / 1e3
    try:
        live_peaks = _live_copy_peaks(dev) if world == 1 else None
    except Exception as e:   # context only; never fails the line
        live_peaks = {"error": str(e)[:200]}
    traffic = traffic_steady = None
    tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")   # per-launch DRAM bytes of the b2b region
    if os.path.exists(tp):
        try:
            tj = json.load(open(tp))
            traffic = tj.get("dram_bytes_per_launch")
            traffic_steady = tj.get("steady_dram_bytes_per_launch")
        except Exception:
            traffic = None

    # N > 1: host->GPU striping over the other GPUs' PCIe links (L120, L178), measured by
    # rank 0 alone on a context spanning every GPU of the node while the others wait
    multipath = None
    stuck = False
    if world > 1 and not args.no_multipath_probe:
        barrier()
        if rank == 0:
            box = {}

            def _mp():
                try:
                    box["r"] = measure_multipath(world, G)
                except Exception as e:  # report, never abort the scaling line
                    box["r"] = {"error": f"{type(e).__name__}: {e}"[:300]}
            th = threading.Thread(target=_mp, daemon=True)
            th.start()
            th.join(args.multipath_timeout)
            stuck = th.is_alive()
            multipath = box.get("r") or {"error": f"timed out after {args.multipath_timeout:.0f} s"}
        dist.barrier(group=CPU_GROUP[0])

    nccl = None
    if world > 1 and dist.get_backend() == "nccl":
        try:   # the library-free baseline of the same NVLink exchange (context only)
            nccl = nccl_ring_baseline(world, rank, dev, n, R, max(1, args.steps // 10))
        except Exception as e:
            nccl = {"error": f"{type(e).__name__}: {e}"[:200]}

    sweep = None
    if rank == 0 and world == 1 and not args.no_sweep:
        try:
            sweep = measure_sweep(G, dev, peak_hbm, link_peak, oracle=not args.no_cpu_baseline)
        except Exception as e:   # reported, never fatal for the line
            sweep = [{"error": f"{type(e).__name__}: {e}"[:300]}]

    cfg2 = None
    if rank == 0 and world == 1 and not args.no_sweep:
        try:
            cfg2 = measure_cfg2(G, dev, oracle=not args.no_cpu_baseline)
        except Exception as e:   # reported, never fatal for the line
            cfg2 = {"error": f"{type(e).__name__}: {e}"[:300]}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline_obj(args.cpu_seconds)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "req/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_max / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u8",
            "data": "synthetic (SplitMix64 payload; every delivered tensor verified on the device)",
            "config": {"workload": WORKLOAD if world == 1 else WORKLOAD_N, "requests_per_step": R,
                       "outstanding": Q, "bytes": N_BYTES,
                       "parallelism": "single GPU" if world == 1 else
                       f"ring of {world} producer->consumer GPU pairs, one process per GPU, no collective",
                       "l2": "inputs larger than L2: 20 x 38.5 MB pinned host sources, 8 rotating 38.5 MB "
                             "device bindings (308 MB)",
                       "copy_kernel": os.environ.get("GR_COPY", "tmas4" if args.tma else "wv8")},
            "gbps": value * N_BYTES / 1e9,
            "host_s": host_s,
            "latency_us": {"p50": pct(lat, 50), "p99": pct(lat, 99), "samples": len(lat),
                           "put_p50": pct(lat_a, 50),
                           "what": "one cfg1 request on an idle GPU: cFn put call -> gFn's data ready "
                                   "(event on the consumer stream observed by the host), R22"},
            "roofline": {"bound": "hbm" if rw == 2 else "nvlink", "achieved": b2b_ach, "peak": kpeak,
                         "unit": "GB/s", "frac": b2b_ach / kpeak, "traffic": traffic,
                         "kernel": "gr_copy (K2') leg B" + (" same-GPU" if rw == 2 else " NVLink push"),
                         "peak_source": peak_src if rw == 2 else "north star: 900 GB/s per direction",
                         "launches": b2b_l, "avg_launch_us": b2b_us, "alg_bytes_per_launch": rw * n,
                         "timing": "leg B's own timed region: the gFn get_into's of 20 HBM-resident 38.5 MB "
                                   "objects into 8 rotating bindings, 200 x 20 launches back to back, CUDA events "
                                   "on the consumer stream the kernels run on / launches (no per-launch events: "
                                   "they would sit between the launches)",
                         "traffic_note": "ncu --set full, per launch (profiles/); steady traffic without "
                                         "cache flushes in traffic_steady", "traffic_steady": traffic_steady,
                         "peak_live": live_peaks,
                         "frac_note": "peak = a measured torch copy_ (read + write bytes), not a hardware limit: "
                                      "the kernel's steady DRAM traffic equals its algorithmic bytes "
                                      "(traffic_steady: ncu, back to back), so a frac a little above 1 is a "
                                      "faster copy than torch's, not skipped bytes",
                         "in_step": {"avg_launch_us": k_us, "achieved": k_ach,
                                     "frac": (k_ach / kpeak) if k_ach else None, "launches": tl,
                                     "kernel_us": tk_ns / tk / 1e3 if tk else None,
                                     "kernel_achieved": (rw * t_bytes / max(tl, 1)) / (tk_ns / tk) if tk else None,
                                     "kernel_frac": ((rw * t_bytes / max(tl, 1)) / (tk_ns / tk) / kpeak) if tk
                                     else None,
                                     "kernel_what": "the same launches timed by the kernel itself: latest CTA end "
                                                    "minus earliest CTA start (%globaltimer), host submission "
                                                    "and launch latency excluded",
                                     "what": "the same kernel inside the workflow's timed region, CUDA events "
                                             "recorded around every launch on its stream (GROUTER_PROFILE): "
                                             "each launch runs alone (requests are PCIe-paced), so the "
                                             "interval also holds the launch latency and the grid's ramp-up "
                                             "that back-to-back launches overlap, and with 4 client threads "
                                             "the host's gap between the start event and the launch call "
                                             "(tools/instep.py: 19-22 us with one client); kernel_us is the "
                                             "kernel's own span in the same launches -- shorter than back to "
                                             "back because the tensor the copy engine has just written is "
                                             "partly still in L2"}},
            "roofline_step": {"bound": "pcie", "achieved": value / world * N_BYTES / 1e9,
                              "peak": link_peak, "unit": "GB/s",
                              "frac": value / world * N_BYTES / 1e9 / link_peak,
                              "what": "per-GPU payload GB/s of the workflow against this box's pinned "
                                      "single-link H2D (bare cudaMemcpyAsync of 256 MiB back to back): the "
                                      "link every request crosses once"},
            "cpu_baseline": cpu,
            "e2e": {"value": e2e_val, "unit": "req/s", "h2d_bytes_per_step": R * N_BYTES,
                    "d2h_bytes_per_step": R * 8, "steps": e2e_steps, "outstanding": Q,
                    "what": "the same closed loop through the C ABI, wall clock, plus an 8 B D2H read of "
                            "each delivered tensor"},
            "gpu_launches": launches,
            "clocks": clocks,
        }
        if cfg2 is not None:
            line["cfg2"] = cfg2
        if sweep is not None:
            line["sweep"] = sweep
        if nccl is not None:
            line["nccl_p2p_baseline"] = nccl
        if multipath is not None:
            line["h2d_multipath"] = multipath
        if same_gpu and world > 1:
            line["note"] = ("GR_BENCH_SAME_GPU: every rank on device 0 (plumbing check): the 'NVLink' push is a "
                            "same-device copy")
        print(json.dumps(line), flush=True)
    if stuck:   # a measurement thread still owns the GPUs: leave without teardown
        sys.stdout.flush()
        os._exit(0)
    try:
        ctx.close()
    except Exception as e:  # the line is out; a teardown failure must not fail the run
        print(f"[bench] teardown: {e}", file=sys.stderr, flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=350,
                    help="timed steps (20 requests each): 350 = ~5 s of closed loop at one GPU (SURVEY §8(d))")
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="grouter", choices=["grouter", "reference"])
    ap.add_argument("--requests", type=int, default=20)
    ap.add_argument("--q", type=int, default=4, help="requests outstanding per GPU (SURVEY §8(d): 4)")
    ap.add_argument("--e2e-steps", type=int, default=10)
    ap.add_argument("--b2b-steps", type=int, default=200)
    ap.add_argument("--lat-samples", type=int, default=200)
    ap.add_argument("--cpu-seconds", type=float, default=10.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-sweep", action="store_true")
    ap.add_argument("--tma", action="store_true")
    ap.add_argument("--ctas", type=int, default=4)
    ap.add_argument("--no-multipath-probe", action="store_true")
    ap.add_argument("--multipath-timeout", type=float, default=300.0,
                    help="N>1: seconds rank 0 waits for the node-wide multipath/D2D measurement")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank)
        return
    # GR_BENCH_SAME_GPU=1 + GR_BENCH_BACKEND=gloo: every rank on GPU 0 (exercises the
    # N>1 plumbing on a 1-GPU box; NCCL refuses two ranks on one GPU)
    if os.environ.get("GR_BENCH_SAME_GPU") == "1":
        local_rank = 0
    if world > 1:
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(local_rank)
        backend = os.environ.get("GR_BENCH_BACKEND", "nccl")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device(f"cuda:{local_rank}"))
        else:
            dist.init_process_group(backend)
        CPU_GROUP[0] = dist.new_group(backend="gloo")   # GPU-free waits and the max over ranks
    run_gpu(args, rank, world, local_rank)
    if world > 1:
        import torch.distributed as dist
        try:
            dist.destroy_process_group()
        except Exception as e:
            print(f"[bench] destroy_process_group: {e}", file=sys.stderr, flush=True)


if __name__ == "__main__":
    main()
