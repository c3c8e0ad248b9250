"""Request traces.  Inputs only.

A trace is a list of op dicts, executed in order by a runner (the oracle's
``oracle.runner`` or the library-side runner under ``tests/``).  Objects are
referenced by the index of the op that created them (``ref``); leases by the
index of the get that produced them (``get``).  ``fn`` is
``{"wf": workflow_id, "fid": function_id, "dev": device}`` with device -1 for a
CPU function (``GROUTER_HOST``).  Payload bytes of a put/alloc op are
``synth.payload.payload(seed, n)``.

ops:
  put       fn n hint consumers seed [src_align]
  alloc     fn n hint consumers seed      (runner fills buffer, then seal op)
  seal      fn ref
  get       fn ref
  get_into  fn ref [dst_align] [cap]
  release   fn get
  free      fn ref
  weight    wf w
  next_use  ref pos
  pool_limit dev bytes
  refresh_cap dev avail      (O10 auto cap with `avail` bytes available to the store)
  flush
"""
from __future__ import annotations

import math
import random

from .payload import op_seed

HOST = -1
NOHINT = -2
MiB = 1 << 20

CFG1_BYTES = 64 * 3 * 224 * 224 * 4            # 38,535,168 (R25)
CFG2_FRAME = 8 * 3 * 640 * 640 * 4             # 39,321,600
CFG2_CROP = 3 * 224 * 224 * 4                  # 602,112
CFG5_KV = 2 * 8 * 8192 * 128 * 2               # 33,554,432 per layer
CFG5_HIDDEN = 8192 * 4096 * 2                  # 67,108,864
CFG5_LAYERS = 32


def fn(wf, fid, dev):
    return {"wf": wf, "fid": fid, "dev": dev}


class Builder:
    def __init__(self, run_seed: int = 1):
        self.ops = []
        self.run_seed = run_seed

    def _add(self, op):
        self.ops.append(op)
        return len(self.ops) - 1

    def seed(self):
        return op_seed(self.run_seed, len(self.ops))

    def put(self, f, n, hint=NOHINT, consumers=0, src_align=0):
        return self._add({"op": "put", "fn": f, "n": n, "hint": hint,
                          "consumers": consumers, "seed": self.seed(), "src_align": src_align})

    def alloc(self, f, n, hint=NOHINT, consumers=0):
        return self._add({"op": "alloc", "fn": f, "n": n, "hint": hint,
                          "consumers": consumers, "seed": self.seed()})

    def seal(self, f, ref):
        return self._add({"op": "seal", "fn": f, "ref": ref})

    def get(self, f, ref):
        return self._add({"op": "get", "fn": f, "ref": ref})

    def get_into(self, f, ref, dst_align=0, cap=None):
        op = {"op": "get_into", "fn": f, "ref": ref, "dst_align": dst_align}
        if cap is not None:
            op["cap"] = cap
        return self._add(op)

    def release(self, f, get):
        return self._add({"op": "release", "fn": f, "get": get})

    def free(self, f, ref):
        return self._add({"op": "free", "fn": f, "ref": ref})

    def weight(self, wf, w):
        return self._add({"op": "weight", "wf": wf, "w": w})

    def tick(self, t_ns):
        return self._add({"op": "tick", "t_ns": t_ns})

    def slo(self, wf, data, slo_ns, infer_ns):
        return self._add({"op": "slo", "wf": wf, "data": data, "slo_ns": slo_ns, "infer_ns": infer_ns})

    def next_use(self, ref, pos):
        return self._add({"op": "next_use", "ref": ref, "pos": pos})

    def pool_limit(self, dev, nbytes):
        return self._add({"op": "pool_limit", "dev": dev, "bytes": nbytes})

    def refresh_cap(self, dev, avail):
        return self._add({"op": "refresh_cap", "dev": dev, "avail": avail})

    def flush(self):
        return self._add({"op": "flush"})


def cfg1(n_gpus: int, iters: int = 20, run_seed: int = 1000, scale: int = 1,
         consumer_mode: str = "get") -> list:
    """Config 1 (R24): cFn put(hint=GPU0) -> gFn on GPU1 get (GPU0 at N=1)."""
    n = CFG1_BYTES // scale
    b = Builder(run_seed)
    cfn = fn(1, 1, HOST)
    gfn = fn(1, 2, 1 if n_gpus > 1 else 0)
    for _ in range(iters):
        o = b.put(cfn, n, hint=0, consumers=1)
        if consumer_mode == "get":
            g = b.get(gfn, o)
            b.flush()
            b.release(gfn, g)
        else:
            b.get_into(gfn, o)
            b.flush()
    return b.ops


def cfg2(n_gpus: int, requests: int = 8, run_seed: int = 2000, scale: int = 1) -> list:
    """Config 2, Traffic: frame put by decode cFn (hint = YOLO GPU y), YOLO get,
    YOLO allocs person/vehicle crops (K ~ Poisson(4) clipped to [0,32]),
    recognition gFns on (y+1)%N and (y+2)%N get them."""
    rng = random.Random(run_seed)
    b = Builder(run_seed)
    frame = CFG2_FRAME // scale
    crop = CFG2_CROP // scale

    def poisson(lam):
        L, k, p = math.exp(-lam), 0, 1.0
        while True:
            p *= rng.random()
            if p <= L:
                return min(k, 32)
            k += 1

    for i in range(requests):
        wf = 10 + i
        y = i % n_gpus
        dec = fn(wf, 1, HOST)
        yolo = fn(wf, 2, y)
        rp = fn(wf, 3, (y + 1) % n_gpus)
        rv = fn(wf, 4, (y + 2) % n_gpus)
        o = b.put(dec, frame, hint=y, consumers=1)
        g = b.get(yolo, o)
        kp, kv = poisson(4.0), poisson(4.0)
        a1 = b.alloc(yolo, kp * crop, consumers=1)
        b.seal(yolo, a1)
        a2 = b.alloc(yolo, kv * crop, consumers=1)
        b.seal(yolo, a2)
        g1 = b.get(rp, a1)
        g2 = b.get(rv, a2)
        b.flush()
        b.release(yolo, g)
        b.release(rp, g1)
        b.release(rv, g2)
    return b.ops


def cfg4(n_gpus: int, rounds: int = 4, run_seed: int = 4000, scale: int = 1,
         weights=(1, 1, 2, 2, 4, 4, 8, 8), slos=None) -> list:
    """Config 4: 8 workflows with weights; each round every tenant puts a
    tensor from host, gets it on GPU t%N, allocs an output and the next GPU
    gets it.  The gets of one round are flushed together (replay-mode
    dispatch log is the compared artefact)."""
    b = Builder(run_seed)
    n = CFG1_BYTES // scale
    T = len(weights) if slos is None else len(slos)
    if slos is None:
        for t, w in enumerate(weights):
            b.weight(100 + t, w)
    else:
        for t, (data, slo_ns, infer_ns) in enumerate(slos):
            b.slo(100 + t, data, slo_ns, infer_ns)
    for r in range(rounds):
        if slos is not None and r == 1:
            b.slo(100, 0, 0, 0)          # tenant 100 drops its SLO: everyone re-weighted
            b.weight(101, 3)             # an explicit weight replaces 101's SLO
        puts = []
        for t in range(T):
            puts.append(b.put(fn(100 + t, 1, HOST), n, hint=NOHINT, consumers=1))
        b.flush()
        gets = []
        for t in range(T):
            gets.append(b.get(fn(100 + t, 2, t % n_gpus), puts[t]))
        b.flush()
        outs = []
        for t in range(T):
            f2 = fn(100 + t, 2, t % n_gpus)
            a = b.alloc(f2, n, consumers=1)
            b.seal(f2, a)
            outs.append(a)
        gets2 = []
        for t in range(T):
            gets2.append(b.get(fn(100 + t, 3, (t + 1) % n_gpus), outs[t]))
        b.flush()
        for t in range(T):
            b.release(fn(100 + t, 2, t % n_gpus), gets[t])
            b.release(fn(100 + t, 3, (t + 1) % n_gpus), gets2[t])
    return b.ops


# SLO variant of cfg4 (L193-L197): (data_bytes, slo_ns, infer_ns) per tenant;
# data = the cfg1 tensor, SLOs 1.5-2x inference time as in L193.
CFG4_SLOS = [(CFG1_BYTES, 60_000_000, 40_000_000), (CFG1_BYTES, 80_000_000, 40_000_000),
             (CFG1_BYTES, 30_000_000, 20_000_000), (2 * CFG1_BYTES, 100_000_000, 50_000_000),
             (CFG1_BYTES, 45_000_000, 30_000_000), (4 * CFG1_BYTES, 200_000_000, 100_000_000)]


def cfg5(n_gpus: int, requests: int = 8, limit_frac=None, run_seed: int = 5000,
         scale: int = 1, layers: int = CFG5_LAYERS) -> list:
    """Config 5: stage-A gFn on GPU a allocs 32 KV objects + hidden states per
    request; stage-B gFn on GPU b gets them in queue order.  Pool limit on a
    is ``limit_frac`` of the working set (None = unlimited); next_use = queue
    position so queue-aware eviction keeps the head of the queue resident."""
    b = Builder(run_seed)
    kv, hid = CFG5_KV // scale, CFG5_HIDDEN // scale
    a_dev, b_dev = 0, (1 if n_gpus > 1 else 0)
    if limit_frac is not None:
        pages = lambda x: -(-x // (2 * MiB)) * (2 * MiB)
        ws = requests * (layers * pages(kv) + pages(hid))
        b.pool_limit(a_dev, int(ws * limit_frac) // (2 * MiB) * (2 * MiB))
    objs = []
    for r in range(requests):
        A = fn(500 + r, 1, a_dev)
        mine = []
        for nb in [kv] * layers + [hid]:
            o = b.alloc(A, nb, consumers=1)
            b.seal(A, o)
            b.next_use(o, r)          # queue position of the consuming stage-B call
            mine.append(o)
        objs.append(mine)
    for r in range(requests):
        B = fn(500 + r, 2, b_dev)
        gs = [b.get(B, o) for o in objs[r]]
        b.flush()
        for g in gs:
            b.release(B, g)
    return b.ops


def cfg5_interleaved(n_gpus: int, requests: int = 8, window: int = 3, limit_frac=0.3,
                     run_seed: int = 5500, scale: int = 1, layers: int = CFG5_LAYERS,
                     hints: bool = True) -> list:
    """Config 5 with interleaved arrivals (Fig. 18 setting):
    ``window`` requests are in flight; stage B of request r consumes (get_into)
    its objects, then stage A of request r + window produces.  The pool limit
    is ``limit_frac`` of the in-flight working set, so consumption releases
    storage that proactive restore (L260) can refill with the queue head."""
    b = Builder(run_seed)
    kv, hid = CFG5_KV // scale, CFG5_HIDDEN // scale
    a_dev, b_dev = 0, (1 if n_gpus > 1 else 0)
    pages = lambda x: -(-x // (2 * MiB)) * (2 * MiB)
    ws = window * (layers * pages(kv) + pages(hid))
    if limit_frac is not None:
        b.pool_limit(a_dev, max(2 * MiB, int(ws * limit_frac) // (2 * MiB) * (2 * MiB)))
    objs = {}

    def produce(r):
        A = fn(500 + r, 1, a_dev)
        mine = []
        for nb in [kv] * layers + [hid]:
            o = b.alloc(A, nb, consumers=1)
            b.seal(A, o)
            if hints:
                b.next_use(o, r)
            mine.append(o)
        objs[r] = mine

    for r in range(min(window, requests)):
        produce(r)
    for r in range(requests):
        B = fn(500 + r, 2, b_dev)
        for o in objs.pop(r):
            b.get_into(B, o)
        b.flush()
        if r + window < requests:
            produce(r + window)
    return b.ops


def random_trace(rng: random.Random, n_gpus: int, n_ops: int = 200, max_n: int = 9 * MiB,
                 n_wf: int = 3, host_ok: bool = True, run_seed: int = 7, flush_every: int = 4,
                 limits: bool = True, small_sizes: bool = True) -> list:
    """Fuzz trace over every op kind, including error cases (bad oids,
    workflow mismatch, double free, unsealed gets)."""
    b = Builder(run_seed)
    live, opened, gets = [], [], []
    sizes = [0, 1, 15, 16, 17, 4095, 4096, 4097, 2 * MiB - 1, 2 * MiB, 2 * MiB + 1]

    def rsize():
        if small_sizes and rng.random() < 0.5:
            return rng.choice(sizes)
        return rng.randint(0, max_n)

    def rdev(allow_host=True):
        if allow_host and host_ok and rng.random() < 0.3:
            return HOST
        return rng.randrange(n_gpus)

    def rfn(wf=None):
        return fn(wf if wf is not None else rng.randrange(1, n_wf + 1), rng.randint(1, 4), rdev())

    for w in range(1, n_wf + 1):
        b.weight(w, rng.choice([1, 2, 4]))
    since = 0
    for _ in range(n_ops):
        r = rng.random()
        if r < 0.22:
            hint = rng.choice([NOHINT, HOST] + list(range(n_gpus)))
            live.append((b.put(rfn(), rsize(), hint=hint, consumers=rng.choice([0, 0, 1, 2]),
                               src_align=rng.choice([0, 0, 1, 3, 8])), None))
        elif r < 0.32:
            f = rfn()
            i = b.alloc(f, rsize(), consumers=rng.choice([0, 1, 2]))
            opened.append((i, f))
        elif r < 0.40 and opened:
            i, f = opened.pop(rng.randrange(len(opened)))
            if rng.random() < 0.1:
                f = dict(f, wf=f["wf"] % n_wf + 1)  # EPERM case
            b.seal(f, i)
            live.append((i, f))
        elif r < 0.62 and live:
            i, _ = rng.choice(live)
            wf = b.ops[i]["fn"]["wf"] if rng.random() < 0.9 else rng.randrange(1, n_wf + 1)
            f = fn(wf, rng.randint(1, 4), rdev())
            gets.append((b.get(f, i), f))
        elif r < 0.70 and live:
            i, _ = rng.choice(live)
            f = fn(b.ops[i]["fn"]["wf"], 9, rdev())
            b.get_into(f, i, dst_align=rng.choice([0, 0, 1, 5, 16]))
        elif r < 0.80 and gets:
            g, f = gets.pop(rng.randrange(len(gets)))
            b.flush()            # the consumer has read its lease before releasing it
            b.release(f, g)
        elif r < 0.86 and live:
            i, _ = live.pop(rng.randrange(len(live)))
            b.free(fn(b.ops[i]["fn"]["wf"], 1, HOST), i)
        elif r < 0.90 and live:
            i, _ = rng.choice(live)
            b.next_use(i, rng.randint(0, 20))
        elif r < 0.915 and limits:
            b.pool_limit(rng.randrange(n_gpus), rng.randint(0, 16) * 2 * MiB)
        elif r < 0.93 and limits:   # O10 auto cap at an arbitrary (unaligned) availability
            b.refresh_cap(rng.randrange(n_gpus), rng.randint(0, 64 * MiB))
        elif r < 0.95 and opened:
            i, f = rng.choice(opened)
            b.get(f, i)  # unsealed -> ENOENT
        since += 1
        if since >= flush_every:
            b.flush()
            since = 0
    b.flush()
    # drain: release outstanding leases
    for g, f in gets:
        b.release(f, g)
    b.flush()
    return b.ops


def sizing_trace(rng: random.Random, n_gpus: int, n_ops: int = 150, run_seed: int = 77) -> list:
    """Pool-sizing trace (L250-L256, R44): a clock that advances by bursty
    intervals (tick ops), functions on several GPUs that put/alloc outputs of
    varying size, consumers that drain some of them, and idle gaps long
    enough for reservation windows to lapse."""
    b = Builder(run_seed)
    t = 0
    live = []
    fns = [fn(rng.randint(1, 3), rng.randint(1, 3), rng.randrange(n_gpus)) for _ in range(5)]
    for _ in range(n_ops):
        r = rng.random()
        if r < 0.25:
            t += rng.choice([1, 10, 100, 1000]) * 10 ** 3 * rng.randint(1, 5)
            if rng.random() < 0.1:
                t += 10 ** 9                       # idle gap: windows lapse
            b.tick(t)
        elif r < 0.6:
            f = rng.choice(fns)
            n = rng.choice([0, 1, 4096, 2 * MiB, 3 * MiB + 5, rng.randint(1, 9 * MiB)])
            if rng.random() < 0.5:
                live.append((f, b.put(f, n, consumers=1)))
            else:
                o = b.alloc(f, n, consumers=1)
                b.seal(f, o)
                live.append((f, o))
        elif live:
            f, o = live.pop(rng.randrange(len(live)))
            c = fn(f["wf"], 9, rng.randrange(n_gpus))
            b.get_into(c, o)
    b.flush()                                      # replay mode dispatches on flush (R31)
    return b.ops
