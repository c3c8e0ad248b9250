"""Chunk splitter -- exact minimum-makespan split.

Paper basis:
* L182 §4.3.1: "GROUTER splits data into small chunks (2 MB by default) and
  precomputes a parallel transfer plan.  Chunks are pipelined across GPU
  streams" -> C = 2 MiB (R1), the plan is computed before any byte moves.
* L242 §4.3.3: chunk size proportional to path capacity ("a 48 GB/s link
  receives twice the chunk size of a 24 GB/s link") -> C_p (R2).
* The paper states no objective for WHICH bytes take which path (R3); the
  reading is the exact min-makespan under the per-path cost T_p, canonical
  fill in route order, interleaved layout (R4).

All arithmetic is on Python ints (R30): bytes, bytes/s, picoseconds.
"""
from __future__ import annotations

from .routes import path_params, route_set

CHUNK = 2 * 1024 * 1024          # L182 "2 MB", read as 2 MiB (R1)
GRANULE = 4096                   # split granule g (O6)
PS = 10**12


def ceil_div(a: int, b: int) -> int:
    return -(-a // b)


def chunk_sizes(betas: list, C: int = CHUNK, g: int = GRANULE) -> list:
    """C_p = max(g, floor((C * beta_p / beta_max) / g) * g)   (L242, R2)."""
    bmax = max(betas)
    return [max(g, (C * b) // (bmax * g) * g) for b in betas]


def path_time(m: int, alpha: int, beta: int, phi: int, Cp: int, g: int = GRANULE) -> int:
    """T_p(m) = 0 if m = 0 else phi + ceil(m*g/C_p)*alpha + ceil(m*g*1e12/beta)  [ps]."""
    if m == 0:
        return 0
    return phi + ceil_div(m * g, Cp) * alpha + ceil_div(m * g * PS, beta)


def path_cap(T: int, N: int, alpha: int, beta: int, phi: int, Cp: int, g: int = GRANULE) -> int:
    """cap_p(T) = max{m <= N : T_p(m) <= T}; T_p is monotone so bisect."""
    lo, hi = 0, N  # invariant: T_p(lo) <= T (T >= 0), answer in [lo, hi]
    while lo < hi:
        mid = (lo + hi + 1) // 2
        if path_time(mid, alpha, beta, phi, Cp, g) <= T:
            lo = mid
        else:
            hi = mid - 1
    return lo


def split_shares(N: int, params: list, Cps: list, g: int = GRANULE) -> tuple:
    """Steps 1-2 of O6.  Returns (T_star, shares) with shares in route order.

    T* = min{T : sum_p cap_p(T) >= N}; s_p = min(cap_p(T*), remaining)."""
    if N == 0:
        return 0, [0] * len(params)
    a0, b0, f0 = params[0]
    hi = path_time(N, a0, b0, f0, Cps[0], g)       # everything on p0 is feasible
    lo = 0
    while lo < hi:
        mid = (lo + hi) // 2
        tot = sum(path_cap(mid, N, a, b, f, c, g) for (a, b, f), c in zip(params, Cps))
        if tot >= N:
            hi = mid
        else:
            lo = mid + 1
    T = lo
    shares, rem = [], N
    for (a, b, f), c in zip(params, Cps):
        s = min(path_cap(T, N, a, b, f, c, g), rem)
        shares.append(s)
        rem -= s
    assert rem == 0
    return T, shares


def layout(n: int, shares: list, Cps: list, routes: list, g: int = GRANULE) -> list:
    """Step 3 of O6: interleaved rounds; each round visits paths in route
    order and emits min(C_p/g, rem_p) granules as one chunk at the running
    offset; the final chunk is clipped to end at n.
    Chunk = dict(offset, bytes, path, route_gpu)."""
    rem = list(shares)
    chunks, off = [], 0
    while any(rem):
        for p, r in enumerate(routes):
            if rem[p] == 0:
                continue
            m = min(Cps[p] // g, rem[p])
            chunks.append({"offset": off, "bytes": m * g, "path": p, "route_gpu": r})
            off += m * g
            rem[p] -= m
    if chunks:
        last = chunks[-1]
        last["bytes"] = n - last["offset"]
    return chunks


def plan_h2d(calib: dict, d: int, n: int, multipath: bool = True,
             C: int = CHUNK, g: int = GRANULE) -> list:
    """Full O6 plan for host -> GPU d over R(d)."""
    if n == 0:
        return []
    routes = route_set(calib, d, multipath)
    params = [path_params(calib, d, r) for r in routes]
    Cps = chunk_sizes([b for _, b, _ in params], C, g)
    N = ceil_div(n, g)
    _, shares = split_shares(N, params, Cps, g)
    return layout(n, shares, Cps, routes, g)


def plan_d2h(calib: dict, s: int, n: int, multipath: bool = True,
             C: int = CHUNK, g: int = GRANULE) -> list:
    """gFn-host plan (L178, Fig. 5a: "data from GPU1 is first routed via NVLink
    to peer GPUs ..., which concurrently stage it to host memory through their
    PCIe links"): GPU s -> r in R(s) -> host.  The calibration measures PCIe in
    the host->GPU direction and the reading takes it as symmetric (R45), so a
    path s -> r -> host has the parameters of host -> r -> s and the split is
    the O6 split of plan_h2d(s, n); route_gpu = the GPU whose copy engine
    moves the chunk to host memory."""
    return plan_h2d(calib, s, n, multipath, C, g)


def plan_single(n: int, route_gpu: int, C: int = CHUNK) -> list:
    """k = 1 plan (D2D, same-GPU copy, D2H): consecutive chunks of C bytes,
    the last one clipped (L182 chunking on a single direct path)."""
    return [{"offset": o, "bytes": min(C, n - o), "path": 0, "route_gpu": route_gpu}
            for o in range(0, n, C)]


def makespan(shares: list, params: list, Cps: list, g: int = GRANULE) -> int:
    return max((path_time(s, a, b, f, c, g) for s, (a, b, f), c in zip(shares, params, Cps)),
               default=0)
