"""Tenant share scheduler -- stride scheduling over batches.

Paper basis:
* L193 §4.3.2: "data from each function is divided into smaller chunks to
  enable fine-grained transfer control ... proportionally schedules data
  chunk transfers".
* L229 "Batched data transfer": chunks are grouped into batches (default 5
  per batch); new functions inject their chunks into subsequent batches.
* North star: per-function bandwidth shares = integer tenant weights (R7).
* Readings R6 (a batch is <= 5 chunks of ONE tenant on ONE server) and R9
  (stride: scale 2**20, join pass = max(pass, V), ties -> lower id).

A server is one shared link: ("h2d", r) the copy engine of route GPU r,
("copy", g) the SM-copy egress of GPU g, ("d2h", g) GPU g's D2H engine.
"""
from __future__ import annotations

from collections import deque

BATCH = 5                 # L229 "default: 5 chunks per batch"
STRIDE_SCALE = 1 << 20    # R9


class StrideServer:
    """One server's per-tenant FIFOs and stride state."""

    def __init__(self):
        self.fifo = {}       # tenant -> deque[(chunk_id, bytes)]
        self.pass_ = {}      # tenant -> pass value (int)
        self.V = 0           # virtual time = pass of the last dispatched tenant

    def backlogged(self):
        return sorted(t for t, q in self.fifo.items() if q)

    def enqueue(self, tenant: int, chunk_id, nbytes: int) -> None:
        q = self.fifo.setdefault(tenant, deque())
        if not q:  # tenant becomes backlogged: join rule
            self.pass_[tenant] = max(self.pass_.get(tenant, 0), self.V)
        q.append((chunk_id, nbytes))

    def dispatch(self, weight_of) -> tuple | None:
        """Pick the backlogged tenant with minimum pass (ties: lower id), take
        up to BATCH chunks, V := pass_t, pass_t += ceil(bytes * 2**20 / w_t)."""
        bl = self.backlogged()
        if not bl:
            return None
        t = min(bl, key=lambda x: (self.pass_[x], x))
        q = self.fifo[t]
        batch = [q.popleft() for _ in range(min(BATCH, len(q)))]
        nbytes = sum(b for _, b in batch)
        w = weight_of(t)
        self.V = self.pass_[t]
        self.pass_[t] += -(-(nbytes * STRIDE_SCALE) // w)
        return t, [c for c, _ in batch], nbytes

    def drain(self, weight_of) -> list:
        out = []
        while True:
            d = self.dispatch(weight_of)
            if d is None:
                return out
            out.append(d)
