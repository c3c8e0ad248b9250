"""Library-side trace runner: drives libgrouter.so (through the ctypes
binding) over a ``synth.traces`` op list and records the same observables as
``oracle.runner`` (status, oid, where, victims, pool usage, delivered bytes,
dispatch log).  PyTorch only supplies device buffers and streams.

Delivered bytes are copied back and compared with the oracle's in full
(``keep_bytes``) or by digest; device payloads are produced with the K9 fill
kernel (test infrastructure) or copied from the host generator.
"""
from __future__ import annotations

import ctypes
import os
import time

import numpy as np
import torch

from oracle.runner import CANARY, GUARD, digest
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G
from synth.payload import payload

HOST = -1


class DevView:
    """Exposes a raw device pointer to torch via __cuda_array_interface__."""

    def __init__(self, ptr, n):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": "|u1", "data": (ptr, False),
                                         "version": 3, "strides": None}


def read_device(ptr: int, n: int, device: int) -> np.ndarray:
    if n == 0:
        return np.zeros(0, np.uint8)
    t = torch.as_tensor(DevView(ptr, n), device=f"cuda:{device}")
    return t.cpu().numpy().copy()


def read_host(ptr: int, n: int) -> np.ndarray:
    if n == 0:
        return np.zeros(0, np.uint8)
    return np.frombuffer((ctypes.c_uint8 * n).from_address(ptr), dtype=np.uint8).copy()


def wait_streams(streams, timeout=60.0):
    t0 = time.time()
    for s in streams:
        while not s.query():
            if time.time() - t0 > timeout:
                raise TimeoutError("stream did not drain (missing completion publish?)")
            time.sleep(0.0005)


class LibRunner:
    def __init__(self, calib, host_store_bytes=1 << 30, pool_cap=None, replay=True, flags=0,
                 keep_bytes=False, pool_floor=64 << 20, chunk_bytes=None, targets=False):
        self.calib = calib
        n = calib["n_gpus"]
        self.n = n
        self.phys = calib.get("device_map", list(range(n)))
        caps = pool_cap if pool_cap is not None else [G.UNLIMITED] * n
        # auto_cap_period_us=0: a trace's refresh_cap ops are the only cap
        # refreshes (the background thread would re-measure free memory)
        kw = dict(host_store_bytes=host_store_bytes, pool_cap=caps, pool_floor_bytes=pool_floor,
                  flags=(G.REPLAY if replay else 0) | flags, auto_cap_period_us=0)
        if chunk_bytes:
            kw["chunk_bytes"] = chunk_bytes
        self.ctx = G.Ctx(G.config_from_calib(calib, **kw))
        self.replay = replay
        self.targets = targets
        if targets:
            self.ctx.set_clock(0)        # the oracle's clock starts at 0 (R44)
        self.streams = [torch.cuda.Stream(device=p) for p in self.phys]
        self.upload = [torch.cuda.Stream(device=p) for p in self.phys]
        self.keep_bytes = keep_bytes
        self.keep = []          # buffers that must outlive their use
        self.pending = []       # (rec, verifier) to check after the next flush

    def close(self):
        self.ctx.close()

    def _stream(self, dev):
        return self.streams[dev].cuda_stream if dev >= 0 else 0

    def _fnc(self, f):
        return G.fn(f["wf"], f["fid"], f["dev"])

    def _verify(self, rec, got):
        rec["digest"] = digest(got)
        if self.keep_bytes:
            rec["bytes"] = got

    def _flush_and_verify(self):
        try:
            wait_streams(self.streams)
        except TimeoutError:
            print(self.ctx.dump(), flush=True)
            raise
        for rec, fnv in self.pending:
            self._verify(rec, fnv())
        self.pending = []

    def run(self, ops):
        recs = []
        ctx = self.ctx
        trace = bool(os.environ.get("GR_TRACE"))
        for i, op in enumerate(ops):
            k = op["op"]
            rec = {"i": i, "op": k}
            if trace:
                print("op", i, {a: b for a, b in op.items() if a != "seed"}, flush=True)
            oid = 0
            if "ref" in op and op["ref"] < len(recs):
                oid = recs[op["ref"]].get("oid", 0)
            if k == "put":
                f, n = op["fn"], op["n"]
                data = payload(op["seed"], n)
                align = op.get("src_align", 0)
                if f["dev"] == HOST:
                    if i % 2 == 0:   # pinned source: DMA straight from the caller's buffer
                        buf = torch.empty(n + align + 1, dtype=torch.uint8, pin_memory=True)
                        arr = buf.numpy()
                    else:            # pageable source: goes through the circular pinned ring
                        arr = np.empty(n + align + 1, np.uint8)
                        buf = arr
                    arr[align:align + n] = data
                    ptr = arr.ctypes.data + align
                else:
                    dev = self.phys[f["dev"]]
                    buf = torch.empty(n + align + 1, dtype=torch.uint8, device=f"cuda:{dev}")
                    # upload on a side stream: in replay mode the caller stream may be
                    # parked on a completion word until the next flush
                    up = self.upload[f["dev"]]
                    with torch.cuda.stream(up):
                        buf[align:align + n].copy_(torch.from_numpy(data).to(f"cuda:{dev}",
                                                                             non_blocking=False))
                    self.streams[f["dev"]].wait_stream(up)
                    ptr = buf.data_ptr() + align
                self.keep.append(buf)
                st, o = ctx.put(self._fnc(f), ptr, n, op["hint"], op["consumers"],
                                self._stream(f["dev"]))
                if st == G.OK:
                    rec["oid"] = oid = o
            elif k == "alloc":
                f, n = op["fn"], op["n"]
                st, buf, o = ctx.alloc(self._fnc(f), n, op["hint"], op["consumers"])
                if st == G.OK:
                    rec["oid"] = oid = o
                    rec["buf"] = buf
                    if n:
                        if f["dev"] == HOST:
                            data = payload(op["seed"], n)   # keep alive across memmove
                            ctypes.memmove(buf, data.ctypes.data, n)
                        else:
                            with torch.cuda.device(self.phys[f["dev"]]):
                                G.check(G.test_fill(buf, n, op["seed"], 0, self._stream(f["dev"])))
            elif k == "seal":
                f = op["fn"]
                st = ctx.seal(self._fnc(f), oid, self._stream(f["dev"]))
            elif k == "get":
                f = op["fn"]
                st, ptr, n = ctx.get(self._fnc(f), oid, self._stream(f["dev"]))
                if st == G.OK:
                    rec["n"], rec["ptr"] = n, ptr
                    dev = f["dev"]
                    if dev == HOST:
                        self._verify(rec, read_host(ptr, n))
                    else:
                        pd = self.phys[dev]
                        self.pending.append((rec, lambda p=ptr, n=n, pd=pd: read_device(p, n, pd)))
                        if not self.replay:
                            self._flush_and_verify()
            elif k == "get_into":
                f = op["fn"]
                o = None
                n_exp = op.get("cap")
                align = op.get("dst_align", 0)
                # size the destination from the oracle-visible object size
                st_w, _ = ctx.where(oid)
                n_obj = self._size_of.get(oid, 0)
                cap = op.get("cap", n_obj)
                total = align + max(cap, n_obj) + GUARD
                dev = f["dev"]
                if dev == HOST:
                    dst = np.full(total, CANARY, np.uint8)
                    dptr = dst.ctypes.data + align
                else:
                    dst = torch.full((total,), CANARY, dtype=torch.uint8, device=f"cuda:{self.phys[dev]}")
                    torch.cuda.default_stream(self.phys[dev]).synchronize()
                    dptr = dst.data_ptr() + align
                self.keep.append(dst)
                st, n = ctx.get_into(self._fnc(f), oid, dptr, cap, self._stream(dev))
                del o, n_exp, st_w
                if st == G.OK:
                    rec["n"] = n

                    def check(dst=dst, align=align, n=n, dev=dev):
                        a = dst if dev == HOST else dst.cpu().numpy()
                        assert (a[:align] == CANARY).all() and (a[align + n:] == CANARY).all(), \
                            "get_into wrote outside [dst, dst+n)"
                        return a[align:align + n].copy()
                    if dev == HOST:
                        self._verify(rec, check())
                    else:
                        self.pending.append((rec, check))
                        if not self.replay:
                            self._flush_and_verify()
            elif k == "release":
                f = op["fn"]
                g = recs[op["get"]]
                gop = ops[op["get"]]
                goid = recs[gop["ref"]].get("oid", 0) if "ref" in gop else 0
                st = ctx.release(self._fnc(f), goid, g.get("ptr", 0), self._stream(f["dev"]))
                oid = goid
            elif k == "free":
                st = ctx.free(self._fnc(op["fn"]), oid)
            elif k == "weight":
                st = ctx.set_tenant_weight(op["wf"], op["w"])
            elif k == "tick":
                st = ctx.set_clock(op["t_ns"])
            elif k == "slo":
                st = ctx.set_tenant_slo(op["wf"], op["data"], op["slo_ns"], op["infer_ns"])
            elif k == "next_use":
                st = ctx.set_next_use(oid, op["pos"])
            elif k == "pool_limit":
                st = ctx.set_pool_limit(op["dev"], op["bytes"])
            elif k == "refresh_cap":
                st, cap = ctx.refresh_cap(op["dev"], op["avail"])
                if st in (G.OK, G.ENOMEM):
                    rec["cap"] = cap
            elif k == "flush":
                st = ctx.flush()
                self._flush_and_verify()
            else:
                raise ValueError(k)
            if st == G.OK and k in ("put", "alloc"):
                self._size_of[rec["oid"]] = op["n"]
            rec["status"] = G.STATUS[st]
            if trace:
                print("   ->", G.STATUS[st], G.last_error() if st else "", flush=True)
            rec["victims"] = ctx.victims()
            rec["restored"] = ctx.restored()
            if self.targets:
                rec["pool_target"] = [ctx.pool_target(d) for d in range(self.n)]
            s = ctx.stats()
            rec["used"] = [s.used[d] for d in range(self.n)]
            rec["host_used"] = s.host_used
            if oid:
                stw, loc = ctx.where(oid)
                rec["where"] = loc if stw == G.OK else None
            recs.append(rec)
        self._flush_and_verify()
        dispatch = ctx.dispatch_log()
        # replay mode may leave transfers no later op waited for queued: the
        # per-tenant totals count every enqueued chunk once dispatched
        G.check(ctx.flush(), "flush")
        G.check(ctx.sync(), "sync")
        tenants = sorted({op["fn"]["wf"] for op in ops if isinstance(op.get("fn"), dict)})
        return {"records": recs, "dispatch": dispatch, "stats": ctx.stats(),
                "tenant_bytes": {wf: ctx.tenant_stats(wf) for wf in tenants}}

    _size_of: dict

    def __call__(self, ops):
        self._size_of = {}
        return self.run(ops)


KIND = {"copy": 0, "h2d": 1, "d2h": 2}


def compare(orc_out, lib_out, check_dispatch=True):
    """Asserts record-by-record parity; returns the number of byte-compared gets."""
    o_recs, l_recs = orc_out["records"], lib_out["records"]
    assert len(o_recs) == len(l_recs)
    compared = 0
    for o, l in zip(o_recs, l_recs):
        ctx = (o["i"], o["op"])
        assert l["status"] == o["status"], (ctx, o, l)
        assert l.get("oid") == o.get("oid"), ctx
        assert l.get("where") == o.get("where"), (ctx, o.get("where"), l.get("where"))
        assert l["victims"] == o["victims"], (ctx, o["victims"], l["victims"])
        assert l.get("restored", []) == o.get("restored", []), (ctx, o.get("restored"), l.get("restored"))
        if "pool_target" in o and "pool_target" in l:
            assert l["pool_target"] == o["pool_target"], (ctx, o["pool_target"], l["pool_target"])
        assert l["used"] == o["used"], (ctx, o["used"], l["used"])
        assert l["host_used"] == o["host_used"], ctx
        assert l.get("cap") == o.get("cap"), (ctx, o.get("cap"), l.get("cap"))
        if o["status"] == "OK" and o["op"] in ("get", "get_into"):
            assert l["n"] == o["n"], ctx
            if "bytes" in o and "bytes" in l:
                if not np.array_equal(l["bytes"], o["bytes"]):
                    bad = np.nonzero(l["bytes"] != o["bytes"])[0]
                    raise AssertionError(f"{ctx}: {bad.size} of {o['n']} bytes differ, first at "
                                         f"{bad[0]}, last at {bad[-1]}; lib[:8]={l['bytes'][bad[0]:bad[0]+8]} "
                                         f"orc[:8]={o['bytes'][bad[0]:bad[0]+8]}")
            assert l["digest"] == o["digest"], ctx
            compared += 1
    if "tenant_bytes" in lib_out and "oracle" in orc_out:
        # per-tenant dispatched bytes per server kind (L193, grouter_tenant_stats):
        # independent of dispatch timing, so real-time runs compare too
        tb = orc_out["oracle"].tenant_bytes
        for wf, got in lib_out["tenant_bytes"].items():
            exp = [tb.get((wf, k), 0) for k in ("copy", "h2d", "d2h")]
            assert got == exp, (wf, got, exp)
    if check_dispatch:
        olog = {}
        for r in o_recs:
            for d in r.get("dispatched", []):
                key = (KIND[d["server"][0]], d["server"][1])
                olog.setdefault(key, []).append((d["tenant"], [tuple(c) for c in d["chunks"]]))
        llog = {}
        for d in lib_out["dispatch"]:
            llog.setdefault((d["kind"], d["dev"]), []).append((d["tenant"], d["chunks"]))
        assert llog == olog
    return compared
