"""Trace runner for the oracle.

Executes a ``synth.traces`` op list against ``model.Oracle`` and records, per
op: status, the created oid, ``where`` of the referenced object after the op,
the ordered victims, the transfer plan, and a digest of the delivered bytes.
At each ``flush`` it records the dispatch log (replay mode).

The runner also checks the identity pin on itself: every delivered byte
string must equal the SplitMix64 payload the producing op wrote (I2).
"""
from __future__ import annotations

import hashlib

import numpy as np

from synth.payload import payload

from .model import HOST, STATUS, Oracle

CANARY = 0xA5
GUARD = 64


def digest(b: np.ndarray) -> str:
    return hashlib.blake2b(np.ascontiguousarray(b).tobytes(), digest_size=16).hexdigest()


def run(ops: list, calib: dict, host_store_bytes: int = 1 << 40, pool_cap=None,
        multipath: bool = True, keep_bytes: bool = False, restore: bool = False,
        pool_floor: int | None = None, targets: bool = False, d2h_multipath: bool = False,
        striped_migration: bool = False, host_centric: bool = False) -> dict:
    kw = {} if pool_floor is None else {"pool_floor": pool_floor}
    kw["d2h_multipath"] = d2h_multipath
    kw["striped_migration"] = striped_migration
    kw["host_centric"] = host_centric
    orc = Oracle(calib, host_store_bytes=host_store_bytes, pool_cap=pool_cap,
                 multipath=multipath, restore=restore, **kw)
    recs = []
    seed_of = {}          # oid -> payload seed
    for i, op in enumerate(ops):
        k = op["op"]
        rec = {"i": i, "op": k}
        oid = 0
        if "ref" in op:
            oid = recs[op["ref"]].get("oid", 0) if op["ref"] < len(recs) else 0
        if k == "put":
            n = op["n"]
            src = payload(op["seed"], n)
            st, out = orc.put(op["fn"], src, n, op["hint"], op["consumers"])
            if st == 0:
                rec["oid"] = out["oid"]
                rec["plan"] = out["plan"]
                seed_of[out["oid"]] = op["seed"]
                oid = out["oid"]
        elif k == "alloc":
            st, out = orc.alloc(op["fn"], op["n"], op["hint"], op["consumers"])
            if st == 0:
                rec["oid"] = out["oid"]
                out["buf"][...] = payload(op["seed"], op["n"])   # the function writes
                seed_of[out["oid"]] = op["seed"]
                oid = out["oid"]
        elif k == "seal":
            st, out = orc.seal(op["fn"], oid)
        elif k == "get":
            st, out = orc.get(op["fn"], oid)
            if st == 0:
                rec["n"] = out["n"]
                rec["handle"] = out["handle"]
                rec["plan"] = out["plan"]
                rec["zero_copy"] = bool(out["handle"] and out["handle"][0] == "obj")
                got = out.get("buf", np.zeros(0, np.uint8))
                assert np.array_equal(got, payload(seed_of[oid], out["n"])), "identity (I2)"
                rec["digest"] = digest(got)
                if keep_bytes:
                    rec["bytes"] = got.copy()
        elif k == "get_into":
            o = orc.objects.get(oid)
            n = o.n if o is not None else 0
            align = op.get("dst_align", 0)
            cap = op.get("cap", n)
            dst = np.full(align + max(cap, n) + GUARD, CANARY, dtype=np.uint8)
            st, out = orc.get_into(op["fn"], oid, dst[align:align + max(cap, 0)], cap)
            if st == 0:
                got = dst[align:align + out["n"]]
                assert np.array_equal(got, payload(seed_of[oid], out["n"])), "identity (I2)"
                assert (dst[:align] == CANARY).all() and (dst[align + out["n"]:] == CANARY).all()
                rec["n"] = out["n"]
                rec["plan"] = out["plan"]
                rec["digest"] = digest(got)
                if keep_bytes:
                    rec["bytes"] = got.copy()
        elif k == "release":
            g = recs[op["get"]]
            handle = g.get("handle")
            goid = recs[ops[op["get"]]["ref"]].get("oid", 0) if "ref" in ops[op["get"]] else 0
            st, out = orc.release(op["fn"], goid, handle)
            oid = goid
        elif k == "free":
            st, out = orc.free(op["fn"], oid)
        elif k == "weight":
            st, out = orc.set_weight(op["wf"], op["w"])
        elif k == "tick":
            st, out = orc.tick(op["t_ns"])
        elif k == "slo":
            st, out = orc.set_slo(op["wf"], op["data"], op["slo_ns"], op["infer_ns"])
        elif k == "next_use":
            st, out = orc.set_next_use(oid, op["pos"])
        elif k == "pool_limit":
            st, out = orc.set_pool_limit(op["dev"], op["bytes"])
        elif k == "refresh_cap":
            st, out = orc.refresh_cap(op["dev"], op["avail"])
            if "cap" in out:
                rec["cap"] = out["cap"]
        elif k == "flush":
            st, out = orc.flush()
            rec["dispatched"] = out["dispatched"]
        else:
            raise ValueError(k)
        if st == 0 and k in ("put", "get", "get_into") and op["fn"]["dev"] == HOST:
            # a CPU caller blocks until its bytes are in place; in replay mode
            # that dispatches everything queued (R31)
            victims, restored = list(orc.victims), list(orc.restored)
            _, fl = orc.flush()
            orc.victims, orc.restored = victims, restored
            rec["dispatched"] = fl["dispatched"]
        rec["status"] = STATUS[st]
        rec["victims"] = list(orc.victims)
        rec["restored"] = list(orc.restored)
        if targets:
            rec["pool_target"] = [orc.pool_target(d) for d in range(orc.ngpu)]
        rec["used"] = list(orc.used)
        rec["host_used"] = orc.host_used
        if oid:
            rec["where"] = orc.where(oid)
        recs.append(rec)
        _check_invariants(orc)
    return {"records": recs, "oracle": orc}


def _check_invariants(orc: Oracle) -> None:
    """I4 capacity (used <= cap unless an over-cap limit could not be met --
    see DESIGN.md R31) and host store bound; I6 refcount sanity."""
    assert 0 <= orc.host_used <= orc.H
    for d in range(orc.ngpu):
        assert orc.used[d] >= 0
    for o in orc.objects.values():
        assert o.pins >= 0
        assert o.loc == HOST or 0 <= o.loc < orc.ngpu
