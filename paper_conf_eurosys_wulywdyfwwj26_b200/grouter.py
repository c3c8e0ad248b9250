"""Thin ctypes binding of include/grouter.h and include/grouter_testing.h.

Argument marshalling only: every step of the data path (placement, planning,
scheduling, eviction, copies, completion) runs inside libgrouter.so and its
sm_100a kernels.  There is no Python or CPU fallback: if the library is not
built, importing this module raises.

Names follow the C ABI (``grouter_put`` ...).  ``Ctx`` is a small
convenience wrapper returning ``(status, outputs...)`` tuples; PyTorch
tensors/streams can be passed as raw integers (``t.data_ptr()``,
``torch.cuda.current_stream().cuda_stream``).
"""
from __future__ import annotations

import ctypes as C
import os
import threading

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libgrouter.so")

MAX_GPUS = 16
MAX_PATHS = 8
HOST = -1
NOHINT = -2
REMOTE = -3
UNLIMITED = (1 << 64) - 1
AUTO_AVAIL = (1 << 64) - 1   # grouter_refresh_cap: measure free memory now

REPLAY, NO_MULTIPATH, PLAN_ONLY, LOG, COPY_TMA, PROFILE, RESTORE, D2H_MULTIPATH = \
    0x1, 0x2, 0x4, 0x8, 0x10, 0x20, 0x40, 0x80
STRIPED_MIGRATION = 0x100   # spills over R(src), restores over R(d) (R47)
NO_POOL = 0x200             # ablation "ES off" (Fig. 16): cudaMalloc/cudaFree per object
NO_TOPOLOGY = 0x400         # ablation "TA off" (Fig. 16): route sets ignore shared PCIe uplinks (R48)
HOST_CENTRIC = 0x800        # ablation "UF off" (Fig. 16): GPU -> GPU copies through host memory (R49)
FORCE_REMOTE = 0x1000       # test only: every copy-kernel round takes the peer (NVLink) branch
CE_RELAY = 0x2000           # striped H2D: route GPUs' copy engines write the destination directly
PULL_ALL = 0x4000           # measurement: cross-GPU copies on an idle server are pulled at any size (R56)

OK, EINVAL, ENOENT, EPERM, ENOMEM, EBUSY, ECUDA, ESTATE = range(8)
STATUS = ["OK", "EINVAL", "ENOENT", "EPERM", "ENOMEM", "EBUSY", "ECUDA", "ESTATE"]


class grouter_fn(C.Structure):
    _fields_ = [("workflow_id", C.c_uint32), ("function_id", C.c_uint32), ("device", C.c_int32)]


class grouter_chunk(C.Structure):
    _fields_ = [("offset", C.c_uint64), ("bytes", C.c_uint64), ("path", C.c_int32),
                ("route_gpu", C.c_int32)]


class grouter_config(C.Structure):
    _fields_ = [
        ("n_gpus", C.c_uint32),
        ("device_map", C.c_int32 * MAX_GPUS),
        ("nvl_Bps", C.c_uint64),
        ("h2d_Bps", C.c_uint64 * MAX_GPUS),
        ("h2d_alpha_ps", C.c_uint64 * MAX_GPUS),
        ("h2d_phi_ps", C.c_uint64 * MAX_GPUS),
        ("relay_phi_ps", C.c_uint64),
        ("h2d_pair_Bps", (C.c_uint64 * MAX_GPUS) * MAX_GPUS),
        ("uplink_group", C.c_int32 * MAX_GPUS),
        ("p2p", (C.c_uint8 * MAX_GPUS) * MAX_GPUS),
        ("chunk_bytes", C.c_uint64),
        ("batch_chunks", C.c_uint32),
        ("granule", C.c_uint64),
        ("pool_floor_bytes", C.c_uint64),
        ("pool_cap_permille", C.c_uint32),
        ("pool_cap_bytes", C.c_uint64 * MAX_GPUS),
        ("host_store_bytes", C.c_uint64),
        ("auto_cap_period_us", C.c_uint64),
        ("copy_ctas_per_sm", C.c_uint32),
        ("flags", C.c_uint32),
    ]


class grouter_stats_t(C.Structure):
    _fields_ = [
        ("used", C.c_uint64 * MAX_GPUS), ("cap", C.c_uint64 * MAX_GPUS),
        ("mapped", C.c_uint64 * MAX_GPUS), ("host_used", C.c_uint64), ("host_cap", C.c_uint64),
        ("spill_count", C.c_uint64), ("spill_bytes", C.c_uint64), ("xfer_count", C.c_uint64),
        ("link_bytes", (C.c_uint64 * MAX_GPUS) * 3), ("kernel_launches", C.c_uint64),
        ("rounds", C.c_uint64), ("timed_launches", C.c_uint64), ("timed_ns", C.c_uint64),
        ("timed_bytes", C.c_uint64), ("restore_count", C.c_uint64), ("restore_bytes", C.c_uint64),
        ("pool_target", C.c_uint64 * MAX_GPUS), ("tracked_functions", C.c_uint64),
        ("tracked_tenants", C.c_uint64), ("peer_launches", C.c_uint64),
        ("timed_kernel_launches", C.c_uint64), ("timed_kernel_ns", C.c_uint64),
        ("auto_avail", C.c_uint64 * MAX_GPUS), ("auto_refreshes", C.c_uint64),
        ("auto_mode", C.c_uint32), ("pad_", C.c_uint32),
    ]


MAX_PATH_NODES = 8


class grouter_path(C.Structure):
    _fields_ = [("bw_Bps", C.c_uint64), ("func", C.c_uint32), ("n_nodes", C.c_uint32),
                ("nodes", C.c_int32 * MAX_PATH_NODES)]


IPC_MAX_SEGS = 8


class grouter_ipc_desc(C.Structure):
    _fields_ = [("magic", C.c_uint32), ("version", C.c_uint32), ("pid", C.c_int32),
                ("ctx_id", C.c_uint32), ("gpu_uuid", C.c_uint8 * 16), ("workflow_id", C.c_uint32),
                ("logical", C.c_int32), ("oid", C.c_uint64), ("n", C.c_uint64),
                ("exporter_ptr", C.c_uint64), ("export_id", C.c_uint64), ("nonce", C.c_uint64 * 2),
                ("alloc_bytes", C.c_uint64)]


class grouter_dispatch(C.Structure):
    _fields_ = [("server_kind", C.c_int32), ("server_dev", C.c_int32), ("tenant", C.c_uint32),
                ("n_chunks", C.c_uint32), ("chunk_ids", C.c_uint64 * 8), ("bytes", C.c_uint64),
                ("inflight", C.c_uint32), ("pad", C.c_uint32)]


_P = C.c_void_p
_U64, _U32, _I32 = C.c_uint64, C.c_uint32, C.c_int32
_ST = C.c_int
_CTX = C.c_void_p

# name -> (restype, argtypes); every symbol declared in include/*.h.  The
# data-path calls take their grouter_fn* and out-pointers as plain addresses
# (c_void_p): a typed POINTER argument costs ~0.2 us of ctypes conversion per
# argument per call, which single small transfers (a few us) would feel.
SIGNATURES = {
    "grouter_config_default": (None, [C.POINTER(grouter_config)]),
    "grouter_probe": (_ST, [C.POINTER(grouter_config), _U64]),
    "grouter_init": (_ST, [C.POINTER(grouter_config), C.POINTER(_CTX)]),
    "grouter_finalize": (_ST, [_CTX]),
    "grouter_put": (_ST, [_CTX, _P, _P, _U64, _I32, _U32, _P, _P]),
    "grouter_alloc": (_ST, [_CTX, _P, _U64, _I32, _U32, _P, _P]),
    "grouter_seal": (_ST, [_CTX, _P, _U64, _P]),
    "grouter_get": (_ST, [_CTX, _P, _U64, _P, _P, _P]),
    "grouter_get_into": (_ST, [_CTX, _P, _U64, _P, _U64, _P, _P]),
    "grouter_release": (_ST, [_CTX, _P, _U64, _P, _P]),
    "grouter_free": (_ST, [_CTX, _P, _U64]),
    "grouter_set_tenant_weight": (_ST, [_CTX, _U32, _U32]),
    "grouter_set_next_use": (_ST, [_CTX, _U64, _U64]),
    "grouter_set_pool_limit": (_ST, [_CTX, _I32, _U64]),
    "grouter_refresh_cap": (_ST, [_CTX, _I32, _U64, C.POINTER(C.c_uint64)]),
    "grouter_flush": (_ST, [_CTX]),
    "grouter_sync": (_ST, [_CTX]),
    "grouter_plan": (_ST, [_CTX, _I32, _I32, _U64, C.POINTER(grouter_chunk), _U64, C.POINTER(_U64)]),
    "grouter_route_set": (_ST, [_CTX, _I32, C.POINTER(_I32), _U32, C.POINTER(_U32)]),
    "grouter_where": (_ST, [_CTX, _U64, C.POINTER(_I32)]),
    "grouter_stats": (_ST, [_CTX, C.POINTER(grouter_stats_t)]),
    "grouter_tenant_stats": (_ST, [_CTX, C.c_uint32, C.POINTER(_U64)]),
    "grouter_tenant_rate": (_ST, [_CTX, C.c_uint32, _U64, C.POINTER(_U64), C.POINTER(_U64), C.POINTER(_I32)]),
    "grouter_victims": (_ST, [_CTX, C.POINTER(_U64), _U64, C.POINTER(_U64)]),
    "grouter_restored": (_ST, [_CTX, C.POINTER(_U64), _U64, C.POINTER(_U64)]),
    "grouter_paths_new": (C.c_void_p, [C.c_uint32, C.c_uint32, C.POINTER(_U64), C.c_uint32]),
    "grouter_paths_free": (None, [C.c_void_p]),
    "grouter_paths_select": (_ST, [C.c_void_p, C.c_uint32, C.c_int32, C.c_int32, C.POINTER(grouter_path),
                                   C.c_uint32, C.POINTER(C.c_uint32)]),
    "grouter_paths_release": (_ST, [C.c_void_p, C.c_uint32]),
    "grouter_paths_table": (_ST, [C.c_void_p, C.POINTER(grouter_path), C.c_uint32, C.POINTER(C.c_uint32)]),
    "grouter_paths_plan": (_ST, [C.c_void_p, C.c_uint32, _U64, _U64, _U64, _U64, C.POINTER(grouter_chunk),
                                 _U64, C.POINTER(_U64)]),
    "grouter_pool_target": (_ST, [_CTX, C.c_int32, C.POINTER(_U64)]),
    "grouter_test_set_clock": (_ST, [_CTX, C.c_int32, _U64]),
    "grouter_set_tenant_slo": (_ST, [_CTX, C.c_uint32, _U64, _U64, _U64]),
    "grouter_slo_weights": (_ST, [C.c_uint32, C.POINTER(C.c_uint32), C.POINTER(_U64), C.POINTER(_U64),
                                  C.POINTER(_U64), _U64, C.POINTER(C.c_uint32)]),
    "grouter_dispatch_log": (_ST, [_CTX, C.POINTER(grouter_dispatch), _U64, C.POINTER(_U64)]),
    "grouter_export_ipc": (_ST, [_CTX, C.POINTER(grouter_fn), _U64, C.POINTER(grouter_ipc_desc)]),
    "grouter_import_ipc": (_ST, [_CTX, C.POINTER(grouter_fn), C.POINTER(grouter_ipc_desc), _U32,
                                 C.POINTER(_U64)]),
    "grouter_sched_new": (_ST, [_U32, C.POINTER(_P)]),
    "grouter_sched_set_weight": (_ST, [_P, _U32, _U32]),
    "grouter_sched_enqueue": (_ST, [_P, _U32, _U64, _U64]),
    "grouter_sched_dispatch": (_ST, [_P, C.POINTER(_U32), C.POINTER(_U64), C.POINTER(_U32),
                                     C.POINTER(_U64), C.POINTER(_U64)]),
    "grouter_sched_account_solo": (_ST, [_P, C.c_uint32, C.c_uint64, C.c_uint64]),
    "grouter_sched_free": (None, [_P]),
    "grouter_strerror": (C.c_char_p, [_ST]),
    "grouter_last_error": (C.c_char_p, []),
    "grouter_build_hash": (C.c_char_p, []),
    "grouter_test_fill": (_ST, [_P, _U64, _U64, _U64, _P]),
    "grouter_test_verify": (_ST, [_P, _U64, _U64, _U64, _P, C.POINTER(_U64), C.POINTER(_U64)]),
    "grouter_test_launch_cost": (_ST, [C.c_int, C.c_int, C.c_int, _P, C.POINTER(C.c_double)]),
    "grouter_test_dump": (_ST, [_CTX, C.c_char_p, _U64, C.POINTER(_U64)]),
    "grouter_test_copy": (_ST, [_P, _P, C.POINTER(grouter_chunk), _U32, _P, C.c_int, _P]),
    "grouter_test_memcpy": (_ST, [_P, _P, C.c_uint64, _P, C.c_int32]),
    "grouter_test_race": (_ST, [C.c_int32, C.POINTER(C.c_int64)]),
    "grouter_test_oob": (_ST, [C.POINTER(C.c_int32)]),
    "grouter_test_inject": (_ST, [_CTX, C.c_int32, C.c_int32]),
}

_lib = None


def load(build_if_missing: bool = False):
    """Loads libgrouter.so (built in-tree).  Raises if missing: no fallback."""
    global _lib
    if _lib is not None:
        return _lib
    from . import _build
    # GROUTER_LIB selects a sanitizer build of the same sources (tsan / asan,
    # _build.SANITIZERS); the default is the product library
    variant = os.environ.get("GROUTER_LIB") or None
    if variant and variant not in _build.SANITIZERS:
        raise ImportError(f"GROUTER_LIB={variant!r}: expected one of {sorted(_build.SANITIZERS)}")
    path = _build.lib_path(variant)
    if not os.path.exists(path):
        if not build_if_missing:
            raise ImportError(f"{path} not built; run __graft_entry__.build()")
        _build.build(variant=variant)
    want = _build.source_hash()
    if _build.built_hash(path) != want:
        if not build_if_missing:
            raise ImportError(f"{path} was built from other sources (hash {_build.built_hash(path)} != "
                              f"{want}); run __graft_entry__.build()")
        _build.build(variant=variant)
    lib = C.CDLL(path)
    for name, (res, args) in SIGNATURES.items():
        f = getattr(lib, name)
        f.restype = res
        f.argtypes = args
    got = lib.grouter_build_hash().decode()
    if got != want:   # the file changed between the scan and dlopen
        raise ImportError(f"{path}: grouter_build_hash() {got} != source hash {want}")
    _lib = lib
    return lib


def last_error() -> str:
    s = load().grouter_last_error()
    return s.decode() if s else ""


class GrouterError(RuntimeError):
    def __init__(self, st, what=""):
        super().__init__(f"{STATUS[st] if 0 <= st < 8 else st}: {what} ({last_error()})")
        self.status = st


def check(st, what=""):
    if st != OK:
        raise GrouterError(st, what)
    return st


# ------------------------------------------------------------------ config
def config_from_calib(calib: dict | None = None, **kw) -> grouter_config:
    """grouter_config from a calibration dict (synth/calib.py format) plus
    overrides (chunk_bytes, host_store_bytes, pool_cap=[...], flags, ...)."""
    lib = load()
    cfg = grouter_config()
    lib.grouter_config_default(C.byref(cfg))
    if calib is not None:
        n = calib["n_gpus"]
        cfg.n_gpus = n
        dm = calib.get("device_map", list(range(n)))
        for i in range(n):
            cfg.device_map[i] = dm[i]
            cfg.h2d_Bps[i] = calib["h2d_Bps"][i]
            cfg.h2d_alpha_ps[i] = calib["h2d_alpha_ps"][i]
            cfg.h2d_phi_ps[i] = calib["h2d_phi_ps"][i]
            for j in range(n):
                cfg.p2p[i][j] = calib["p2p"][i][j]
        cfg.nvl_Bps = calib["nvl_Bps"]
        cfg.relay_phi_ps = calib["relay_phi_ps"]
        if "uplink_groups" in calib:
            for gi, g in enumerate(calib["uplink_groups"]):
                for x in g:
                    cfg.uplink_group[x] = gi
        else:
            for i in range(MAX_GPUS):
                cfg.uplink_group[i] = -1
            for i in range(n):
                for j in range(n):
                    cfg.h2d_pair_Bps[i][j] = calib["h2d_pair_Bps"][i][j]
    caps = kw.pop("pool_cap", None)
    if caps is not None:
        for i, v in enumerate(caps):
            cfg.pool_cap_bytes[i] = v
    for k, v in kw.items():
        setattr(cfg, k, v)
    return cfg


def probe(devices, probe_bytes: int = 256 << 20) -> dict:
    """Runs grouter_probe on CUDA ordinals `devices`; returns a calibration
    dict in synth/calib.py format (device_map = devices)."""
    lib = load()
    cfg = grouter_config()
    lib.grouter_config_default(C.byref(cfg))
    cfg.n_gpus = len(devices)
    for i, d in enumerate(devices):
        cfg.device_map[i] = d
    check(lib.grouter_probe(C.byref(cfg), probe_bytes), "grouter_probe")
    n = len(devices)
    return {"name": "probed", "n_gpus": n, "device_map": list(devices), "nvl_Bps": cfg.nvl_Bps,
            "h2d_Bps": [cfg.h2d_Bps[i] for i in range(n)],
            "h2d_alpha_ps": [cfg.h2d_alpha_ps[i] for i in range(n)],
            "h2d_phi_ps": [cfg.h2d_phi_ps[i] for i in range(n)],
            "relay_phi_ps": cfg.relay_phi_ps,
            "h2d_pair_Bps": [[cfg.h2d_pair_Bps[i][j] for j in range(n)] for i in range(n)],
            "p2p": [[cfg.p2p[i][j] for j in range(n)] for i in range(n)]}


def fn(wf: int, fid: int, dev: int) -> grouter_fn:
    return grouter_fn(wf, fid, dev)


def _fa(f: grouter_fn) -> int:
    """Address of a grouter_fn (cached on the object: it never moves)."""
    try:
        return f._a
    except AttributeError:
        if not isinstance(f, grouter_fn):
            raise TypeError("expected a grouter_fn") from None
        f._a = C.addressof(f)
        return f._a


_tls = threading.local()


def _out():
    """This thread's out-parameter slots (4 x u64) and their address; the
    library writes them only on success, so they are zeroed per call."""
    try:
        b, a = _tls.b, _tls.a
    except AttributeError:
        b = _tls.b = (C.c_uint64 * 4)()
        a = _tls.a = C.addressof(b)
    b[0] = b[1] = 0
    return b, a


class Ctx:
    """Owns a grouter_ctx; methods mirror the C calls and return statuses."""

    def __init__(self, cfg: grouter_config):
        self.lib = load()
        h = C.c_void_p()
        check(self.lib.grouter_init(C.byref(cfg), C.byref(h)), "grouter_init")
        self.h = h

    def close(self):
        if self.h:
            self.lib.grouter_finalize(self.h)
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # data path (per-thread out-parameter slots: one context serves several client threads)
    def put(self, f, src: int, n: int, hint=NOHINT, consumers=0, stream=0):
        b, a = _out()
        st = self.lib.grouter_put(self.h, _fa(f), src, n, hint, consumers, stream, a)
        return st, b[0]

    def alloc(self, f, n: int, hint=NOHINT, consumers=0):
        b, a = _out()
        st = self.lib.grouter_alloc(self.h, _fa(f), n, hint, consumers, a, a + 8)
        return st, b[0], b[1]

    def seal(self, f, oid: int, stream=0):
        return self.lib.grouter_seal(self.h, _fa(f), oid, stream)

    def get(self, f, oid: int, stream=0):
        b, a = _out()
        st = self.lib.grouter_get(self.h, _fa(f), oid, stream, a, a + 8)
        return st, b[0], b[1]

    def get_into(self, f, oid: int, dst: int, cap: int, stream=0):
        b, a = _out()
        st = self.lib.grouter_get_into(self.h, _fa(f), oid, dst, cap, stream, a)
        return st, b[0]

    def release(self, f, oid: int, ptr: int, stream=0):
        return self.lib.grouter_release(self.h, _fa(f), oid, ptr, stream)

    def free(self, f, oid: int):
        return self.lib.grouter_free(self.h, _fa(f), oid)

    # cross-process handoff
    def export_ipc(self, f, oid):
        d = grouter_ipc_desc()
        st = self.lib.grouter_export_ipc(self.h, C.byref(f), oid, C.byref(d))
        return st, bytes(d)

    def import_ipc(self, f, desc: bytes, consumers=0):
        d = grouter_ipc_desc.from_buffer_copy(desc)
        oid = C.c_uint64(0)
        st = self.lib.grouter_import_ipc(self.h, C.byref(f), C.byref(d), consumers, C.byref(oid))
        return st, oid.value

    @staticmethod
    def desc_exporter_ptr(desc: bytes) -> int:
        return grouter_ipc_desc.from_buffer_copy(desc).exporter_ptr

    # control
    def set_tenant_weight(self, wf, w):
        return self.lib.grouter_set_tenant_weight(self.h, wf, w)

    def pool_target(self, dev):
        v = C.c_uint64(0)
        check(self.lib.grouter_pool_target(self.h, dev, C.byref(v)), "pool_target")
        return v.value

    def inject_round_failures(self, count):
        """Fault injection (tests only): the next `count` dispatch rounds fail."""
        return self.lib.grouter_test_inject(self.h, 1, count)

    def set_clock(self, t_ns=None):
        """Fix the pool-sizing clock to t_ns (None: back to the monotonic clock)."""
        return self.lib.grouter_test_set_clock(self.h, 0 if t_ns is None else 1, t_ns or 0)

    def set_tenant_slo(self, wf, data_bytes, slo_ns, infer_ns):
        return self.lib.grouter_set_tenant_slo(self.h, wf, data_bytes, slo_ns, infer_ns)

    def set_next_use(self, oid, pos):
        return self.lib.grouter_set_next_use(self.h, oid, pos)

    def set_pool_limit(self, dev, nbytes):
        return self.lib.grouter_set_pool_limit(self.h, dev, nbytes)

    def refresh_cap(self, dev, avail=AUTO_AVAIL):
        """O10 auto cap: (status, cap applied)."""
        cap = C.c_uint64(0)
        st = self.lib.grouter_refresh_cap(self.h, dev, avail, C.byref(cap))
        return st, cap.value

    def flush(self):
        return self.lib.grouter_flush(self.h)

    def sync(self):
        return self.lib.grouter_sync(self.h)

    # introspection
    def plan(self, src, dst, n):
        cnt = C.c_uint64(0)
        st = self.lib.grouter_plan(self.h, src, dst, n, None, 0, C.byref(cnt))
        if st not in (OK, EINVAL) or (st == EINVAL and cnt.value == 0):
            return st, []
        arr = (grouter_chunk * max(cnt.value, 1))()
        st = self.lib.grouter_plan(self.h, src, dst, n, arr, cnt.value, C.byref(cnt))
        return st, [(c.offset, c.bytes, c.path, c.route_gpu) for c in arr[:cnt.value]]

    def route_set(self, d):
        arr, cnt = (C.c_int32 * MAX_GPUS)(), C.c_uint32(0)
        st = self.lib.grouter_route_set(self.h, d, arr, MAX_GPUS, C.byref(cnt))
        return st, list(arr[:cnt.value])

    def where(self, oid):
        loc = C.c_int32(0)
        st = self.lib.grouter_where(self.h, oid, C.byref(loc))
        return st, loc.value

    def tenant_stats(self, workflow_id: int):
        """Bytes of this tenant's chunks dispatched per server kind [SM copy, H2D, D2H]."""
        arr = (_U64 * 3)()
        check(self.lib.grouter_tenant_stats(self.h, workflow_id, arr), "tenant_stats")
        return list(arr)

    def tenant_rate(self, workflow_id: int, window_ns: int):
        """(dispatched B/s over the window, Rate_least B/s (0 without SLO), backlogged)."""
        r, least, bl = _U64(0), _U64(0), _I32(0)
        check(self.lib.grouter_tenant_rate(self.h, workflow_id, window_ns, C.byref(r), C.byref(least),
                                           C.byref(bl)), "tenant_rate")
        return r.value, least.value, bool(bl.value)

    def stats(self) -> grouter_stats_t:
        s = grouter_stats_t()
        check(self.lib.grouter_stats(self.h, C.byref(s)), "stats")
        return s

    def dump(self) -> str:
        n = C.c_uint64(0)
        self.lib.grouter_test_dump(self.h, None, 0, C.byref(n))
        buf = C.create_string_buffer(n.value + 1)
        self.lib.grouter_test_dump(self.h, buf, n.value + 1, C.byref(n))
        return buf.value.decode()

    def victims(self):
        arr, cnt = (C.c_uint64 * 4096)(), C.c_uint64(0)
        check(self.lib.grouter_victims(self.h, arr, 4096, C.byref(cnt)), "victims")
        return list(arr[:cnt.value])

    def restored(self):
        arr, cnt = (C.c_uint64 * 4096)(), C.c_uint64(0)
        check(self.lib.grouter_restored(self.h, arr, 4096, C.byref(cnt)), "restored")
        return list(arr[:cnt.value])

    def dispatch_log(self):
        out = []
        arr, cnt = (grouter_dispatch * 4096)(), C.c_uint64(0)
        while True:
            check(self.lib.grouter_dispatch_log(self.h, arr, 4096, C.byref(cnt)), "dispatch_log")
            for d in arr[:cnt.value]:
                out.append({"kind": d.server_kind, "dev": d.server_dev, "tenant": d.tenant,
                            "chunks": [(x >> 32, x & 0xFFFFFFFF) for x in d.chunk_ids[:d.n_chunks]],
                            "bytes": d.bytes, "inflight": d.inflight})
            if cnt.value < 4096:
                return out


# ------------------------------------------------------------------ test kernels (K9)
class Paths:
    """grouter_paths_*: the Alg. 1 NVLink path planner (host only)."""

    def __init__(self, topo, n_gpus, max_edges=3):
        self.lib = load()
        n = len(topo)
        flat = (C.c_uint64 * (n * n))(*[topo[u][v] for u in range(n) for v in range(n)])
        self.h = self.lib.grouter_paths_new(n, n_gpus, flat, max_edges)
        if not self.h:
            raise GrouterError(EINVAL, "grouter_paths_new")

    @staticmethod
    def _conv(p):
        return (p.func, p.bw_Bps, tuple(p.nodes[:p.n_nodes]))

    def select(self, func, gs, gd):
        arr, cnt = (grouter_path * 64)(), C.c_uint32(0)
        st = self.lib.grouter_paths_select(self.h, func, gs, gd, arr, 64, C.byref(cnt))
        return st, [(list(x[2]), x[1]) for x in map(self._conv, arr[:cnt.value])]

    def release(self, func):
        return self.lib.grouter_paths_release(self.h, func)

    def table(self):
        arr, cnt = (grouter_path * 1024)(), C.c_uint32(0)
        check(self.lib.grouter_paths_table(self.h, arr, 1024, C.byref(cnt)), "paths_table")
        return [self._conv(p) for p in arr[:cnt.value]]

    def plan(self, func, n, chunk_bytes, relay_phi_ps, granule=4096):
        cnt = C.c_uint64(0)
        self.lib.grouter_paths_plan(self.h, func, n, chunk_bytes, granule, relay_phi_ps, None, 0, C.byref(cnt))
        arr = (grouter_chunk * max(cnt.value, 1))()
        check(self.lib.grouter_paths_plan(self.h, func, n, chunk_bytes, granule, relay_phi_ps, arr, cnt.value,
                                          C.byref(cnt)), "paths_plan")
        return [(c.offset, c.bytes, c.path, c.route_gpu) for c in arr[:cnt.value]]

    def close(self):
        if self.h:
            self.lib.grouter_paths_free(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def slo_weights(slos: dict, bw_all: int) -> dict:
    """grouter_slo_weights: {wf: (data_bytes, slo_ns, infer_ns)} -> {wf: weight}."""
    lib = load()
    n = len(slos)
    ids = (C.c_uint32 * max(n, 1))(*slos.keys())
    d = (C.c_uint64 * max(n, 1))(*[v[0] for v in slos.values()])
    s = (C.c_uint64 * max(n, 1))(*[v[1] for v in slos.values()])
    i = (C.c_uint64 * max(n, 1))(*[v[2] for v in slos.values()])
    out = (C.c_uint32 * max(n, 1))()
    check(lib.grouter_slo_weights(n, ids, d, s, i, bw_all, out), "slo_weights")
    return dict(zip(slos.keys(), out[:n]))


def test_fill(ptr: int, n: int, seed: int, offset: int = 0, stream: int = 0):
    return load().grouter_test_fill(ptr or None, n, seed, offset, stream or None)


def test_verify(ptr: int, n: int, seed: int, offset: int = 0, stream: int = 0):
    mism, first = C.c_uint64(0), C.c_uint64(0)
    st = load().grouter_test_verify(ptr or None, n, seed, offset, stream or None, C.byref(mism),
                                    C.byref(first))
    return st, mism.value, first.value


def test_memcpy(dst: int, src: int, n: int, stream: int = 0, wait: bool = True):
    """Measured baseline: one bare cudaMemcpyAsync (+ wait for completion)."""
    return load().grouter_test_memcpy(dst or None, src or None, n, stream or None, 1 if wait else 0)


def test_copy(dst: int, src: int, chunks, counts: int = 0, tma: bool = False, stream: int = 0):
    arr = (grouter_chunk * max(len(chunks), 1))(*[grouter_chunk(o, b, p, r) for o, b, p, r in chunks])
    return load().grouter_test_copy(dst or None, src or None, arr, len(chunks), counts or None,
                                    int(tma), stream or None)


class Sched:
    """The library's stride scheduler (standalone; no GPU needed)."""

    def __init__(self, batch=5):
        self.lib = load()
        self.h = C.c_void_p()
        check(self.lib.grouter_sched_new(batch, C.byref(self.h)), "sched_new")

    def set_weight(self, t, w):
        return self.lib.grouter_sched_set_weight(self.h, t, w)

    def enqueue(self, t, cid, nbytes):
        return self.lib.grouter_sched_enqueue(self.h, t, cid, nbytes)

    def account_solo(self, t, n, chunk):
        return self.lib.grouter_sched_account_solo(self.h, t, n, chunk)

    def dispatch(self):
        t, n, b, p = C.c_uint32(0), C.c_uint32(0), C.c_uint64(0), C.c_uint64(0)
        ids = (C.c_uint64 * 8)()
        st = self.lib.grouter_sched_dispatch(self.h, C.byref(t), ids, C.byref(n), C.byref(b), C.byref(p))
        if st != OK:
            return None
        return t.value, list(ids[:n.value]), b.value, p.value

    def __del__(self):
        try:
            self.lib.grouter_sched_free(self.h)
        except Exception:
            pass
