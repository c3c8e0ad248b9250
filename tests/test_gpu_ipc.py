"""Cross-process zero-copy handoff (PAPER.md L167 (1), L269: pool pages mapped
into the consuming function's address space via CUDA IPC; L394: workflow
authentication, pre-mapped storage only).  On one B200: (a) two contexts of
one process, (b) two processes.  Zero copy is proven by aliasing: a canary
written through the exporter's pointer after the import is read through the
importer's mapping, and the reverse -- a copy would fail both.  get_into
copies with the SM kernel; other workflows get EPERM; a wrong nonce or a
freed export is refused; an importer's mapping keeps the object's pages
(never reused by the exporter's pool) after the exporter frees it."""
import os
import subprocess
import sys
import textwrap

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

from paper_conf_eurosys_wulywdyfwwj26_b200 import _build          # noqa: E402
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G    # noqa: E402
from synth.calib import b200_hgx                                   # noqa: E402
from synth.payload import payload                                  # noqa: E402
from tests.lib_runner import DevView, read_device                  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _poke(ptr, n, value):
    """Writes `value` into n bytes at a raw device address (through a torch
    alias of the address, no copy)."""
    t = torch.as_tensor(DevView(ptr, n), device="cuda")
    t.fill_(value)
    torch.cuda.synchronize()


def _ctx():
    c = b200_hgx(1)
    c["device_map"] = [0]
    return G.Ctx(G.config_from_calib(c, host_store_bytes=64 << 20, pool_cap=[G.UNLIMITED],
                                     pool_floor_bytes=64 << 20))


@pytest.fixture(scope="module", autouse=True)
def lib():
    _build.build()
    G.load()


@pytest.mark.parametrize("n", [1, 4096, 3 * (1 << 20) + 7, 38_535_168])
def test_two_contexts_one_process(n):
    a, b = _ctx(), _ctx()
    try:
        s = torch.cuda.Stream()
        src = torch.empty(n, dtype=torch.uint8, device="cuda")
        G.check(G.test_fill(src.data_ptr(), n, 321, 0, s.cuda_stream))
        producer = G.fn(7, 1, 0)
        st, oid = a.put(producer, src.data_ptr(), n, G.NOHINT, 0, s.cuda_stream)
        assert st == G.OK
        st, desc = a.export_ipc(producer, oid)
        assert st == G.OK
        # another workflow may not import it (L394)
        assert b.import_ipc(G.fn(8, 1, 0), desc)[0] == G.EPERM
        consumer = G.fn(7, 2, 0)
        st, roid = b.import_ipc(consumer, desc)
        assert st == G.OK and b.where(roid) == (G.OK, G.REMOTE)
        # zero copy: same GPU -> the import aliases the exporter's pages
        st, ptr, nn = b.get(consumer, roid, s.cuda_stream)
        assert st == G.OK and nn == n
        s.synchronize()
        assert np.array_equal(read_device(ptr, min(n, 1 << 20), 0), payload(321, min(n, 1 << 20)))
        exp_ptr = G.Ctx.desc_exporter_ptr(desc)
        assert ptr != exp_ptr                        # a different mapping of the same pages
        # the import is exactly the object's own 2 MiB pages (R52), no neighbour's
        dd = G.grouter_ipc_desc.from_buffer_copy(desc)
        assert dd.alloc_bytes == -(-n // (2 << 20)) * (2 << 20) and dd.version == 2
        # aliasing, both ways: a copy would see neither write
        k = min(n, 4096)
        _poke(exp_ptr, k, 0x3C)
        assert (read_device(ptr, k, 0) == 0x3C).all()
        _poke(ptr, k, 0xC3)
        assert (read_device(exp_ptr, k, 0) == 0xC3).all()
        G.check(G.test_fill(exp_ptr, k, 321, 0, 0))   # put the payload back
        torch.cuda.synchronize()
        # get_into: the SM copy kernel reads the imported mapping
        dst = torch.full((n + 32,), 0xA5, dtype=torch.uint8, device="cuda")
        torch.cuda.synchronize()
        st, nn = b.get_into(consumer, roid, dst.data_ptr() + 16, n, s.cuda_stream)
        assert st == G.OK
        s.synchronize()
        st2, bad, _ = G.test_verify(dst.data_ptr() + 16, n, 321, 0, 0)
        assert st2 == G.OK and bad == 0
        d = dst.cpu().numpy()
        assert (d[:16] == 0xA5).all() and (d[16 + n:] == 0xA5).all()
        assert b.release(consumer, roid, ptr, s.cuda_stream) == G.OK
        assert b.free(consumer, roid) == G.OK
        assert a.release(producer, oid, exp_ptr, 0) == G.OK
        assert a.free(producer, oid) == G.OK
        a.sync()
        assert a.stats().used[0] == 0 and b.stats().used[0] == 0
    finally:
        b.close()
        a.close()


EXPORTER = textwrap.dedent("""
    import sys, os
    sys.path.insert(0, {root!r})
    import torch
    from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G
    from synth.calib import b200_hgx
    from tests.lib_runner import DevView
    c = b200_hgx(1); c["device_map"] = [0]
    ctx = G.Ctx(G.config_from_calib(c, host_store_bytes=64 << 20, pool_cap=[G.UNLIMITED],
                                    pool_floor_bytes=64 << 20))
    n = {n}
    src = torch.empty(n, dtype=torch.uint8, device="cuda")
    G.check(G.test_fill(src.data_ptr(), n, 99, 0, 0))
    torch.cuda.synchronize()
    f = G.fn(5, 1, 0)
    st, oid = ctx.put(f, src.data_ptr(), n, G.NOHINT, 0, 0)
    st, desc = ctx.export_ipc(f, oid)
    ptr = G.Ctx.desc_exporter_ptr(desc)
    print(desc.hex(), flush=True)
    keep = []
    for line in sys.stdin:
        cmd = line.split()
        if cmd[0] == "poke":            # write through the exporter's own pointer
            torch.as_tensor(DevView(ptr, 4096), device="cuda").fill_(int(cmd[1]))
            torch.cuda.synchronize()
            print("ok", flush=True)
        elif cmd[0] == "peek":          # read through the exporter's own pointer
            print(int(torch.as_tensor(DevView(ptr, 4096), device="cuda")[:4096].min().item()),
                  int(torch.as_tensor(DevView(ptr, 4096), device="cuda")[:4096].max().item()), flush=True)
        elif cmd[0] == "free":          # end the export, then churn the pool with other data
            r = (ctx.release(f, oid, ptr, 0), ctx.free(f, oid))
            ctx.sync()
            for i in range(8):
                st, o2 = ctx.put(f, src.data_ptr(), n, G.NOHINT, 0, 0)
                keep.append(o2)
            junk = torch.full((n,), 0xEE, dtype=torch.uint8, device="cuda")
            for o2 in keep:
                ctx.get_into(f, o2, junk.data_ptr(), n, 0)
            ctx.sync()
            print(*r, flush=True)
        elif cmd[0] == "done":
            for o2 in keep:
                ctx.free(f, o2)
            ctx.sync()
            print(ctx.stats().used[0], flush=True)
            break
    ctx.close()
""")


def test_two_processes():
    """Two processes: the importer's mapping aliases the exporter's pages
    (canaries both ways), a forged nonce and a freed export are refused, and
    the importer's view survives the exporter freeing the object and reusing
    its pool (the pages are the object's own allocation, never recycled)."""
    n = 5 * (1 << 20) + 3
    p = subprocess.Popen([sys.executable, "-c", EXPORTER.format(root=ROOT, n=n)], stdin=subprocess.PIPE,
                         stdout=subprocess.PIPE, text=True)

    def cmd(c):
        p.stdin.write(c + "\n")
        p.stdin.flush()
        return p.stdout.readline().split()
    try:
        desc = bytes.fromhex(p.stdout.readline().strip())
        b = _ctx()
        try:
            f = G.fn(5, 2, 0)
            # a forged capability (wrong nonce) is refused by the exporter
            forged = G.grouter_ipc_desc.from_buffer_copy(desc)
            forged.nonce[1] ^= 1
            assert b.import_ipc(f, bytes(forged))[0] == G.ENOENT
            st, roid = b.import_ipc(f, desc, consumers=0)
            assert st == G.OK
            dst = torch.empty(n, dtype=torch.uint8, device="cuda")
            s = torch.cuda.Stream()
            st, nn = b.get_into(f, roid, dst.data_ptr(), n, s.cuda_stream)   # SM copy from the mapping
            assert st == G.OK and nn == n
            s.synchronize()
            st2, bad, _ = G.test_verify(dst.data_ptr(), n, 99, 0, 0)
            assert st2 == G.OK and bad == 0
            st, ptr, nn = b.get(f, roid, s.cuda_stream)                      # zero copy: the mapping
            assert st == G.OK
            s.synchronize()
            assert cmd("poke 90") == ["ok"]                                  # exporter writes ...
            assert (read_device(ptr, 4096, 0) == 90).all()                   # ... importer sees it
            _poke(ptr, 4096, 165)                                            # importer writes ...
            assert cmd("peek") == ["165", "165"]                             # ... exporter sees it
            assert cmd("free") == ["0", "0"]           # exporter frees the object and churns its pool
            # the importer's mapping still holds the object's pages, untouched by the churn
            assert (read_device(ptr, 4096, 0) == 165).all()
            assert np.array_equal(read_device(ptr + 4096, n - 4096, 0), payload(99, n - 4096, 4096))
            # the export is over: a new import of the same descriptor is refused
            assert b.import_ipc(f, desc)[0] == G.ENOENT
            assert b.release(f, roid, ptr, s.cuda_stream) == G.OK
            assert b.free(f, roid) == G.OK
            assert b.where(roid)[0] == G.ENOENT
        finally:
            b.close()
        assert cmd("done") == ["0"]
    finally:
        p.wait(timeout=60)


def test_export_free_trim_reexport():
    """ADVICE r01 (stale descriptors): export A, import it, free A, let the
    pool trim, put and export B, import B.  B's import reads B's bytes, A's
    old descriptor is refused, and the mapping of A taken before the free
    still reads A's bytes (its pages were A's own allocation, never
    recycled by the pool)."""
    import time
    a, b = _ctx(), _ctx()
    try:
        n = 6 * (1 << 20) + 11
        src = torch.empty(n, dtype=torch.uint8, device="cuda")
        f, g = G.fn(4, 1, 0), G.fn(4, 2, 0)
        G.check(G.test_fill(src.data_ptr(), n, 61, 0, 0))
        torch.cuda.synchronize()
        st, oa = a.put(f, src.data_ptr(), n, G.NOHINT, 0, 0)
        st, da = a.export_ipc(f, oa)
        assert st == G.OK
        st, ra = b.import_ipc(g, da)
        assert st == G.OK
        st, pa, _ = b.get(g, ra, 0)
        assert st == G.OK
        assert a.release(f, oa, G.Ctx.desc_exporter_ptr(da), 0) == G.OK and a.free(f, oa) == G.OK
        a.sync()
        time.sleep(1.3)                                    # the daemon trims excess pool segments after 1 s
        G.check(G.test_fill(src.data_ptr(), n, 62, 0, 0))
        torch.cuda.synchronize()
        st, ob = a.put(f, src.data_ptr(), n, G.NOHINT, 0, 0)
        st, db = a.export_ipc(f, ob)
        assert st == G.OK
        assert b.import_ipc(g, da)[0] == G.ENOENT           # A's export ended with A
        st, rb = b.import_ipc(g, db)
        assert st == G.OK
        dst = torch.empty(n, dtype=torch.uint8, device="cuda")
        st, nn = b.get_into(g, rb, dst.data_ptr(), n, 0)
        assert st == G.OK
        assert G.test_verify(dst.data_ptr(), n, 62, 0, 0)[1] == 0      # B's bytes
        assert np.array_equal(read_device(pa, n, 0), payload(61, n))   # A's pages, still A's bytes
        assert b.release(g, ra, pa, 0) == G.OK
        for roid in (ra, rb):
            assert b.free(g, roid) == G.OK
        assert a.release(f, ob, G.Ctx.desc_exporter_ptr(db), 0) == G.OK and a.free(f, ob) == G.OK
    finally:
        b.close()
        a.close()


def test_export_requires_no_zero_copy_leases():
    """The first export moves the object into its own allocation; an object a
    zero-copy lease still aliases cannot move (EBUSY), once the lease is
    released the export succeeds, and a second export reuses the allocation
    (same exporter pointer, no second move)."""
    a = _ctx()
    try:
        n = 3 << 20
        src = torch.empty(n, dtype=torch.uint8, device="cuda")
        G.check(G.test_fill(src.data_ptr(), n, 5, 0, 0))
        torch.cuda.synchronize()
        f = G.fn(3, 1, 0)
        st, oid = a.put(f, src.data_ptr(), n, G.NOHINT, 0, 0)
        st, lp, nn = a.get(f, oid, 0)
        assert st == G.OK
        assert a.export_ipc(f, oid)[0] == G.EBUSY
        assert a.release(f, oid, lp, 0) == G.OK
        st, d1 = a.export_ipc(f, oid)
        assert st == G.OK
        st, d2 = a.export_ipc(f, oid)
        assert st == G.OK and G.Ctx.desc_exporter_ptr(d1) == G.Ctx.desc_exporter_ptr(d2)
        e = G.Ctx.desc_exporter_ptr(d1)
        assert np.array_equal(read_device(e, n, 0), payload(5, n))   # the move kept the bytes
        for _ in range(2):
            assert a.release(f, oid, e, 0) == G.OK
        assert a.free(f, oid) == G.OK
        a.sync()
        assert a.stats().used[0] == 0
    finally:
        a.close()


def test_stalled_peer_does_not_block_imports_or_close():
    """A same-uid peer that connects to the exporter's socket and never sends
    its request holds the serving thread for at most its 1 s I/O timeout:
    a real import behind it still succeeds, and close() does not hang."""
    import socket
    import time
    a, b = _ctx(), _ctx()
    stalled = []
    try:
        n = 1 << 20
        src = torch.empty(n, dtype=torch.uint8, device="cuda")
        G.check(G.test_fill(src.data_ptr(), n, 77, 0, 0))
        torch.cuda.synchronize()
        producer, consumer = G.fn(8, 1, 0), G.fn(8, 2, 0)
        st, oid = a.put(producer, src.data_ptr(), n, G.NOHINT, 0, 0)
        G.check(st, "put")
        st, desc = a.export_ipc(producer, oid)
        G.check(st, "export")
        d = G.grouter_ipc_desc.from_buffer_copy(desc)
        for _ in range(3):   # connect, send nothing
            s = socket.socket(socket.AF_UNIX, socket.SOCK_STREAM)
            s.connect(b"\0" + f"grouter.{d.pid}.{d.ctx_id}".encode())
            stalled.append(s)
        t0 = time.time()
        st, rid = b.import_ipc(consumer, desc)
        assert st == G.OK, G.last_error()
        assert time.time() - t0 < 8.0
        dst = torch.empty(n, dtype=torch.uint8, device="cuda")
        G.check(b.get_into(consumer, rid, dst.data_ptr(), n, 0)[0], "get_into")
        torch.cuda.synchronize()
        st2, bad, _ = G.test_verify(dst.data_ptr(), n, 77, 0, 0)
        assert st2 == G.OK and bad == 0
        assert b.free(consumer, rid) == G.OK
        assert a.release(producer, oid, G.Ctx.desc_exporter_ptr(desc), 0) == G.OK
        assert a.free(producer, oid) == G.OK
    finally:
        if stalled:   # one more stalled peer at close
            s = socket.socket(socket.AF_UNIX, socket.SOCK_STREAM)
            s.connect(stalled[0].getpeername())
            stalled.append(s)
        t0 = time.time()
        b.close()
        a.close()
        assert time.time() - t0 < 8.0
        for s in stalled:
            s.close()
