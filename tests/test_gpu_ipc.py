"""Cross-process zero-copy handoff (PAPER.md L167 (1), L269: pool pages mapped
into the consuming function's address space via CUDA IPC; L394: workflow
authentication).  On one B200: (a) two contexts of one process, (b) two
processes.  Importers see the exporter's bytes without a copy (zero copy on
the same GPU: a write through the exporter is visible through the import),
get_into copies them with the SM kernel, other workflows get EPERM."""
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
from tests.lib_runner import read_device                           # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


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
    print(desc.hex(), flush=True)
    sys.stdin.readline()                      # importer done
    print(ctx.release(f, oid, G.Ctx.desc_exporter_ptr(desc), 0), ctx.free(f, oid), flush=True)
    ctx.sync()
    print(ctx.stats().used[0], flush=True)
    ctx.close()
""")


def test_two_processes():
    n = 5 * (1 << 20) + 3
    p = subprocess.Popen([sys.executable, "-c", EXPORTER.format(root=ROOT, n=n)], stdin=subprocess.PIPE,
                         stdout=subprocess.PIPE, text=True)
    try:
        desc = bytes.fromhex(p.stdout.readline().strip())
        b = _ctx()
        try:
            f = G.fn(5, 2, 0)
            st, roid = b.import_ipc(f, desc, consumers=1)
            assert st == G.OK
            dst = torch.empty(n, dtype=torch.uint8, device="cuda")
            s = torch.cuda.Stream()
            st, nn = b.get_into(f, roid, dst.data_ptr(), n, s.cuda_stream)   # consumes -> unmapped
            assert st == G.OK and nn == n
            s.synchronize()
            st2, bad, _ = G.test_verify(dst.data_ptr(), n, 99, 0, 0)
            assert st2 == G.OK and bad == 0
            assert b.where(roid)[0] == G.ENOENT
        finally:
            b.close()
        p.stdin.write("done\n")
        p.stdin.flush()
        rel, used = p.stdout.readline().split(), p.stdout.readline().strip()
        assert rel == ["0", "0"] and used == "0"
    finally:
        p.wait(timeout=60)
