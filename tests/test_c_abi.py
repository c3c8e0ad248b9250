"""The boundary from C (not Python): tests/c/abi_consumer.c is compiled as
C99 with warnings as errors against include/grouter.h, linked against the
in-tree libgrouter.so, and run here without a GPU."""
import os
import shutil
import subprocess

import pytest

from paper_conf_eurosys_wulywdyfwwj26_b200 import _build

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_eurosys_wulywdyfwwj26_b200")


@pytest.mark.skipif(shutil.which("gcc") is None, reason="needs gcc")
def test_c99_consumer(tmp_path):
    _build.build()
    exe = tmp_path / "abi_consumer"
    cmd = ["gcc", "-std=c99", "-Wall", "-Wextra", "-Werror", "-I", os.path.join(ROOT, "include"),
           os.path.join(ROOT, "tests", "c", "abi_consumer.c"), "-o", str(exe), "-L", PKG, "-l:libgrouter.so",
           f"-Wl,-rpath,{PKG}"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    assert r.returncode == 0, r.stderr
    r = subprocess.run([str(exe)], capture_output=True, text=True, timeout=60)
    assert r.returncode == 0, (r.returncode, r.stdout, r.stderr)
    assert "route mask 0x55" in r.stdout          # R(0) = GPUs 0, 2, 4, 6 (L178, one per uplink)
    import torch
    if not torch.cuda.is_available():
        assert "GROUTER_ECUDA" in r.stdout, r.stdout   # no CPU fallback


@pytest.mark.skipif(shutil.which("g++") is None, reason="needs g++")
def test_ce_run_builder(tmp_path):
    """The copy-engine run builder (csrc/ce_run.h) on hand-written chunk
    lists: contiguous chunks -> one copy, a route's interleaved chunks of one
    transfer -> one 2-D copy, never across transfers, breaks on stride,
    direction or pitch limit (tests/c/ce_run_test.cpp)."""
    exe = tmp_path / "ce_run_test"
    r = subprocess.run(["g++", "-std=c++17", "-Wall", "-Wextra", "-Werror", "-O1",
                        os.path.join(ROOT, "tests", "c", "ce_run_test.cpp"), "-o", str(exe)],
                       capture_output=True, text=True)
    assert r.returncode == 0, r.stderr
    r = subprocess.run([str(exe)], capture_output=True, text=True, timeout=60)
    assert r.returncode == 0, r.stdout
    assert r.stdout.count(": ok") == 9, r.stdout
