"""Builds libgrouter.so in-tree with nvcc for sm_100a (no JIT, no torch).

cudart is linked statically and only ``grouter_*`` symbols are exported
(linker version script), so the library never interposes on, or is
interposed by, the CUDA runtime PyTorch ships.

The library carries the SHA-256 of the sources it was built from (every
input file's bytes, and the compile flags): ``grouter_build_hash()`` returns
it and the marker ``GROUTER_SRC_HASH=<hex>`` is in the binary.  A build is
reused only when that hash equals the current sources' (not by mtime), and
``grouter.load()`` refuses a library whose hash differs from the tree.
"""
from __future__ import annotations

import hashlib
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libgrouter.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
SOURCES = ["api.cpp", "engine.cpp", "ipc.cpp", "paths.cpp", "plan.cpp", "pool.cpp", "probe.cpp", "kernels.cu"]
HEADERS = ["ce_run.h", "common.h", "ctx.h", "kernels.h", "plan.h", "stride.h"]


def _inputs():
    files = [os.path.join(CSRC, f) for f in SOURCES + HEADERS]
    files += [os.path.join(ROOT, "include", f) for f in ("grouter.h", "grouter_testing.h")]
    files.append(os.path.abspath(__file__))
    return files


COMMON = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC"]


def source_hash() -> str:
    """SHA-256 over every input file (name + bytes) and the compile flags."""
    h = hashlib.sha256()
    h.update(" ".join(COMMON + ARCH).encode())
    for f in _inputs():
        h.update(os.path.basename(f).encode() + b"\0")
        with open(f, "rb") as fh:
            h.update(fh.read())
    return h.hexdigest()


def built_hash(path: str = LIB) -> str | None:
    """The source hash embedded in a built library (marker scan, no dlopen)."""
    if not os.path.exists(path):
        return None
    data = open(path, "rb").read()
    k = data.find(b"GROUTER_SRC_HASH=")
    if k < 0:
        return None
    return data[k + 17:k + 17 + 64].decode("ascii", "replace")


def up_to_date() -> bool:
    return built_hash() == source_hash()


# Sanitizer builds of the host code (race detection): a separate
# library selected at load time with GROUTER_LIB (run the process with the
# sanitizer runtime preloaded, e.g. LD_PRELOAD=$(gcc -print-file-name=libtsan.so)).
SANITIZERS = {"tsan": ["-fsanitize=thread"], "asan": ["-fsanitize=address"]}


def lib_path(variant: str | None = None) -> str:
    return LIB if not variant else os.path.join(HERE, f"libgrouter_{variant}.so")


def build(force: bool = False, verbose: bool = False, variant: str | None = None) -> str:
    target = lib_path(variant)
    if not force and built_hash(target) == source_hash():
        return target
    objdir = os.path.join(HERE, "build" if not variant else f"build_{variant}")
    os.makedirs(objdir, exist_ok=True)
    digest = source_hash()
    san = SANITIZERS[variant] if variant else []
    san_cc = [x for f in san + (["-fno-omit-frame-pointer", "-g"] if san else []) for x in ("-Xcompiler", f)]
    common = COMMON + san_cc + ["-I", os.path.join(ROOT, "include"), f"-DGROUTER_SRC_HASH=\"{digest}\""] + ARCH
    objs = []
    procs = []
    for src in SOURCES:
        obj = os.path.join(objdir, src + ".o")
        objs.append(obj)
        cmd = [NVCC] + common + ["-c", os.path.join(CSRC, src), "-o", obj]
        if src.endswith(".cu"):
            cmd += ["-Xptxas", "-v"] if verbose else []
        procs.append((cmd, subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT)))
    for cmd, p in procs:
        out, _ = p.communicate()
        if p.returncode != 0:
            sys.stderr.write(out.decode())
            raise RuntimeError("nvcc failed: " + " ".join(cmd))
        if verbose and out:
            sys.stderr.write(out.decode())
    vscript = os.path.join(objdir, "exports.map")
    with open(vscript, "w") as f:
        f.write("{ global: grouter_*; local: *; };\n")
    tmp = target + ".tmp"
    link = [NVCC] + ARCH + ["-shared", "-cudart=static", "-o", tmp] + objs + [
        "-Xlinker", "--version-script=" + vscript, "-Xlinker", "-Bsymbolic",
        "-lpthread", "-ldl", "-lrt"] + [x for f in san for x in ("-Xcompiler", f)]
    r = subprocess.run(link, stdout=subprocess.PIPE, stderr=subprocess.STDOUT)
    if r.returncode != 0:
        sys.stderr.write(r.stdout.decode())
        raise RuntimeError("link failed")
    os.replace(tmp, target)
    return target


if __name__ == "__main__":
    var = next((a[2:] for a in sys.argv[1:] if a[2:] in SANITIZERS), None)   # --tsan / --asan
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv, variant=var))
