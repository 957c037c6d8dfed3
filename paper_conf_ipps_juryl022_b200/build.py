"""Build libmstamp_b200.so for sm_100a (in-tree, so the .so travels with the repo snapshot).

The kernel templates are instantiated in several translation units (csrc/inst_*.cu, committed:
one explicit instantiation each) compiled in parallel, then linked with the host ABI.  The
library is rebuilt whenever the sources, headers or flags differ from the ones it was built
from: a content hash is stored next to it (lib/libmstamp_b200.so.sha256), so a shipped tree
with a stale library (timestamps do not travel reliably) is rebuilt, not reused.
"""
from __future__ import annotations

import concurrent.futures as cf
import hashlib
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
LIBDIR = os.path.join(HERE, "lib")
OBJDIR = os.path.join(HERE, "build")
LIB = os.path.join(LIBDIR, "libmstamp_b200.so")
NVCC = os.environ.get("NVCC", "nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "--expt-relaxed-constexpr", "-Xcompiler", "-fPIC", "-I", os.path.join(HERE, "..", "include")]

SOURCES = ["mp_kernels.cu", "mp_seed_tc.cu", "mp_api.cpp"]


def _sources():
    return [os.path.join(CSRC, s) for s in SOURCES] + [
        os.path.join(CSRC, f) for f in sorted(os.listdir(CSRC)) if f.startswith("inst_") and f.endswith(".cu")]


def _deps():
    return [os.path.join(CSRC, f) for f in os.listdir(CSRC)]


HASH = LIB + ".sha256"


def _digest():
    h = hashlib.sha256()
    h.update(" ".join([NVCC] + ARCH + FLAGS).encode())
    inc = os.path.join(HERE, "..", "include")
    for f in sorted(_deps()) + sorted(os.path.join(inc, x) for x in os.listdir(inc)):
        h.update(os.path.basename(f).encode())
        with open(f, "rb") as fh:
            h.update(fh.read())
    return h.hexdigest()


def _stale():
    if not os.path.exists(LIB) or not os.path.exists(HASH):
        return True
    with open(HASH) as f:
        return f.read().strip() != _digest()


def _obj_digest(src, cmd):
    """Content hash of one object's inputs: the command, the source and every header it can
    include (host sources: include/ and the internal header; CUDA sources: all csrc headers)."""
    h = hashlib.sha256()
    h.update(" ".join(cmd).encode())
    inc = os.path.join(HERE, "..", "include")
    hdrs = [os.path.join(inc, x) for x in os.listdir(inc)]
    if src.endswith(".cpp"):
        hdrs.append(os.path.join(CSRC, "mp_internal.h"))
    else:
        hdrs += [os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith((".cuh", ".h"))]
    for f in [src] + sorted(hdrs):
        with open(f, "rb") as fh:
            h.update(fh.read())
    return h.hexdigest()


def _compile(src):
    obj = os.path.join(OBJDIR, os.path.basename(src) + ".o")
    cmd = [NVCC] + ARCH + FLAGS + ["-c", src, "-o", obj]
    if os.environ.get("MP_PTXAS_V"):
        cmd += ["-Xptxas", "-v"]
    dg = _obj_digest(src, cmd)
    stamp = obj + ".sha256"
    if os.path.exists(obj) and os.path.exists(stamp) and open(stamp).read().strip() == dg:
        return obj   # unchanged inputs: reuse the object (incremental rebuild)
    subprocess.check_call(cmd)
    with open(stamp, "w") as f:
        f.write(dg + "\n")
    return obj


def build(force: bool = False, verbose: bool = True) -> str:
    if not force and not _stale():
        return LIB
    os.makedirs(LIBDIR, exist_ok=True)
    os.makedirs(OBJDIR, exist_ok=True)
    srcs = _sources()
    with cf.ThreadPoolExecutor(max_workers=min(len(srcs), os.cpu_count() or 4)) as ex:
        objs = list(ex.map(_compile, srcs))
    cmd = [NVCC] + ARCH + ["-shared", "-o", LIB] + objs + ["-lcudart"]
    subprocess.check_call(cmd)
    with open(HASH, "w") as f:
        f.write(_digest() + "\n")
    if verbose:
        print(f"built {LIB}", file=sys.stderr)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv)
