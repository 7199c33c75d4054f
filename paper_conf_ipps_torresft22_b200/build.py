"""Build libsomier.so in-tree: nvcc for sm_100a, -lineinfo, static cudart.

Sources: csrc/*.cpp (host driver, spread descriptor), csrc/*.cu and
csrc/kernels/*.cu (kernels). The public headers are include/spread.h and
include/somier.h at the repo root. Objects are compiled in parallel; the
library is relinked only when a source or header is newer than it.
"""
from __future__ import annotations

import concurrent.futures as cf
import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
# SOMIER_BUILD_TAG / SOMIER_NVCC_DEFS: variant builds for experiments (tools/variants.sh)
_TAG = os.environ.get("SOMIER_BUILD_TAG", "")
BUILD = os.path.join(PKG, "_build" + (("_" + _TAG) if _TAG else ""))
LIB = os.path.join(PKG, "libsomier%s.so" % (("_" + _TAG) if _TAG else ""))
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
COMMON = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC,-Wall,-Wno-unknown-pragmas",
          "-I" + INCLUDE, "-I" + CSRC]
# variant macros apply to host sources too: box shapes (driver_util.hpp) must match the kernels
DEFS = os.environ.get("SOMIER_NVCC_DEFS", "").split()
CU_FLAGS = ARCH + ["-Xptxas", "-v", "--expt-relaxed-constexpr"] + DEFS


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cpp")) + glob.glob(os.path.join(CSRC, "*.cu"))
                  + glob.glob(os.path.join(CSRC, "kernels", "*.cu")))


def headers():
    return (glob.glob(os.path.join(CSRC, "**", "*.hpp"), recursive=True)
            + glob.glob(os.path.join(CSRC, "**", "*.cuh"), recursive=True)
            + glob.glob(os.path.join(INCLUDE, "*.h")))


def _obj(src):
    rel = os.path.relpath(src, CSRC).replace(os.sep, "_")
    return os.path.join(BUILD, rel + ".o")


def _compile(src, newest_hdr, verbose):
    obj = _obj(src)
    if os.path.exists(obj) and os.path.getmtime(obj) >= max(os.path.getmtime(src), newest_hdr):
        return obj, ""
    cmd = [NVCC, *COMMON, "-c", src, "-o", obj]
    if src.endswith(".cu"):
        cmd[1:1] = CU_FLAGS
    else:
        cmd[1:1] = ARCH + DEFS
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("nvcc failed for %s:\n%s\n%s" % (src, " ".join(cmd), r.stderr))
    return obj, r.stderr if verbose else ""


def build(force: bool = False, verbose: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    srcs = sources()
    newest_hdr = max(os.path.getmtime(h) for h in headers())
    if force:
        for s in srcs:
            if os.path.exists(_obj(s)):
                os.remove(_obj(s))
    with cf.ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 4)) as ex:
        results = list(ex.map(lambda s: _compile(s, newest_hdr, verbose), srcs))
    objs = [o for o, _ in results]
    if verbose:
        for _, log in results:
            if log:
                sys.stderr.write(log)
    if not os.path.exists(LIB) or os.path.getmtime(LIB) < max(os.path.getmtime(o) for o in objs):
        tmp = LIB + ".tmp.%d" % os.getpid()
        cmd = [NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-cudart", "static", "-lrt", "-lpthread", "-ldl"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError("link failed:\n%s\n%s" % (" ".join(cmd), r.stderr))
        os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
