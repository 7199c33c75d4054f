"""Compile the C oracle into oracle/liboracle.so (TEST INFRASTRUCTURE).

Called by __graft_entry__.build() ("building the checker is not using it") and
lazily by oracle.somier when the .so is missing. Plain gcc, no FMA contraction.
"""
import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "somier_oracle.c")
LIB = os.path.join(HERE, "liboracle.so")
LIB_OMP = os.path.join(HERE, "liboracle_omp.so")
FLAGS = ["-O2", "-std=gnu11", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared", "-Wall"]


def _build(lib, extra, force):
    hdr = os.path.join(HERE, "somier_oracle.h")
    if not force and os.path.exists(lib):
        newest = max(os.path.getmtime(SRC), os.path.getmtime(hdr), os.path.getmtime(__file__))
        if os.path.getmtime(lib) >= newest:
            return lib
    tmp = lib + ".tmp.%d" % os.getpid()
    subprocess.check_call(["gcc", *FLAGS, *extra, "-o", tmp, SRC, "-lm"])
    os.replace(tmp, lib)
    return lib


def build(force: bool = False) -> str:
    """The sequential oracle (the OpenMP pragmas are ignored)."""
    return _build(LIB, ["-Wno-unknown-pragmas"], force)


def build_omp(force: bool = False) -> str:
    """The optional all-cores build: the same source with -fopenmp
    (bench.py's second CPU-baseline line; bit-identical, tests/test_oracle_omp.py)."""
    return _build(LIB_OMP, ["-fopenmp"], force)


if __name__ == "__main__":
    print(build(force=True))
    print(build_omp(force=True))
