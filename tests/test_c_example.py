"""The C ABI used from a plain C program (examples/somier_c.c): compiles and
links against libsomier.so with gcc (no Python, no torch in the binary); on a
GPU its centres equal the oracle's bit for bit, without a GPU it fails
cleanly with SPREAD_ENODEV."""
import os
import re
import subprocess

import pytest

import oracle as O

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIBDIR = os.path.join(ROOT, "paper_conf_ipps_torresft22_b200")


def _build(tmp_path):
    exe = str(tmp_path / "somier_c")
    subprocess.check_call(["gcc", "-O2", "-Wall", "-Werror", "-I", os.path.join(ROOT, "include"),
                           os.path.join(ROOT, "examples", "somier_c.c"), "-L", LIBDIR, "-lsomier",
                           "-Wl,-rpath," + LIBDIR, "-o", exe])
    return exe


def test_c_example_builds_and_runs_spread_logic(tmp_path):
    exe = _build(tmp_path)
    out = subprocess.run(["ldd", exe], capture_output=True, text=True).stdout
    assert "libsomier.so" in out and "torch" not in out
    r = subprocess.run([exe, "16", "2", "5"], capture_output=True, text=True, timeout=120)
    assert "chunk 1: device 0, omp_spread_start 6, omp_spread_size 5, map(to: X[5:7])" in r.stdout
    try:
        import torch
        gpu = torch.cuda.is_available()
    except Exception:
        gpu = False
    if not gpu:
        assert r.returncode == 1 and "SPREAD_ENODEV" in r.stderr


@pytest.mark.gpu
def test_c_example_centre_equals_oracle(tmp_path):
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    exe = _build(tmp_path)
    r = subprocess.run([exe, "24", "10", "7"], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr
    m = re.search(r"centre \(([^,]+), ([^,]+), ([^)]+)\) vmax (\S+)", r.stdout)
    assert m, r.stdout
    _, st = O.run(O.init(O.Params(n=(24, 24, 24), seed=42)), 10)
    assert tuple(float(m.group(i)) for i in (1, 2, 3)) == st.centre
    assert float(m.group(4)) == st.vmax
    hist = re.findall(r"history step (\d+) centre \(([^,]+), ([^,]+), ([^)]+)\) vmax (\S+)", r.stdout)
    assert [int(h[0]) for h in hist] == [7, 8, 9, 10]
    s = O.init(O.Params(n=(24, 24, 24), seed=42))
    for t in range(1, 11):
        s, st = O.step(s)
        if t >= 7:
            h = hist[t - 7]
            assert tuple(float(v) for v in h[1:4]) == st.centre and float(h[4]) == st.vmax
