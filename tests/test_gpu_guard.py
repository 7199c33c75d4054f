"""SOMIER_GUARD: the device-memory bounds check of the GPU suite (guard.hpp).

Guard zones around every region of the resident chunks and the host-streamed
slots, verified at each synchronising call: an out-of-bounds write by a
kernel, a fused halo store or a copy fails the call. This is the device-memory
check where compute-sanitizer is not available (tests/test_gpu_sanitizer.py
skips there): the check itself is tested by fault injection, then the parity,
stream and logical-device suites and the sanitizer's kernel-path case run
under it."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

_PROBE = r"""
import sys
sys.path.insert(0, %r)
import numpy as np
import paper_conf_ipps_torresft22_b200 as P
n = (12, 14, 40)
sp = P.SomierParams(n=n, seed=5)
try:  # init synchronises too (the zones are checked there first)
    s = P.Somier(P.Spread([0, 1], 1, n[0] - 2), sp, cuda_devices=[0, 0])
    print("bytes", s.device_bytes)
    s.step(2)
    s.sync()
    print("resident ok")
except P.SpreadError as e:
    print("resident error:", e)
try:
    st = P.SomierStream(P.Spread([0], 1, n[0] - 2, chunk=4), sp, buffers=2)
    X, V = st.generate()
    st.step(X, V, np.zeros_like(X))
    print("stream ok")
except P.SpreadError as e:
    print("stream error:", e)
"""


def _run(code_or_args, env_extra, timeout=900):
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    env = dict(os.environ, PYTHONPATH=ROOT, **env_extra)
    args = [sys.executable, "-c", code_or_args] if isinstance(code_or_args, str) else [sys.executable] + code_or_args
    return subprocess.run(args, capture_output=True, text=True, timeout=timeout, env=env, cwd=ROOT)


def test_guard_detects_an_out_of_bounds_byte():
    off = _run(_PROBE % ROOT, {"SOMIER_GUARD": "0"})
    assert off.returncode == 0, off.stderr[-3000:]
    assert "resident ok" in off.stdout and "stream ok" in off.stdout, off.stdout
    on = _run(_PROBE % ROOT, {"SOMIER_GUARD": "1"})
    assert on.returncode == 0, on.stderr[-3000:]
    assert "resident ok" in on.stdout and "stream ok" in on.stdout, on.stdout
    b_off = int(off.stdout.split("bytes")[1].split()[0])
    b_on = int(on.stdout.split("bytes")[1].split()[0])
    assert b_on > b_off  # the zones exist
    # fault injection: one byte of the zone after X_0 (resident) / X in (stream) clobbered
    bad = _run(_PROBE % ROOT, {"SOMIER_GUARD": "1", "SOMIER_GUARD_SELFTEST": "1"})
    assert bad.returncode == 0, bad.stderr[-3000:]
    assert "resident error:" in bad.stdout and "SOMIER_GUARD: 1 byte(s)" in bad.stdout, bad.stdout
    assert "guard zone before X_1 of chunk 0" in bad.stdout, bad.stdout
    assert "stream error:" in bad.stdout and "guard zone before X out of slot 0" in bad.stdout, bad.stdout


def test_kernel_paths_clean_under_guard():
    r = _run([os.path.join(ROOT, "tools", "sanitize_case.py")], {"SOMIER_GUARD": "1", "SOMIER_NO_GRAPH": "1"})
    assert r.returncode == 0, (r.stdout + r.stderr)[-4000:]
    assert "sanitize case ok" in r.stdout


@pytest.mark.parametrize("suite", ["test_gpu_parity.py", "test_gpu_stream.py", "test_gpu_logical_devices.py",
                                   "test_gpu_stats_history.py"])
def test_suite_clean_under_guard(suite):
    r = _run(["-m", "pytest", "-q", "-x", "-p", "no:cacheprovider", os.path.join(ROOT, "tests", suite)],
             {"SOMIER_GUARD": "1"}, timeout=1500)
    assert r.returncode == 0, (r.stdout + r.stderr)[-4000:]
