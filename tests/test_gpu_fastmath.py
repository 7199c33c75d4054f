"""The branch-free correctly rounded sqrt / division of the spring law
(csrc/kernels/node_math.cuh) are bit-identical to CUDA's __dsqrt_rn /
__ddiv_rn over the operating range (tools/fastmath/check.cu, ~1e9 samples of
random and adversarial operands, signed zeros included)."""
import os
import subprocess

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_fast_sqrt_div_bit_identical_to_library(tmp_path):
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    exe = str(tmp_path / "check")
    subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3",
                           "-std=c++17", "-o", exe, os.path.join(ROOT, "tools", "fastmath", "check.cu")])
    r = subprocess.run([exe, "4000"], capture_output=True, text=True, timeout=300)
    print(r.stdout)
    assert r.returncode == 0, r.stdout + r.stderr
    assert "sqrt_mismatch 0 div_mismatch 0 fused_mismatch 0" in r.stdout
