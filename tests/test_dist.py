"""Multi-process (one process per list position) tests, world_size 2.

CPU (gloo): the distributed host logic -- chunk ownership by list position,
the halo-plane exchange pattern, exact cross-rank stats -- on oracle numbers;
result bit-identical to the full-grid oracle.
GPU: the product multi-process path (somier_init_local + CUDA IPC + fused
in-kernel exchange with flag waits), both ranks on cuda:0.
"""
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

import oracle as O

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
WORKER = os.path.join(ROOT, "tests", "_dist_worker.py")


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _launch(mode, out, n, steps, chunk, seed=3, timeout=300, kernel=None, exchange=None):
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr=127.0.0.1", "--master-port=%d" % _free_port(), WORKER, mode, out,
           *map(str, n), str(steps), str(chunk), str(seed)]
    env = dict(os.environ, OMP_NUM_THREADS="1", PYTHONPATH=ROOT)
    if kernel is not None:
        env["SOMIER_TEST_KERNEL"] = str(kernel)
    if exchange is not None:
        env["SOMIER_TEST_EXCHANGE"] = str(exchange)
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=timeout, env=env)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    return np.load(out)


def _check(res, n, steps, seed):
    ref, rst = O.run(O.init(O.Params(n=n, seed=seed)), steps)
    state = res["state"]
    assert np.array_equal(state[:3], ref.X)
    assert np.array_equal(state[3:], ref.V)
    assert [int(v) for v in res["sums"]] == list(rst.sums)
    assert int(str(res["vmax2"])) == rst.vmax2_bits
    assert tuple(res["centre"]) == rst.centre


@pytest.mark.parametrize("chunk", [0, 1, 3, 5])
def test_gloo_two_ranks_slab_exchange_bit_identical(tmp_path, chunk):
    n, steps, seed = (14, 9, 11), 6, 3
    res = _launch("oracle-slabs", str(tmp_path / "r.npz"), n, steps, chunk, seed)
    _check(res, n, steps, seed)
    assert int(res["nodes"]) == n[0] * n[1] * n[2]


@pytest.mark.gpu
@pytest.mark.parametrize("kernel", [0, 4])  # K1_AUTO (one-step kernel at this size), K1_TB2 (deep-halo exchange)
@pytest.mark.parametrize("chunk", [0, 2, 5])
def test_gpu_two_processes_ipc_fused_exchange(tmp_path, chunk, kernel):
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    n, steps, seed = (20, 12, 40), 15, 4
    res = _launch("gpu-ipc", str(tmp_path / "g.npz"), n, steps, chunk, seed, timeout=600, kernel=kernel)
    _check(res, n, steps, seed)
    # every step's global stats (per-rank history partials combined exactly)
    s = O.init(O.Params(n=n, seed=seed))
    for t in range(steps):
        s, st = O.step(s)
        assert [int(v) for v in res["hist_sums"][t]] == list(st.sums)
        assert int(str(res["hist_vmax2"][t])) == st.vmax2_bits


@pytest.mark.gpu
@pytest.mark.parametrize("kernel", [0, 4])
def test_gpu_two_processes_ipc_copy_exchange(tmp_path, kernel):
    """SOMIER_EXCHANGE_COPY across processes: cudaMemcpyAsync into the neighbour's
    IPC-mapped halo, then cuStreamWriteValue64 of its flag."""
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    n, steps, seed = (20, 12, 40), 15, 4
    res = _launch("gpu-ipc", str(tmp_path / "g.npz"), n, steps, 3, seed, timeout=600, kernel=kernel, exchange=1)
    _check(res, n, steps, seed)
