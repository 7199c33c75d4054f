"""bench.py's contract: the JSON line the driver parses, for the reference arm
(the oracle, CPU) and for our arm at N = 1 and N = 2 (two ranks sharing one
GPU through CUDA IPC, gloo plumbing) -- the launch shapes of the round-end
runs, at small sizes."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
METRIC = json.load(open(os.path.join(ROOT, "BASELINE.json")))["metric"]


def _run(args, timeout=600, env=None):
    e = dict(os.environ)
    e.update(env or {})
    r = subprocess.run([sys.executable, *args], cwd=ROOT, capture_output=True, text=True, timeout=timeout, env=e)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    return lines, r


def _torchrun(nproc, port):
    return ["-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=%d" % nproc, "--master-addr=127.0.0.1",
            "--master-port=%d" % port]


def _check_common(d, n_gpus, steps, warmup):
    assert d["metric"] == METRIC
    assert d["unit"] == "node-updates/s" and d["higher_is_better"] is True
    assert d["n_gpus"] == n_gpus and d["steps"] == steps and d["warmup"] >= warmup
    assert d["value"] > 0 and d["ms_per_step"] > 0
    assert d["dtype"] == "f64" and d["data"] == "synthetic"
    assert d["config"]["workload"]
    assert d["vs_baseline"] is None


def test_reference_arm_json_line():
    lines, _ = _run(["bench.py", "--impl", "reference", "--steps", "2", "--warmup", "3"])
    assert len(lines) == 1
    d = json.loads(lines[0])
    _check_common(d, 1, 2, 3)
    assert d["impl"] == "reference"
    cb = d["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] == 1 and cb["value"] == d["value"]
    # the C-side timer, the CPU model, nproc and "1 of N cores"
    assert cb["cpu_model"] and cb["nproc"] >= 1 and cb["cores_label"] == "1 of %d cores" % cb["nproc"]
    assert cb["seconds"] > 0 and cb["steps"] == 2 and "oracle_run_timed" in cb["sample"]
    assert d["e2e"] == {"value": d["value"], "unit": d["unit"], "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}


def test_reference_arm_under_torchrun_prints_once():
    lines, _ = _run(_torchrun(2, 29561) + ["bench.py", "--impl", "reference", "--gpus", "2", "--steps", "2",
                                           "--warmup", "3"], env={"OMP_NUM_THREADS": "1"})
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["value"] > 0


def test_warmup_below_three_is_refused():
    r = subprocess.run([sys.executable, "bench.py", "--steps", "2", "--warmup", "1"], cwd=ROOT, capture_output=True,
                       text=True, timeout=120)
    assert r.returncode != 0


@pytest.mark.gpu
def test_our_arm_json_line_one_gpu():
    lines, _ = _run(["bench.py", "--grid", "64", "--steps", "4", "--warmup", "3", "--no-cpu-baseline", "--no-e2e",
                     "--verify", "--sustained-s", "0.2"])
    assert len(lines) == 1
    d = json.loads(lines[0])
    _check_common(d, 1, 4, 3)
    assert d["gpu_launches"] > 0
    r = d["roofline"]
    assert r["bound"] == "hbm" and r["unit"] == "GB/s" and r["peak"] > 0
    assert abs(r["frac"] - r["achieved"] / r["peak"]) < 1e-9
    # 96 B per node-update (24 n1 n2 per X plane + 72 per interior node)
    assert 90 < r["algorithmic_bytes_per_node_update"] < 110
    assert "sm_mhz" in d["clocks"] and "reasons" in d["clocks"]
    assert d["verify"]["ok"] and d["verify"]["nodes_checked"] > 0
    assert d["sustained"]["steps"] >= 2 and d["sustained"]["value"] > 0
    assert d["stats"]["every_step"] is True
    steps = [h["step"] for h in d["stats"]["last_steps"]]
    assert steps == list(range(d["stats"]["step"] - 3, d["stats"]["step"] + 1))


@pytest.mark.gpu
def test_our_arm_two_ranks_share_one_gpu():
    """N = 2 through torchrun (the driver's launch), both ranks on cuda:0 over
    CUDA IPC: one JSON line, whole-job value, the fused exchange's halo bytes."""
    lines, r = _run(_torchrun(2, 29563) + ["bench.py", "--gpus", "2", "--grid", "64", "--steps", "4", "--warmup",
                                           "3", "--share-gpu", "--no-cpu-baseline", "--e2e-steps", "2",
                                           "--stream-chunk", "8", "--verify", "--sustained-s", "0.2"],
                    env={"OMP_NUM_THREADS": "1"})
    assert len(lines) == 1, r.stdout[-2000:]
    d = json.loads(lines[0])
    _check_common(d, 2, 4, 3)
    assert d["gpu_launches"] > 0
    h = d["halo"]
    assert h["bytes_per_step_total"] > 0 and h["measured_wait_ms_per_launch"]["max"] >= 0
    assert len(d["roofline"]["per_rank"]) == 2
    # the same e2e cycle as at N = 1: host-streamed over devices(0, 1), one process
    assert d["e2e"]["value"] > 0 and d["e2e"]["h2d_bytes_per_step"] > 0 and "somier_stream_run" in d["e2e"]["cycle"]
    assert d["verify"]["ok"] and d["verify"]["nodes_checked"] > 0


@pytest.mark.gpu
def test_our_arm_four_ranks_same_fields_as_one():
    """N = 4 (ranks sharing cuda:0): the line carries the same field set as
    N = 1, plus per-rank roofline entries, and the verify pass is green."""
    common = ["--grid", "64", "--steps", "4", "--warmup", "3", "--no-cpu-baseline", "--e2e-steps", "2",
              "--stream-chunk", "8", "--verify", "--sustained-s", "0.2"]
    l1, _ = _run(["bench.py"] + common)
    l4, r = _run(_torchrun(4, 29567) + ["bench.py", "--gpus", "4", "--share-gpu"] + common,
                 env={"OMP_NUM_THREADS": "1"})
    assert len(l1) == 1 and len(l4) == 1, r.stdout[-2000:]
    d1, d4 = json.loads(l1[0]), json.loads(l4[0])
    assert set(d4) == set(d1)
    assert set(d4["roofline"]) == set(d1["roofline"]) | {"per_rank"}
    assert set(d4["e2e"]) == set(d1["e2e"]) and set(d4["halo"]) == set(d1["halo"])
    assert len(d4["roofline"]["per_rank"]) == 4 and d4["verify"]["ok"] and d4["n_gpus"] == 4



@pytest.mark.gpu
def test_our_arm_odd_steps_with_two_step_kernel():
    """An odd K with K1_TB2 (two steps per launch): the last launch is a
    one-step launch; the line reports K steps and a consistent roofline."""
    lines, _ = _run(["bench.py", "--grid", "64", "--kernel", "tb2", "--steps", "5", "--warmup", "3",
                     "--no-cpu-baseline", "--no-e2e", "--sustained-s", "0"])
    d = json.loads(lines[0])
    _check_common(d, 1, 5, 3)
    assert d["config"]["kernel"] == "K1_TB2" and d["gpu_launches"] == 3
    assert 90 < d["roofline"]["algorithmic_bytes_per_node_update"] < 110
