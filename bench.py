#!/usr/bin/env python3
"""bench.py -- Somier node-updates/s on 1..8 B200 (BASELINE.json metric).

Workload (BASELINE.json configs[3]): Somier 512^3 grid, fp64, strong scaling
over 1/2/4/8 GPUs; the spread is devices(0..N-1) over the i-loop [1, 511) with
spread_schedule(static, ceil(510/N)) -- one slab per GPU. One bench "step" is
one Somier time step: the fused K1 kernel per chunk (forces, accelerations,
velocities, positions, centers, halo exchange). State = 12.9 GB >> 126 MB L2,
so no L2 flush is needed between steps.

  python bench.py [--gpus N --steps K --warmup W] [--grid 512] [--impl ours|reference]

N>1: launched by torch.distributed.run, one process per GPU (RANK/LOCAL_RANK/
WORLD_SIZE); the halo exchange is fused into the kernel over CUDA IPC/NVLink.
Rank 0 prints ONE JSON line. --impl reference times the CPU oracle (the
"reference arm" of this tier) on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "Somier node-updates/sec at 1/2/4/8 B200; % of HBM peak; parallel efficiency"
UNIT = "node-updates/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=6)
    ap.add_argument("--grid", type=int, nargs="+", default=[512],
                    help="grid nodes (one value: cube); not --n, which torch.distributed.run would claim")
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--kernel", choices=["auto", "direct", "march", "march2", "tb2"], default="auto")
    ap.add_argument("--chunk", type=int, default=0, help="spread_schedule(static, chunk); 0 = one slab per GPU")
    ap.add_argument("--exchange", choices=["fused", "copy", "nccl"], default="fused",
                    help="halo exchange route (somier_params.exchange)")
    ap.add_argument("--math", choices=["exact", "fma"], default="exact",
                    help="somier_params.math: exact = the oracle's operation order (bitwise), "
                         "fma = north_star's allowed FMA contraction (within 1e-10, DESIGN.md S22)")
    ap.add_argument("--e2e-steps", type=int, default=8)
    ap.add_argument("--stream-chunk", type=int, default=64, help="planes per chunk in the host-streamed e2e")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--no-cpu-all-cores", action="store_true", help="skip the all-cores (-fopenmp) oracle line")
    ap.add_argument("--oracle-child", default=None, help=argparse.SUPPRESS)
    ap.add_argument("--share-gpu", action="store_true",
                    help="testing only: all ranks on cuda:0 with gloo plumbing (exercises the N>1 path on 1 GPU)")
    ap.add_argument("--verify", action="store_true",
                    help="after the measurements: a fresh run of a few steps, nodes on both sides of every chunk "
                         "border (and the grid's first / last planes) checked bit for bit against the CPU oracle "
                         "through their light cone")
    ap.add_argument("--sustained-s", type=float, default=1.2,
                    help="seconds of the sustained pass after the timed region (0: skip)")
    ap.add_argument("--copy-check", action="store_true",
                    help="also time a sustained torch copy of the same byte volume (context for the roofline)")
    a = ap.parse_args()
    a.n = tuple(a.grid * 3 if len(a.grid) == 1 else a.grid)
    return a


def workload_name(n):
    return "Somier %dx%dx%d grid, fp64, strong scaling 1/2/4/8 B200 (BASELINE configs[3])" % n


def interior(n):
    return (n[0] - 2) * (n[1] - 2) * (n[2] - 2)


def algorithmic_bytes(n, start, size):
    """Per K1 launch over one chunk: read X_t on the owned planes + 2 halo planes
    (24 B/node), read V, write V, write X_{t+1} on interior nodes (72 B/node)."""
    return 24 * (size + 2) * n[1] * n[2] + 72 * size * (n[1] - 2) * (n[2] - 2)


def interior_of(n, size):
    """Interior nodes of a chunk of `size` planes."""
    return size * (n[1] - 2) * (n[2] - 2)


# fp64 lane-instructions per node-update of node_math.cuh with each spring
# evaluated once: 3 springs x 26 (3 sub, d^2 5, sqrt + 1/d 10 --
# its y/2 is an integer exponent decrement --, d-L and K* 2, quotient 3, f*d 3)
# + force sum 15 + kick/drift 12 = 105, and the fused stats of every step 15
# (3 x 3 exact-split centre terms, v.v 5, max 1). SOMIER_MATH_FMA: d^2 as an
# FMA chain (-2 per spring) and the kick/drift as 6 FMAs (-6): 93.
FP64_OPS_STEP, FP64_OPS_STEP_FMA, FP64_OPS_STATS = 105, 93, 15


def fp64_ops_per_node_update(math="exact"):
    return (FP64_OPS_STEP_FMA if math == "fma" else FP64_OPS_STEP) + FP64_OPS_STATS


def load_fp64_peak():
    """fp64 pipe peak (lane-instructions/s): tools/microbench/fp64_rate (DFMA,
    DADD, DMUL chains) measured on a B200 of this pool (profiles/fp64_rate.json),
    else 148 SMs x 64 fp64 lanes x 1.965 GHz."""
    try:
        with open(os.path.join(ROOT, "profiles", "fp64_rate.json")) as f:
            d = json.load(f)
        return float(d["fp64_tinstr_s"]), "measured (profiles/fp64_rate.json: %s)" % d.get("how", "")
    except Exception:
        return 148 * 64 * 1.965e9 / 1e12, "derived: 148 SMs x 64 fp64 lanes/clk x 1.965 GHz"


def load_peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(path) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


KERNEL_SRC = {"tb2": "k1_tb2.cu", "march2": "k1_march2.cu", "march": "k1_march.cu", "direct": "k1_direct.cu"}


def kernel_source_sha(kernel):
    """sha1 of the kernel's source files (its .cu + the shared headers): ties a
    committed ncu capture to the code it measured."""
    import hashlib

    kdir = os.path.join(ROOT, "paper_conf_ipps_torresft22_b200", "csrc", "kernels")
    h = hashlib.sha1()
    for name in [KERNEL_SRC.get(kernel, ""), "node_math.cuh", "stats.cuh", "signal.cuh", "tma.cuh"]:
        path = os.path.join(kdir, name)
        if os.path.exists(path):
            with open(path, "rb") as f:
                h.update(f.read())
    return h.hexdigest()


def load_traffic(n, kernel):
    """DRAM bytes per K1 launch (dram__bytes_read.sum + dram__bytes_write.sum)
    from the committed ncu --set full capture of this workload
    (profiles/k1_traffic.json); None unless the capture was taken on the
    kernel source as it is now (source_sha)."""
    path = os.path.join(ROOT, "profiles", "k1_traffic.json")
    try:
        with open(path) as f:
            d = json.load(f)
        e = d.get("%dx%dx%d/%s" % (n[0], n[1], n[2], kernel))
        if e is None or e.get("source_sha") != kernel_source_sha(kernel):
            return None, None
        return float(e["dram_bytes_per_launch"]), e.get("source")
    except Exception:
        return None, None


class ClockSampler:
    """nvidia-smi clocks, power and throttle reasons sampled every 20 ms during
    the run; only the samples whose timestamps fall inside the timed region
    (mark_start / mark_end) are summarised."""

    FIELDS = ("timestamp,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")
    NAMES = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.t0 = self.t1 = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), "--query-gpu=" + self.FIELDS,
                                          "--format=csv,noheader,nounits", "-lms", "20"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None

    def mark_start(self):
        self.t0 = time.time()

    def mark_end(self):
        self.t1 = time.time()

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.05)
        self.proc.terminate()
        out, _ = self.proc.communicate(timeout=10)
        import datetime
        sms, maxes, power, reasons, n_all = [], [], [], set(), 0
        for line in out.strip().splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) < 8:
                continue
            n_all += 1
            try:
                ts = datetime.datetime.strptime(f[0], "%Y/%m/%d %H:%M:%S.%f").timestamp()
            except ValueError:
                continue
            if self.t0 is not None and not (self.t0 <= ts <= (self.t1 or ts)):
                continue
            try:
                sms.append(float(f[1]))
                maxes.append(float(f[2]))
                power.append(float(f[3]))
            except ValueError:
                continue
            for nm, v in zip(self.NAMES, f[4:8]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        if not sms:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples in the timed region"],
                    "samples_total": n_all}
        return {"sm_mhz": statistics.median(sms), "sm_min_mhz": min(sms), "sm_max_mhz": max(maxes),
                "power_w_median": statistics.median(power), "reasons": sorted(reasons), "samples": len(sms)}


# --------------------------------------------------------------------------- oracle arm

def host_cpu():
    """CPU model, logical CPUs of the host, and the CPUs this process may use."""
    model = "unknown"
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    allowed = sorted(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else list(range(os.cpu_count() or 1))
    return model, os.cpu_count() or len(allowed), allowed


def oracle_child(spec):
    """Child process of the CPU baseline (bench.py --oracle-child JSON): the C
    oracle as it stands (oracle_run_timed: the step loop timed with the steady
    clock inside C, no per-step Python copies) on a (planes+2) x n1 x n2 slab of
    the workload's cross-section -- one calibration step, then enough steps for
    ~budget seconds. Prints one JSON object."""
    import oracle as O

    d = json.loads(spec)
    n1, n2, planes, omp = d["n1"], d["n2"], d["planes"], d["omp"]
    s = O.init(O.Params(n=(planes + 2, n1, n2), seed=42))
    if d.get("steps"):
        if d.get("warmup"):
            s, _, _, _ = O.run_timed(s, d["warmup"], omp=omp)
        steps = int(d["steps"])
    else:
        s, _, t1, _ = O.run_timed(s, 1, omp=omp)
        steps = max(1, int(d["budget"] / max(t1, 1e-6)))
    s, st, sec, threads = O.run_timed(s, steps, omp=omp)
    print(json.dumps({"steps": steps, "seconds": sec, "threads": threads,
                      "node_updates": planes * (n1 - 2) * (n2 - 2) * steps, "vmax": st.vmax}), flush=True)


def oracle_sample(n, budget_s=12.0, omp=False, planes=None, steps=None, warmup=0):
    """Time the CPU oracle on a bounded sample of the workload in a child
    process pinned to ONE core (sequential build), or to every core this
    process may use (the all-cores -fopenmp build, OMP_NUM_THREADS = that
    count). Returns the cpu_baseline object."""
    model, ncpu, allowed = host_cpu()
    cpus = allowed if omp else allowed[:1]
    if planes is None:
        planes = max(8, 4 * len(cpus)) if omp else 8  # the all-cores build splits the i loop
    planes = min(planes, n[0] - 2)
    spec = json.dumps({"n1": n[1], "n2": n[2], "planes": planes, "omp": omp, "budget": budget_s,
                       "steps": steps, "warmup": warmup})
    env = dict(os.environ)
    env["OMP_NUM_THREADS"] = str(len(cpus))
    env["OMP_PROC_BIND"] = "close"

    def pin():
        if hasattr(os, "sched_setaffinity"):
            os.sched_setaffinity(0, set(cpus))

    r = subprocess.run([sys.executable, os.path.abspath(__file__), "--oracle-child", spec], env=env,
                       preexec_fn=pin, capture_output=True, text=True, timeout=600)
    if r.returncode != 0:
        raise RuntimeError("oracle child failed: %s" % r.stderr[-2000:])
    d = json.loads(r.stdout.strip().splitlines()[-1])
    rate = d["node_updates"] / d["seconds"]
    build = ("oracle/liboracle_omp.so (the same somier_oracle.c, -fopenmp, %d threads)" % d["threads"] if omp
             else "oracle/liboracle.so (sequential fp64, gcc -O2 -ffp-contract=off)")
    desc = ("CPU oracle %s: oracle_run_timed (steady clock around the C step loop; every step's five kernels "
            "incl. centers) on a %d-plane slab of the %dx%dx%d cross-section (+2 halo planes), %d steps = %.3g "
            "node-updates in %.2f s; pinned to CPU%s %s" % (build, planes, n[0], n[1], n[2], d["steps"],
                                                          d["node_updates"], d["seconds"],
                                                          "s" if len(cpus) > 1 else "",
                                                          _cpu_list(cpus)))
    return {"value": rate, "unit": UNIT, "cores": len(cpus), "kind": "oracle", "sample": desc,
            "cpu_model": model, "nproc": ncpu, "cores_label": "%d of %d cores" % (len(cpus), ncpu),
            "steps": d["steps"], "seconds": d["seconds"], "threads": d["threads"]}


def _cpu_list(cpus):
    if len(cpus) > 1 and cpus == list(range(cpus[0], cpus[-1] + 1)):
        return "%d-%d" % (cpus[0], cpus[-1])
    return ",".join(str(c) for c in cpus)


def run_reference(a):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    n = a.n
    # Bound the whole --steps K --warmup W run to a few minutes: one oracle
    # node-update costs ~0.1 us on one core, so a step over P planes of the
    # n1 x n2 cross-section costs ~1e-7 * P * n1 * n2 s; budget ~120 s total.
    per_plane = 1.2e-7 * n[1] * n[2]
    planes = int(max(1, min(8, 120.0 / (max(1, a.steps + a.warmup) * per_plane))))
    cpu = oracle_sample(n, omp=False, planes=planes, steps=a.steps, warmup=a.warmup)
    line = {
        "impl": "reference", "metric": METRIC, "value": cpu["value"], "unit": UNIT, "n_gpus": a.gpus,
        "steps": a.steps, "warmup": a.warmup, "ms_per_step": 1e3 * cpu["seconds"] / cpu["steps"],
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": workload_name(n), "n": list(n), "sample": "%d-plane slab per step" % planes},
        "cpu_baseline": cpu,
        "e2e": {"value": cpu["value"], "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# --------------------------------------------------------------------------- our arm

def roofline_obj(achieved, peak, peak_src, traffic, traffic_src, k1_ms, kname, alg, alg_step, nu_launch, per_call,
                 step_dist, copy_gbs, fp64_frac):
    """The dominant kernel against HBM (SURVEY.md §8(d)'s algorithmic bytes: 96 B
    per node-update), the actual DRAM bytes of the committed ncu capture of this
    code (if any), and which roof is closest."""
    r = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
         "traffic": traffic, "peak_source": peak_src, "kernel": "k1_%s_kernel" % kname,
         "algorithmic_bytes_per_node_update": alg / nu_launch, "node_updates_per_launch": nu_launch,
         "algorithmic_bytes_per_launch": alg, "avg_launch_ms": k1_ms, "launch_ms_distribution": step_dist,
         "sustained_copy_gbs": copy_gbs, "steps_per_launch": per_call}
    if traffic:
        r["dram_actual"] = {"gbs": traffic / (k1_ms * 1e-3) / 1e9, "frac": traffic / (k1_ms * 1e-3) / 1e9 / peak,
                            "bytes_per_node_update": traffic / nu_launch, "source": traffic_src}
    fr = {"fp64 pipe (roofline_fp64)": fp64_frac}
    if traffic:
        fr["HBM (actual DRAM bytes)"] = r["dram_actual"]["frac"]
    closest = max(fr, key=fr.get)
    if per_call == 2:
        r["note"] = ("K1_TB2 advances two steps per pass over HBM, so it moves about half of §8(d)'s 96 B per "
                     "node-update (one pass = %d B per launch): 'frac' can exceed 1 against the one-step "
                     "algorithmic bytes. The roof that binds is the fp64 issue / latency: neither the fp64 pipe nor HBM is "
                     "saturated; closest: %s at %.2f" % (alg_step, closest, fr[closest]))
    else:
        r["note"] = "one step per launch; closest roof: %s at %.2f" % (closest, fr[closest])
    r["closest_roof"] = {"name": closest, "frac": fr[closest]}
    return r


def halo_info(n, chunks, world, two_step, ranks):
    """Halo traffic of the fused exchange: each chunk boundary between list
    positions moves one X plane (24 B per node of the n1 x n2 cross-section)
    each way per step, stored by K1 straight into the neighbour's halo slot
    (NVLink P2P / IPC); K1_TB2 moves two X planes and one V plane each way per
    two-step launch (36 B per cross-section node per step). Measured per rank
    (somier_set_timing, diagnostic pass): the time its stream sat in the
    neighbour-flag waits (neighbours' previous launch: their halo stores and
    their skew) and the kernel time, in which the peer stores run. Compared
    with the time the same bytes take at the measured 770 GB/s per-direction
    peer rate (B200_PROFILING.md; nominal NVLink 5: 900 GB/s)."""
    plane = (36 if two_step else 24) * n[1] * n[2]
    cross = sum(1 for a, b in zip(chunks, chunks[1:]) if a.device_pos != b.device_pos)
    total = 2 * cross * plane
    per_rank = total / max(1, world)
    per_launch = per_rank * (2 if two_step else 1)
    waits = [r["diag_wait_ms_per_launch"] for r in ranks]
    kern = [r["diag_kernel_ms_per_launch"] for r in ranks]
    return {"bytes_per_step_total": total, "bytes_per_step_per_rank": per_rank,
            "bytes_per_launch_per_rank": per_launch,
            "ideal_us_per_launch_at_770_gbs": per_launch / 770e9 * 1e6,
            "measured_wait_ms_per_launch": {"min": min(waits), "max": max(waits)},
            "measured_kernel_ms_per_launch": {"min": min(kern), "max": max(kern)},
            "wait_frac_of_launch": max(w / max(1e-9, w + k) for w, k in zip(waits, kern)),
            "mechanism": "in-kernel peer stores (NVLink P2P / CUDA IPC) + release-stored completion flag, "
                         "cuStreamWaitValue64 before the next launch"}


def run_verify(a, n, params, world, rank, local, multi):
    """A fresh run of a few steps in the benched configuration, then nodes on
    both sides of every chunk border (and near the grid's first / last planes)
    read back and compared bit for bit with the CPU oracle on a window reaching
    steps+1 nodes around each (a node after S steps depends only on initial
    values within distance S: tests/test_oracle_pins.py pins the window).
    Proves the cross-device exchange (peer stores, flags, waits) of this exact
    launch configuration. Each rank checks the planes it owns."""
    import numpy as np

    import oracle as O
    import paper_conf_ipps_torresft22_b200 as P
    from paper_conf_ipps_torresft22_b200 import dist as PD

    steps = 6
    if multi:
        s = PD.open_local(params, chunk=a.chunk, cuda_device=local)
    else:
        s = P.Somier(P.Spread([local], 1, n[0] - 2, chunk=a.chunk), params)
    mine = [c for c in s.spread.chunks() if (not multi) or c.device_pos == rank]
    s.step(steps)
    s.sync()
    planes = set()
    for c in mine:
        for i in (c.start, c.start + 1, c.start + c.size - 2, c.start + c.size - 1):
            if c.start <= i < c.start + c.size:
                planes.add(i)
    jk = [(1, 1), (n[1] // 2, n[2] // 2), (n[1] - 2, n[2] - 2), (n[1] // 3, n[2] - 2), (22, 31)]
    jk = [(j, k) for j, k in jk if 0 < j < n[1] - 1 and 0 < k < n[2] - 1]
    op = O.Params(n=n, seed=params.seed, spacing=params.spacing, rest_len=params.rest_len, k_spring=params.k_spring,
                  mass=params.mass, dt=params.dt, amplitude=params.amplitude)
    bad, checked = [], 0
    for i in sorted(planes):
        X, V = s.read_planes(i, 1)
        for j, k in jk:
            node = (i, j, k)
            lo = [max(0, node[d] - steps - 1) for d in range(3)]
            hi = [min(n[d], node[d] + steps + 2) for d in range(3)]
            win, _ = O.run(O.init_window(op, lo, [hi[d] - lo[d] for d in range(3)]), steps)
            r = tuple(node[d] - lo[d] for d in range(3))
            xo, vo = win.X[(slice(None),) + r], win.V[(slice(None),) + r]
            if params.math == P.MATH_EXACT:
                ok = np.array_equal(X[:, 0, j, k], xo) and np.array_equal(V[:, 0, j, k], vo)
            else:  # FMA contraction: north_star's 1e-10 bar, normwise over the window
                ok = (np.max(np.abs(X[:, 0, j, k] - xo)) <= 1e-10 * np.max(np.abs(win.X))
                      and np.max(np.abs(V[:, 0, j, k] - vo)) <= 1e-10 * max(np.max(np.abs(win.V)), 1e-300))
            checked += 1
            if not ok:
                bad.append(list(node))
    s.close()
    res = {"rank": rank, "checked": checked, "bad": bad}
    allr = PD.all_gather_obj(res) if multi else [res]
    nbad = sum(len(r["bad"]) for r in allr)
    return {"steps": steps, "nodes_checked": sum(r["checked"] for r in allr), "mismatches": nbad,
            "bad_nodes": [b for r in allr for b in r["bad"]][:20], "ok": nbad == 0,
            "what": "nodes on both sides of every chunk border, %s vs the CPU oracle (light-cone windows)"
                    % ("bitwise" if params.math == P.MATH_EXACT else "within 1e-10 (FMA mode)")}


def pcie_rates(devices, nbytes=None):
    """Pinned host<->device copy rates (GB/s) of the GPUs in `devices` (distinct
    CUDA ordinals), all at once: H2D alone, D2H alone, and both directions
    concurrently -- the roofline of the host-streamed mode."""
    import torch

    devs = sorted(set(devices))
    if nbytes is None:  # 1 GiB per buffer on one GPU, at least 256 MiB each on several
        nbytes = max(1 << 28, (1 << 30) // len(devs))
    hs = [torch.empty(nbytes // 8, dtype=torch.float64, pin_memory=True) for _ in range(2 * len(devs))]
    ds = [torch.empty(nbytes // 8, dtype=torch.float64, device="cuda:%d" % d) for d in devs for _ in range(2)]
    st = [torch.cuda.Stream(device=d) for d in devs for _ in range(2)]

    def run(h2d, d2h, reps=3):
        for d in devs:
            torch.cuda.synchronize(d)
        t0 = time.perf_counter()
        for _ in range(reps):
            for q in range(len(devs)):
                if h2d:
                    with torch.cuda.stream(st[2 * q]):
                        ds[2 * q].copy_(hs[2 * q], non_blocking=True)
                if d2h:
                    with torch.cuda.stream(st[2 * q + 1]):
                        hs[2 * q + 1].copy_(ds[2 * q + 1], non_blocking=True)
        for d in devs:
            torch.cuda.synchronize(d)
        return reps * len(devs) * nbytes * (int(h2d) + int(d2h)) / (time.perf_counter() - t0) / 1e9

    run(True, True, 1)
    res = {"h2d": run(True, False), "d2h": run(False, True), "bidir_total": run(True, True), "gpus": len(devs)}
    del hs, ds
    torch.cuda.empty_cache()
    return res


def e2e_stream(n, params, devices, a, two_step, cuda_devices=None):
    """End to end through the public C ABI with HOST buffers: the state lives in
    pinned host memory and every launch maps each chunk to the GPU (X with halo
    planes, V), runs the fused step(s) and maps X, V back -- the paper's `target
    spread` cycle with double buffering (3 device slots, 3 streams) and
    chunk-level dependencies between launches (the paper's future-work
    `depend`) instead of a barrier per step. Wall-clock
    timed: every host<->device copy and the read-back of every launch's stats
    is inside the timed region.
    The headline is the one-step cycle (somier_stream_run: every step's state
    mapped in and out, every step's stats read back). two_step (the resident
    kernel is K1_TB2): somier_stream_run2 -- two steps per round trip (X halo
    2, V halo 1, V double-buffered on the host), stats after every second step
    as on the resident handle -- is measured too and reported beside it."""
    import torch

    import paper_conf_ipps_torresft22_b200 as P

    chunk = a.stream_chunk
    st = P.SomierStream(P.Spread(list(devices), 1, n[0] - 2, chunk=chunk), params, buffers=3,
                        cuda_devices=cuda_devices)
    grids = [torch.empty(tuple(n), dtype=torch.float64, pin_memory=True) for _ in range(12 if two_step else 9)]
    ptr = [g.data_ptr() for g in grids]
    X, V, XN = ptr[0:3], ptr[3:6], ptr[6:9]
    st.generate_ptrs(X + V)
    k = max(2, a.e2e_steps + (a.e2e_steps & 1))
    rates = pcie_rates(cuda_devices if cuda_devices is not None else devices)

    def one_step():
        st.run_ptrs(X, V, XN, 1)  # warm-up step
        t0 = time.perf_counter()
        stats = st.run_ptrs(XN, V, X, k)[-1]
        wall = time.perf_counter() - t0
        tr = st.traffic()
        b = tr["h2d_bytes"] + tr["d2h_bytes"]
        return {"value": interior(n) * k / wall, "h2d_bytes_per_step": tr["h2d_bytes"],
                "d2h_bytes_per_step": tr["d2h_bytes"] + 88, "steps": k, "wall_s": wall,
                "frac_pcie": b / (wall / k) / 1e9 / rates["bidir_total"], "achieved_gbs": b / (wall / k) / 1e9,
                "last_step_vmax": stats.vmax}

    def two_steps():
        VN = ptr[9:12]
        st.run2_ptrs(X, V, XN, VN, 2)  # warm-up launch
        t0 = time.perf_counter()
        stats = st.run2_ptrs(XN, VN, X, V, k)[-1]
        wall = time.perf_counter() - t0
        tr = st.traffic2()
        b = (tr["h2d_bytes"] + tr["d2h_bytes"]) / 2
        return {"value": interior(n) * k / wall, "h2d_bytes_per_step": tr["h2d_bytes"] // 2,
                "d2h_bytes_per_step": (tr["d2h_bytes"] + 88) // 2, "steps": k, "wall_s": wall,
                "frac_pcie": b / (wall / k) / 1e9 / rates["bidir_total"], "achieved_gbs": b / (wall / k) / 1e9,
                "last_step_vmax": stats.vmax}

    r1 = one_step()
    r2 = two_steps() if two_step else None
    st.close()
    del grids
    # the headline is the strict cycle: every step's inputs mapped in and every
    # step's result read back; the two-step cycle is reported beside it
    r = r1
    cyc1 = ("somier_stream_run on pinned host grids, one host process driving devices(%s): per chunk of %d "
            "planes map(to: X[start-1:size+2], V[start:size]) -> fused K1 -> map(from: X[start:size], "
            "V[start:size]); 3 device slots per GPU, H2D/K1/D2H overlapped, steps chained by per-chunk events (no "
            "barrier per step); every step's stats read back" % (",".join(str(d) for d in devices), chunk))
    cyc2 = ("somier_stream_run2 on pinned host grids: per chunk of %d planes map(to: X[start-2:size+4], "
            "V[start-1:size+2]) -> K1_TB2 (two steps) -> map(from: X[start:size], V[start:size]) into the other "
            "host buffers; 3 device slots, H2D/K1/D2H overlapped, launches chained by per-chunk events; every "
            "step's stats read back" % chunk)
    out = {"value": r["value"], "unit": UNIT, "h2d_bytes_per_step": r["h2d_bytes_per_step"],
           "d2h_bytes_per_step": r["d2h_bytes_per_step"], "steps": k, "wall_s": r["wall_s"],
           "cycle": cyc1,
           "roofline": {"bound": "pcie", "achieved_gbs": r["achieved_gbs"],
                        "peak_gbs_bidir_measured": rates["bidir_total"], "h2d_gbs": rates["h2d"],
                        "d2h_gbs": rates["d2h"], "frac": r["frac_pcie"], "gpus": rates["gpus"]},
           "last_step_vmax": r["last_step_vmax"]}
    if two_step:
        out["two_step_cycle"] = {"value": r2["value"], "h2d_bytes_per_step": r2["h2d_bytes_per_step"],
                                 "d2h_bytes_per_step": r2["d2h_bytes_per_step"], "frac_pcie": r2["frac_pcie"],
                                 "cycle": cyc2}
    return out


def sustained_copy(device, stream, gib=6, iters=30):
    """Context only: a plain torch copy (read+write bytes) sustained back to back,
    the way K1 runs inside the bench, to compare against the burst hbm_gbs."""
    import torch

    n = gib * (1 << 30) // 8
    a = torch.empty(n, dtype=torch.float64, device=device)
    b = torch.empty_like(a)
    a.fill_(1.0)
    with torch.cuda.stream(stream):
        for _ in range(3):
            b.copy_(a)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(iters):
            b.copy_(a)
        e1.record(stream)
    e1.synchronize()
    gbs = 2 * n * 8 * iters / (e0.elapsed_time(e1) * 1e-3) / 1e9
    del a, b
    torch.cuda.empty_cache()
    return gbs


def run_ours(a):
    import numpy as np
    import torch

    import paper_conf_ipps_torresft22_b200 as P
    from paper_conf_ipps_torresft22_b200 import dist as PD

    rank, world, local = PD.env_rank()
    if world != a.gpus:
        raise SystemExit("--gpus %d but WORLD_SIZE %d" % (a.gpus, world))
    multi = world > 1
    if a.share_gpu:  # test mode: every rank on cuda:0 (IPC within one device), gloo plumbing
        local = 0
    torch.cuda.set_device(local)
    dev = "cpu" if a.share_gpu else "cuda"
    if multi:
        import torch.distributed as dist
        if a.share_gpu:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        # host-side waits (no NCCL kernel spinning on the GPUs rank 0 drives in the e2e)
        cpu_group = dist.new_group(backend="gloo") if not a.share_gpu else None

    def all_max(x, dtype=torch.float64):
        t = torch.tensor([x], device=dev, dtype=dtype)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        return t.item()

    def all_sum(x):
        t = torch.tensor([x], device=dev, dtype=torch.int64)
        torch.distributed.all_reduce(t)
        return int(t.item())
    n = a.n
    kernel = {"auto": P.K1_AUTO, "direct": P.K1_DIRECT, "march": P.K1_MARCH, "march2": P.K1_MARCH2,
              "tb2": P.K1_TB2}[a.kernel]
    exchange = {"fused": P.EXCHANGE_FUSED, "copy": P.EXCHANGE_COPY, "nccl": P.EXCHANGE_NCCL}[a.exchange]
    params = P.SomierParams(n=n, seed=42, kernel=kernel, exchange=exchange,
                            math={"exact": P.MATH_EXACT, "fma": P.MATH_FMA}[a.math])
    if multi:
        s = PD.open_local(params, chunk=a.chunk, cuda_device=local)
    else:
        s = P.Somier(P.Spread([local], 1, n[0] - 2, chunk=a.chunk), params)
    spread = s.spread
    my_chunks = [c for c in spread.chunks() if (not multi) or c.device_pos == rank]

    stream = torch.cuda.Stream(device=local)
    s.set_stream(rank if multi else 0, stream.cuda_stream)

    def barrier():
        torch.cuda.synchronize(local)
        if multi:
            torch.distributed.barrier()

    # warm-up (K1_TB2 runs steps in pairs: an odd W gets one more step so that
    # the timed region starts on an even step; "warmup" reports the steps done)
    if s.kernel_in_use == P.K1_TB2 and a.warmup % 2:
        a.warmup += 1
    with torch.cuda.stream(stream):
        s.step(a.warmup)
    s.sync()
    barrier()

    clocks = ClockSampler(local)
    clocks.start()
    time.sleep(0.5)
    # K1_TB2 (AUTO on one chunk) advances two steps per launch (an odd K ends
    # with one one-step launch: the roofline uses the mean steps per launch)
    in_use = s.kernel_in_use
    per_call = 2 if in_use == P.K1_TB2 else 1
    l0 = s.launches
    barrier()
    t_start = torch.cuda.Event(enable_timing=True)
    t_end = torch.cuda.Event(enable_timing=True)
    clocks.mark_start()
    # The K steps are ONE somier_step(K) call: CUDA-graph replay of (even, odd)
    # step pairs with programmatic dependent launch between consecutive K1s --
    # nothing of ours sits between two launches, so the mean launch duration is
    # (t_end - t_start) / launches, gaps included.
    t_start.record(stream)
    s.step(a.steps)
    t_end.record(stream)
    s.sync()
    clocks.mark_end()
    barrier()
    clk = clocks.stop()
    launches = my_launches = s.launches - l0
    ms = t_start.elapsed_time(t_end)
    if multi:
        ms = float(all_max(ms))
        launches = all_sum(launches)
    value = interior(n) * a.steps / (ms * 1e-3)
    # diagnostic only (not part of the timed region): per-launch durations of a
    # few more steps, each bracketed by events -- shows the power-cap ramp --
    # with the library's launch timing on (somier_set_timing: flag-wait and
    # kernel time of every launch on this rank; graph replay off)
    nd = min(a.steps, 20)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(nd)]
    s.set_timing(True)
    with torch.cuda.stream(stream):
        for i in range(0, nd, per_call):
            ev[i][0].record(stream)
            s.step(per_call)
            ev[i][1].record(stream)
    s.sync()
    tim = s.take_timing()
    s.set_timing(False)
    barrier()
    per_step = [ev[i][0].elapsed_time(ev[i][1]) for i in range(0, nd, per_call)]  # per launch

    step_dist = {"min": min(per_step), "median": statistics.median(per_step), "max": max(per_step),
                 "first5": statistics.mean(per_step[:5]), "last5": statistics.mean(per_step[-5:]),
                 "note": "diagnostic pass after the timed region, %d launches each bracketed by events" % len(per_step)}

    # sustained: >= --sustained-s seconds of steps in one somier_step call (the
    # board's steady state under its power cap), with its own clock samples
    sustained = None
    if a.sustained_s > 0:
        ss = int(a.sustained_s * 1e3 / max(1e-3, ms / a.steps))
        ss = max(per_call, ss - ss % per_call)  # whole launches
        if multi:
            ss = int(all_max(ss))
        csus = ClockSampler(local)
        csus.start()
        time.sleep(0.3)
        barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        csus.mark_start()
        e0.record(stream)
        s.step(ss)
        e1.record(stream)
        s.sync()
        csus.mark_end()
        barrier()
        sms = e0.elapsed_time(e1)
        if multi:
            sms = float(all_max(sms))
        sustained = {"steps": ss, "seconds": sms * 1e-3, "value": interior(n) * ss / (sms * 1e-3),
                     "ms_per_step": sms / ss, "clocks": csus.stop(),
                     "note": "one somier_step(%d) call after the timed region, CUDA events, max over ranks" % ss}

    # roofline of the dominant kernel (K1) on this rank's launches: mean launch
    # duration over the timed region (this rank's time / this rank's launches)
    k1_ms = t_start.elapsed_time(t_end) / max(1, my_launches)
    c0 = my_chunks[0]
    # algorithmic bytes = 24 n1 n2 per X_t plane read + 72 B per
    # interior node (V read + write, X_{t+1} write) per STEP (~96 B per
    # node-update); a launch processes spl steps of its chunk on average
    spl = a.steps * len(my_chunks) / max(1, my_launches)
    alg_step = sum(algorithmic_bytes(n, c.start, c.size) for c in my_chunks) / len(my_chunks)
    alg = alg_step * spl
    nu_launch = sum(interior_of(n, c.size) for c in my_chunks) / len(my_chunks) * spl
    peak, peak_src = load_peaks()
    achieved = alg / (k1_ms * 1e-3) / 1e9
    kname = {P.K1_MARCH: "march", P.K1_MARCH2: "march2", P.K1_DIRECT: "direct", P.K1_TB2: "tb2"}[in_use]
    # the same launches against the fp64 pipe: the method's fp64 instructions
    # per node-update (FP64_OPS_* below) x node-updates per launch
    fp64_alg = nu_launch * fp64_ops_per_node_update(a.math)
    fp64_peak, fp64_src = load_fp64_peak()
    fp64_achieved = fp64_alg / (k1_ms * 1e-3) / 1e12
    traffic, traffic_src = load_traffic(n, kname) if len(my_chunks) == 1 and c0.size == n[0] - 2 else (None, None)
    copy_gbs = sustained_copy(local, stream) if a.copy_check else None
    st = PD.gather_stats(s) if multi else s.stats()
    # every step's centres are kept (somier_stats_history): the last few, exact global values
    last = (PD.gather_stats_history(s, st.step - 3, 4) if multi else s.stats_history(st.step - 3, 4)) \
        if st.step >= 4 else []
    roof = roofline_obj(achieved, peak, peak_src, traffic, traffic_src, k1_ms, kname, alg, alg_step, nu_launch,
                        per_call, step_dist, copy_gbs, fp64_achieved / fp64_peak)
    # per rank: this rank's launch time, flag-wait time and kernel time
    mine = {"rank": rank, "chunks": [[c.start, c.size] for c in my_chunks], "avg_launch_ms": k1_ms,
            "hbm_frac": achieved / peak, "fp64_frac": fp64_achieved / fp64_peak,
            "diag_wait_ms_per_launch": tim["wait_ms"] / max(1, tim["launches"]),
            "diag_kernel_ms_per_launch": tim["kernel_ms"] / max(1, tim["launches"]),
            "diag_wait_max_ms": tim["wait_max_ms"]}
    ranks = PD.all_gather_obj(mine) if multi else [mine]
    halo = halo_info(n, spread.chunks(), world, per_call == 2, ranks)
    if multi:
        roof["per_rank"] = ranks

    # end-to-end through the public C ABI with HOST buffers, the same cycle at
    # every N: the host-streamed Somier (somier_stream_run, the paper's own
    # experiment) over devices(0..N-1) from ONE host process (the paper's model,
    # PAPER.md:346-399) -- at N > 1 rank 0 drives every GPU after all ranks
    # released their resident grids; the other ranks wait.
    e2e = None
    s.close()
    torch.cuda.empty_cache()
    barrier()
    if not a.no_e2e and rank == 0:
        cuda_devs = [0] * world if a.share_gpu else list(range(world))
        e2e = e2e_stream(n, params, list(range(world)), a, two_step=(in_use == P.K1_TB2), cuda_devices=cuda_devs)
    if multi:
        torch.distributed.barrier(group=cpu_group)  # the other ranks wait on the host
    barrier()

    verify = run_verify(a, n, params, world, rank, local, multi) if a.verify else None

    cpu = None
    if rank == 0 and not multi and not a.no_cpu_baseline:
        cpu = oracle_sample(n, budget_s=a.cpu_seconds)
        if not a.no_cpu_all_cores and len(host_cpu()[2]) > 1:
            cpu["all_cores"] = oracle_sample(n, budget_s=a.cpu_seconds / 2, omp=True)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": a.steps, "warmup": a.warmup,
            "ms_per_step": ms / a.steps, "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": "f64", "data": "synthetic",
            "config": {"workload": workload_name(n), "n": list(n), "parallelism": "spread%d" % world,
                       "spread": "devices(%s) range(1:%d) spread_schedule(static,%d)"
                                 % (",".join(str(d) for d in spread.devices), n[0] - 2, spread.chunk_size),
                       "kernel": "K1_" + kname.upper(), "exchange": a.exchange, "math": a.math,
                       "l2": "no flush: 12.9 GB state >> 126 MB L2",
                       "seed": 42},
            "roofline": roof,
            "roofline_fp64": {"bound": "alu", "achieved": fp64_achieved, "peak": fp64_peak, "unit": "Tinstr/s",
                              "frac": fp64_achieved / fp64_peak, "peak_source": fp64_src,
                              "alg_instr_per_launch": fp64_alg,
                              "alg_instr_per_node_update": fp64_ops_per_node_update(a.math),
                              "note": "fp64 lane-instructions of node_math.cuh / stats.cuh per node-update with "
                                      "spring reuse and every step's stats (DESIGN.md §6); recomputed ring / tile "
                                      "padding not counted"},
            "clocks": clk, "gpu_launches": launches, "e2e": e2e, "cpu_baseline": cpu,
            "halo": halo, "sustained": sustained,
            "stats": {"step": st.step, "centre": st.centre, "vmax": st.vmax, "every_step": True,
                      "last_steps": [{"step": h.step, "centre": h.centre, "vmax": h.vmax} for h in last],
                      "note": "centres and vmax of every step are computed inside the timed region "
                              "(somier_stats_history reads any of the last %d)" % P.STATS_HISTORY},
        }
        if verify is not None:
            line["verify"] = verify
        print(json.dumps(line), flush=True)
    if multi:
        torch.distributed.barrier()
        torch.distributed.destroy_process_group()
    return 0


def main():
    a = parse()
    if a.oracle_child is not None:
        return oracle_child(a.oracle_child)
    if a.warmup < 3:
        raise SystemExit("--warmup must be >= 3")
    if a.impl == "reference":
        return run_reference(a)
    return run_ours(a)


if __name__ == "__main__":
    sys.exit(main())
