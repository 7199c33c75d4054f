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
    ap.add_argument("--e2e-steps", type=int, default=8)
    ap.add_argument("--stream-chunk", type=int, default=64, help="planes per chunk in the host-streamed e2e")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--share-gpu", action="store_true",
                    help="testing only: all ranks on cuda:0 with gloo plumbing (exercises the N>1 path on 1 GPU)")
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
# evaluated once: 3 springs x 27 (3 sub, d^2 5, sqrt + 1/d 11,
# d-L and K* 2, quotient 3, f*d 3) + force sum 15 + kick/drift 12 = 108, and the
# fused stats of every step 16 (3 x 4 exact-split centre terms, v.v 3, max 1).
FP64_OPS_STEP, FP64_OPS_STATS = 108, 16


def fp64_ops_per_node_update(two_step=False):
    return FP64_OPS_STEP + FP64_OPS_STATS


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


def load_traffic(n, kernel):
    """DRAM bytes per K1 launch from the committed ncu --set full capture, if it
    was taken on this workload (profiles/k1_traffic.json)."""
    path = os.path.join(ROOT, "profiles", "k1_traffic.json")
    try:
        with open(path) as f:
            d = json.load(f)
        e = d.get("%dx%dx%d/%s" % (n[0], n[1], n[2], kernel))
        return None if e is None else float(e["dram_bytes_per_launch"])
    except Exception:
        return None


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

def oracle_sample(n, budget_s, max_steps=None, warmup=0, planes=8):
    """Time the CPU oracle (as it stands) on a bounded sample of the workload: a
    (planes+2) x n1 x n2 slab -- `planes` interior planes of the full cross
    section -- stepped repeatedly. Returns (node-updates/s, sample description, steps)."""
    import oracle as O

    p = O.Params(n=(planes + 2, n[1], n[2]), seed=42)
    s = O.init(p)
    per_step = planes * (n[1] - 2) * (n[2] - 2)
    for _ in range(warmup):
        s, _ = O.step(s)
    t0 = time.perf_counter()
    steps = 0
    while True:
        s, _ = O.step(s)
        steps += 1
        el = time.perf_counter() - t0
        if max_steps is not None and steps >= max_steps:
            break
        if max_steps is None and el >= budget_s:
            break
    rate = per_step * steps / el
    desc = ("CPU oracle (oracle/somier_oracle.c, sequential fp64, gcc -O2) on a %d-plane slab of the %dx%dx%d "
            "cross-section (+2 halo planes), %d steps = %.3g node-updates in %.1f s"
            % (planes, n[0], n[1], n[2], steps, per_step * steps, el))
    return rate, desc, steps, el


def run_reference(a):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    n = a.n
    # Bound the whole --steps K --warmup W run to a few minutes: one oracle
    # node-update costs ~0.1-0.2 us on one core, so a step over P planes of the
    # n1 x n2 cross-section costs ~2e-7 * P * n1 * n2 s; budget ~150 s total.
    per_plane = 2e-7 * n[1] * n[2]
    planes = int(max(1, min(8, 150.0 / (max(1, a.steps + a.warmup) * per_plane))))
    rate, desc, steps, el = oracle_sample(n, budget_s=None, max_steps=a.steps, warmup=a.warmup, planes=planes)
    line = {
        "impl": "reference", "metric": METRIC, "value": rate, "unit": UNIT, "n_gpus": a.gpus, "steps": a.steps,
        "warmup": a.warmup, "ms_per_step": 1e3 * el / steps, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": workload_name(n), "n": list(n), "sample": "%d-plane slab per step" % planes},
        "cpu_baseline": {"value": rate, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": desc},
        "e2e": {"value": rate, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# --------------------------------------------------------------------------- our arm

def halo_info(n, chunks, world, two_step=False):
    """Halo traffic of the fused exchange: each chunk boundary between list
    positions moves one X plane (24 B per node of the n1 x n2 cross-section)
    each way per step, stored by K1 straight into the neighbour's halo slot
    (NVLink P2P / IPC); K1_TB2 moves two X planes and one V plane each way per
    two-step launch (36 B per cross-section node per step). Reported against
    the measured 770 GB/s peer rate (B200_PROFILING.md); the stores overlap the
    step, so this is a bound on the exchange's cost, not a separate phase."""
    plane = (36 if two_step else 24) * n[1] * n[2]
    cross = sum(1 for a, b in zip(chunks, chunks[1:]) if a.device_pos != b.device_pos)
    total = 2 * cross * plane
    per_rank = total / max(1, world)
    return {"bytes_per_step_total": total, "bytes_per_step_per_rank": per_rank,
            "est_us_at_770_gbs": per_rank / 770e9 * 1e6, "mechanism": "in-kernel peer stores + completion flag"}


def pcie_rates(local, nbytes=1 << 30):
    """Pinned host<->device copy rates (GB/s), one direction at a time and both
    directions concurrently -- the roofline of the host-streamed mode."""
    import torch

    h1 = torch.empty(nbytes // 8, dtype=torch.float64, pin_memory=True)
    h2 = torch.empty_like(h1, pin_memory=True)
    d1 = torch.empty(nbytes // 8, dtype=torch.float64, device="cuda")
    d2 = torch.empty_like(d1)
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    res = {}
    for name, fn in (("h2d", lambda: d1.copy_(h1, non_blocking=True)),
                     ("d2h", lambda: h1.copy_(d1, non_blocking=True))):
        fn()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        res[name] = 3 * nbytes / (time.perf_counter() - t0) / 1e9
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(3):
        with torch.cuda.stream(s1):
            d1.copy_(h1, non_blocking=True)
        with torch.cuda.stream(s2):
            h2.copy_(d2, non_blocking=True)
    torch.cuda.synchronize()
    res["bidir_total"] = 6 * nbytes / (time.perf_counter() - t0) / 1e9
    del h1, h2, d1, d2
    torch.cuda.empty_cache()
    return res


def e2e_stream(n, params, local, a, two_step):
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
    st = P.SomierStream(P.Spread([local], 1, n[0] - 2, chunk=chunk), params, buffers=3)
    grids = [torch.empty(tuple(n), dtype=torch.float64, pin_memory=True) for _ in range(12 if two_step else 9)]
    ptr = [g.data_ptr() for g in grids]
    X, V, XN = ptr[0:3], ptr[3:6], ptr[6:9]
    st.generate_ptrs(X + V)
    k = max(2, a.e2e_steps + (a.e2e_steps & 1))
    rates = pcie_rates(local)

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
    cyc1 = ("somier_stream_run on pinned host grids: per chunk of %d planes map(to: X[start-1:size+2], "
            "V[start:size]) -> fused K1 -> map(from: X[start:size], V[start:size]); 3 device slots, H2D/K1/D2H "
            "overlapped, steps chained by per-chunk events (no barrier per step); every step's stats read back" % chunk)
    cyc2 = ("somier_stream_run2 on pinned host grids: per chunk of %d planes map(to: X[start-2:size+4], "
            "V[start-1:size+2]) -> K1_TB2 (two steps) -> map(from: X[start:size], V[start:size]) into the other "
            "host buffers; 3 device slots, H2D/K1/D2H overlapped, launches chained by per-chunk events; every "
            "launch's stats (each second step) read back" % chunk)
    out = {"value": r["value"], "unit": UNIT, "h2d_bytes_per_step": r["h2d_bytes_per_step"],
           "d2h_bytes_per_step": r["d2h_bytes_per_step"], "steps": k, "wall_s": r["wall_s"],
           "cycle": cyc1,
           "roofline": {"bound": "pcie", "achieved_gbs": r["achieved_gbs"],
                        "peak_gbs_bidir_measured": rates["bidir_total"], "h2d_gbs": rates["h2d"],
                        "d2h_gbs": rates["d2h"], "frac": r["frac_pcie"]},
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
    params = P.SomierParams(n=n, seed=42, kernel=kernel)
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
    # K1_TB2 (AUTO on one chunk) advances two steps per launch: K even, so every
    # timed launch is a two-step launch
    in_use = s.kernel_in_use
    per_call = 2 if in_use == P.K1_TB2 else 1
    if a.steps % per_call:
        raise SystemExit("K1_TB2 runs steps in pairs: --steps must be even")
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
    # few more steps, each bracketed by events -- shows the power-cap ramp
    nd = min(a.steps, 20)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(nd)]
    with torch.cuda.stream(stream):
        for i in range(0, nd, per_call):
            ev[i][0].record(stream)
            s.step(per_call)
            ev[i][1].record(stream)
    s.sync()
    barrier()
    per_step = [ev[i][0].elapsed_time(ev[i][1]) for i in range(0, nd, per_call)]  # per launch

    step_dist = {"min": min(per_step), "median": statistics.median(per_step), "max": max(per_step),
                 "first5": statistics.mean(per_step[:5]), "last5": statistics.mean(per_step[-5:]),
                 "note": "diagnostic pass after the timed region, %d launches each bracketed by events" % len(per_step)}
    # roofline of the dominant kernel (K1) on this rank's launches: mean launch
    # duration over the timed region (this rank's time / this rank's launches)
    k1_ms = t_start.elapsed_time(t_end) / max(1, my_launches)
    c0 = my_chunks[0]
    alg = algorithmic_bytes(n, c0.start, c0.size)
    peak, peak_src = load_peaks()
    achieved = alg / (k1_ms * 1e-3) / 1e9
    kname = {P.K1_MARCH: "march", P.K1_MARCH2: "march2", P.K1_DIRECT: "direct", P.K1_TB2: "tb2"}[in_use]
    # the same launches against the fp64 pipe: the method's fp64 instructions
    # per node-update (FP64_OPS_* below) x node-updates per launch
    fp64_alg = interior_of(n, c0.size) * per_call * fp64_ops_per_node_update(per_call == 2)
    fp64_peak, fp64_src = load_fp64_peak()
    fp64_achieved = fp64_alg / (k1_ms * 1e-3) / 1e12
    traffic = load_traffic(n, kname) if not multi and len(my_chunks) == 1 else None
    copy_gbs = sustained_copy(local, stream) if a.copy_check else None
    st = PD.gather_stats(s) if multi else s.stats()

    # end-to-end through the public API with pinned host buffers. N = 1: the
    # host-streamed cycle (e2e_stream: one step per round trip; the two-step
    # cycle beside it when the resident kernel is K1_TB2). N > 1: per step, map(to) the whole state (X
    # with halos, V), one step, read the centers result and map(from) the
    # state -- the paper's One Buffer cycle, in core.
    e2e = None
    if not a.no_e2e and not multi:
        s.close()  # free the resident grid: the streamed mode needs only a few chunk buffers
        torch.cuda.empty_cache()
        e2e = e2e_stream(n, params, local, a, two_step=(in_use == P.K1_TB2))
    elif not a.no_e2e:
        shape = tuple(n)
        host = [torch.empty(shape, dtype=torch.float64, pin_memory=True) for _ in range(6)]
        ptrs = [h.data_ptr() for h in host]
        s.read_ptrs(ptrs)
        h2d = d2h = 0
        for c in my_chunks:
            plane = n[1] * n[2] * 8
            h2d += 3 * (c.size + 2) * plane + 3 * c.size * plane
            d2h += 3 * c.size * plane * 2 + (3 * plane if c.start == 1 else 0) + (3 * plane if c.start + c.size == n[0] - 1 else 0)
        # warm-up cycle
        s.load_ptrs(ptrs)
        s.step(1)
        s.stats()
        s.read_ptrs(ptrs)
        barrier()
        k = max(1, a.e2e_steps)
        t0 = time.perf_counter()
        e_start = torch.cuda.Event(enable_timing=True)
        e_end = torch.cuda.Event(enable_timing=True)
        e_start.record(stream)
        for _ in range(k):
            s.load_ptrs(ptrs)
            if multi:
                s.sync()
                torch.distributed.barrier()
            s.step(1)
            if multi:
                PD.gather_stats(s)
            else:
                s.stats()
            s.read_ptrs(ptrs)
        e_end.record(stream)
        s.sync()
        barrier()
        e_ms = e_start.elapsed_time(e_end)
        wall = time.perf_counter() - t0
        if multi:
            e_ms = float(all_max(e_ms))
        e2e = {"value": interior(n) * k / (e_ms * 1e-3), "unit": UNIT, "h2d_bytes_per_step": int(h2d * world),
               "d2h_bytes_per_step": int(d2h * world) + 88 * world, "steps": k, "wall_s": wall,
               "cycle": "somier_load (map to: X[start-1:size+2], V) -> somier_step(1) -> somier_stats -> "
                        "somier_read (map from) per step, pinned host buffers"}
        del host

    cpu = None
    if rank == 0 and not multi and not a.no_cpu_baseline:
        rate, desc, steps, el = oracle_sample(n, budget_s=a.cpu_seconds)
        cpu = {"value": rate, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": desc}

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": a.steps, "warmup": a.warmup,
            "ms_per_step": ms / a.steps, "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": "f64", "data": "synthetic",
            "config": {"workload": workload_name(n), "n": list(n), "parallelism": "spread%d" % world,
                       "spread": "devices(%s) range(1:%d) spread_schedule(static,%d)"
                                 % (",".join(str(d) for d in spread.devices), n[0] - 2, spread.chunk_size),
                       "kernel": "K1_" + kname.upper(), "l2": "no flush: 12.9 GB state >> 126 MB L2",
                       "seed": 42},
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": traffic, "peak_source": peak_src,
                         "kernel": "k1_%s_kernel" % kname, "algorithmic_bytes_per_launch": alg,
                         "avg_launch_ms": k1_ms, "launch_ms_distribution": step_dist,
                         "sustained_copy_gbs": copy_gbs, "steps_per_launch": per_call,
                         "one_step_equivalent_gbs": alg * per_call / (k1_ms * 1e-3) / 1e9,
                         "note": ("K1_TB2 advances two steps per pass over HBM: 'achieved' counts the bytes a launch "
                                  "must move (one pass); one_step_equivalent_gbs is the rate the one-step method "
                                  "would need for the same node-updates/s" if per_call == 2 else
                                  "one step per launch")},
            "roofline_fp64": {"bound": "alu", "achieved": fp64_achieved, "peak": fp64_peak, "unit": "Tinstr/s",
                              "frac": fp64_achieved / fp64_peak, "peak_source": fp64_src,
                              "alg_instr_per_launch": fp64_alg,
                              "alg_instr_per_node_update": fp64_ops_per_node_update(per_call == 2),
                              "note": "fp64 lane-instructions of node_math.cuh per node-update with spring reuse "
                                      "(DESIGN.md §6); recomputed ring / tile padding not counted"},
            "clocks": clk, "gpu_launches": launches, "e2e": e2e, "cpu_baseline": cpu,
            "halo": halo_info(n, spread.chunks(), world, per_call == 2),
            "stats": {"step": st.step, "centre": st.centre, "vmax": st.vmax},
        }
        print(json.dumps(line), flush=True)
    s.close()
    if multi:
        torch.distributed.barrier()
        torch.distributed.destroy_process_group()
    return 0


def main():
    a = parse()
    if a.warmup < 3:
        raise SystemExit("--warmup must be >= 3")
    if a.impl == "reference":
        return run_reference(a)
    return run_ours(a)


if __name__ == "__main__":
    sys.exit(main())
