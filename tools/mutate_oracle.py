#!/usr/bin/env python3
"""Mutation check of the oracle's pins.

Each mutant is one plausible mistake in oracle/somier_oracle.c (a dropped term,
a wrong sign or index, a swapped operand, the wrong parameter). The mutant is
compiled to a temporary library, tests/test_oracle_pins.py runs against it
(ORACLE_LIB), and the mutant counts as killed when at least one pin fails.
A surviving mutant means a part of the oracle is "parity unpinned".

  python tools/mutate_oracle.py [--out profiles/r02_oracle_mutants.json] [--only NAME ...]
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "oracle", "somier_oracle.c")
sys.path.insert(0, ROOT)

# (name, original text, mutated text): each original must occur exactly once
MUTANTS = [
    ("accel_f_times_m", "double oracle_acceleration_1(double f, double m) { return f / m; }",
     "double oracle_acceleration_1(double f, double m) { return f * m; }"),
    ("forces_rest_len_is_spacing", "oracle_spring(xp, xq, p->k_spring, p->rest_len, gs[s]);",
     "oracle_spring(xp, xq, p->k_spring, p->spacing, gs[s]);"),
    ("accels_mass_is_dt", "ax[g] = oracle_acceleration_1(fx[g], p->mass);",
     "ax[g] = oracle_acceleration_1(fx[g], p->dt);"),
    ("spring_sign", "double dx = xq[0] - xp[0];", "double dx = xp[0] - xq[0];"),
    ("spring_drop_dz2", "double d2 = (dx * dx + dy * dy) + dz * dz;", "double d2 = (dx * dx + dy * dy);"),
    ("spring_d_plus_L", "double f = (K * (d - L)) / d;", "double f = (K * (d + L)) / d;"),
    ("spring_no_divide", "double f = (K * (d - L)) / d;", "double f = (K * (d - L));"),
    ("forces_left_to_right_sum",
     "F[c] = ((gs[0][c] + gs[1][c]) + (gs[2][c] + gs[3][c])) + (gs[4][c] + gs[5][c]);",
     "F[c] = ((((gs[0][c] + gs[1][c]) + gs[2][c]) + gs[3][c]) + gs[4][c]) + gs[5][c];"),
    ("forces_drop_k_springs",
     "F[c] = ((gs[0][c] + gs[1][c]) + (gs[2][c] + gs[3][c])) + (gs[4][c] + gs[5][c]);",
     "F[c] = ((gs[0][c] + gs[1][c]) + (gs[2][c] + gs[3][c]));"),
    ("forces_wrong_neighbour", "IDX(p, i, j - 1, k), IDX(p, i, j + 1, k),", "IDX(p, i, j - 1, k), IDX(p, i, j - 1, k),"),
    ("velocity_explicit_euler_order", "oracle_velocities(p, ax, ay, az, vx, vy, vz);      /* velocities    */\n"
     "    oracle_positions(p, x, y, z, vx, vy, vz, xn, yn, zn); /* positions  */",
     "oracle_positions(p, x, y, z, vx, vy, vz, xn, yn, zn); /* positions  */\n"
     "    oracle_velocities(p, ax, ay, az, vx, vy, vz);      /* velocities    */"),
    ("velocity_minus", "double oracle_velocity_1(double v, double a, double dt) { return v + a * dt; }",
     "double oracle_velocity_1(double v, double a, double dt) { return v - a * dt; }"),
    ("position_no_dt", "double oracle_position_1(double x, double v, double dt) { return x + v * dt; }",
     "double oracle_position_1(double x, double v, double dt) { return x + v; }"),
    ("faces_move", "return i > 0 && i < p->n[0] - 1 && j > 0", "return i > 0 && i < p->n[0] && j > 0"),
    ("init_drop_amplitude", "v = x0[c] + p->amplitude * s;             /* 2 roundings */",
     "v = x0[c] + s;             /* 2 roundings */"),
    ("init_counter_off_by_one", "oracle_splitmix64_at(p->seed, 3u * (uint64_t)g + (uint64_t)c);\n"
     "                        double u = (double)(r >> 11) * 0x1.0p-53; /* u in [0,1), 53 bits */",
     "oracle_splitmix64_at(p->seed, 3u * (uint64_t)g + (uint64_t)c + 1u);\n"
     "                        double u = (double)(r >> 11) * 0x1.0p-53; /* u in [0,1), 53 bits */"),
    ("lattice_not_centred", "out[c] = ((double)idx[c] - centre) * p->spacing;", "out[c] = ((double)idx[c]) * p->spacing;"),
    ("centre_floor_quantise", "return (__int128)nearbyint(s);", "return (__int128)floor(s);"),
    ("centre_divides_by_interior", "out->centre[c] = ldexp((double)sum[c], -60) / (double)n;",
     "out->centre[c] = ldexp((double)sum[c], -60) / (double)(n - 1);"),
    ("vmax_drop_vz", "double v2 = (vx[g] * vx[g] + vy[g] * vy[g]) + vz[g] * vz[g];",
     "double v2 = (vx[g] * vx[g] + vy[g] * vy[g]);"),
    ("stencil3_drop_right", "b[i] = a[i - 1] + a[i] + a[i + 1];", "b[i] = a[i - 1] + a[i];"),
    ("gauss_seidel_positions", "xn[g] = oracle_position_1(x[g], vx[g], p->dt);",
     "xn[g] = oracle_position_1(x[g], vx[g], p->dt); ((double*)x)[g] = xn[g];"),
]


def build(src_text, out):
    with tempfile.NamedTemporaryFile("w", suffix=".c", delete=False, dir=os.path.dirname(out)) as f:
        f.write(src_text)
        cpath = f.name
    try:
        subprocess.check_call(["gcc", "-O2", "-std=gnu11", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared",
                               "-I", os.path.join(ROOT, "oracle"), "-o", out, cpath, "-lm"])
    finally:
        os.unlink(cpath)


def run_pins(lib, select=None, timeout=600):
    env = dict(os.environ, ORACLE_LIB=lib)
    cmd = [sys.executable, "-m", "pytest", "-q", "-x", "-p", "no:cacheprovider",
           os.path.join(ROOT, "tests", "test_oracle_pins.py")]
    if select:
        cmd += ["-k", select]
    t0 = time.time()
    r = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=timeout, cwd=ROOT)
    failed = [ln.split(" ")[1] for ln in r.stdout.splitlines() if ln.startswith("FAILED ")]
    return r.returncode, failed, time.time() - t0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    ap.add_argument("--only", nargs="*")
    a = ap.parse_args()
    base = open(SRC).read()
    results = []
    with tempfile.TemporaryDirectory() as td:
        lib0 = os.path.join(td, "orig.so")
        build(base, lib0)
        rc, failed, el = run_pins(lib0)
        results.append({"mutant": "(unmodified)", "killed": rc != 0, "first_failure": failed[:1], "s": round(el, 1)})
        for name, orig, mut in MUTANTS:
            if a.only and name not in a.only:
                continue
            if base.count(orig) != 1:
                raise SystemExit("mutant %s: original text occurs %d times" % (name, base.count(orig)))
            lib = os.path.join(td, name + ".so")
            build(base.replace(orig, mut), lib)
            rc, failed, el = run_pins(lib)
            results.append({"mutant": name, "killed": rc != 0, "first_failure": failed[:1], "s": round(el, 1)})
            print("%-32s %s %s" % (name, "killed" if rc else "SURVIVED", failed[:1]), flush=True)
    survived = [r["mutant"] for r in results[1:] if not r["killed"]]
    summary = {"oracle": "oracle/somier_oracle.c", "pins": "tests/test_oracle_pins.py",
               "unmodified_passes": not results[0]["killed"], "mutants": len(results) - 1,
               "killed": len(results) - 1 - len(survived), "survived": survived, "results": results}
    print(json.dumps({k: v for k, v in summary.items() if k != "results"}))
    if a.out:
        with open(a.out, "w") as f:
            json.dump(summary, f, indent=1)
    return 1 if survived or not summary["unmodified_passes"] else 0


if __name__ == "__main__":
    sys.exit(main())
