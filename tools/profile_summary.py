#!/usr/bin/env python3
"""Write a committed profile summary (profiles/<name>.md) from an ncu --set full
report and an ncu launch list (gpu__time_duration.sum), both read here."""
import collections
import csv
import io
import subprocess
import sys

METRICS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active", "sm__inst_executed.sum",
    "smsp__inst_executed.sum", "sm__warps_active.avg.per_cycle_active", "launch__registers_per_thread",
    "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem", "launch__grid_size",
    "launch__block_size", "sm__cycles_elapsed.avg.per_second", "lts__t_bytes.sum",
    "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_not_selected_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
    "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active",
    "sass__inst_executed_local_loads", "sass__inst_executed_local_stores",
]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {}
        for m in METRICS:
            if m in hdr:
                i = hdr.index(m)
                d[m] = (r[i], units[i])
        d["name"] = r[hdr.index("Kernel Name")] if "Kernel Name" in hdr else "?"
        res.append(d)
    return res


def launches(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if r and r[0] == "ID"][0]
    hdr, data = rows[hi], rows[hi + 1:]
    ki, vi = hdr.index("Kernel Name"), hdr.index("Metric Value")
    agg = collections.OrderedDict()
    for r in data:
        try:
            agg.setdefault(r[ki], []).append(float(r[vi].replace(",", "")))
        except (ValueError, IndexError):
            pass
    return agg


def main():
    rep, lcsv, out, title = sys.argv[1:5]
    note = sys.argv[5] if len(sys.argv) > 5 else ""
    lines = ["# %s" % title, "", note, ""]
    lines += ["## Launch list (ncu --metrics gpu__time_duration.sum --clock-control none; cold, serialised)", "",
              "| kernel | launches | mean us | share of listed time |", "|---|---|---|---|"]
    agg = launches(lcsv)
    tot = sum(sum(v) for v in agg.values())
    for k, v in agg.items():
        lines.append("| `%s` | %d | %.1f | %.3f |" % (k[:90], len(v), sum(v) / len(v) / 1e3, sum(v) / tot))
    lines += ["", "## ncu --set full (per launch)", ""]
    for d in raw(rep):
        lines.append("### `%s`" % d.pop("name")[:120])
        lines.append("")
        lines.append("| metric | value | unit |")
        lines.append("|---|---|---|")
        for m, (v, u) in d.items():
            lines.append("| %s | %s | %s |" % (m, v, u))
        lines.append("")
        break
    sass = subprocess.run([sys.executable, __file__.replace("profile_summary.py", "ncu_sass_summary.py"), rep],
                          capture_output=True, text=True).stdout
    lines += ["## SASS opcode mix (warp instructions executed, stall samples)", "", "```", sass.strip(), "```", ""]
    open(out, "w").write("\n".join(lines))
    print(out)


if __name__ == "__main__":
    main()
