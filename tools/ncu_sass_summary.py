#!/usr/bin/env python3
"""Summarise an ncu --set full report's SASS source page: executed warp
instructions and stall samples grouped by opcode, for the first kernel."""
import collections
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
kfilter = sys.argv[2] if len(sys.argv) > 2 else None
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
blocks = out.split('"Kernel Name"')
for blk in blocks[1:2] if not kfilter else [b for b in blocks[1:] if kfilter in b.splitlines()[0]][:1]:
    lines = blk.splitlines()
    print("kernel:", lines[0][:120])
    rd = csv.reader(io.StringIO("\n".join(lines[1:])))
    hdr = next(rd)
    ix = {h: i for i, h in enumerate(hdr)}
    inst = collections.Counter()
    stall = collections.Counter()
    total_i = total_s = 0
    for r in rd:
        if len(r) < len(hdr):
            continue
        op = r[ix["Source"]].strip().split()
        if not op:
            continue
        o = op[0]
        if o.startswith("@"):
            o = op[1] if len(op) > 1 else o
        o = o.split(".")[0]
        try:
            ie = int(r[ix["Instructions Executed"]] or 0)
            ss = int(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
        except ValueError:
            continue
        inst[o] += ie
        stall[o] += ss
        total_i += ie
        total_s += ss
    print("total warp instructions %d, stall samples %d" % (total_i, total_s))
    print("%-12s %14s %6s %8s" % ("opcode", "warp-inst", "%inst", "%stall"))
    for o, c in inst.most_common(40):
        print("%-12s %14d %6.1f %8.1f" % (o, c, 100.0 * c / total_i, 100.0 * stall[o] / max(1, total_s)))
