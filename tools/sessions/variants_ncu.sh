#!/bin/bash
# For each variant tag: bench line + one ncu launch with DRAM bytes.
mkdir -p gpurun_out/vncu
for tag in "$@"; do
  L=$PWD/paper_conf_ipps_torresft22_b200/libsomier_$tag.so
  SOMIER_LIB=$L timeout 300 python bench.py --steps 100 --warmup 5 --no-e2e --no-cpu-baseline ${VBENCH} > gpurun_out/vncu/$tag.json 2>/dev/null
  SOMIER_LIB=$L timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum --clock-control none -k regex:k1_ -s 4 -c 1 --csv python bench.py --steps 6 --warmup 3 --no-e2e --no-cpu-baseline ${VBENCH} > gpurun_out/vncu/$tag.csv 2>/dev/null
  python - "$tag" <<'PY'
import csv, json, sys
tag = sys.argv[1]
d = json.load(open("gpurun_out/vncu/%s.json" % tag)); r = d["roofline"]
vals = {}
for row in csv.reader(open("gpurun_out/vncu/%s.csv" % tag)):
    if len(row) > 14 and row[12] in ("dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__time_duration.sum", "lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum"):
        vals[row[12]] = row[13] + " " + row[14]
print(tag, "%.4g" % d["value"], "ms %.4f first5 %.4f last5 %.4f" % (d["ms_per_step"], r["launch_ms_distribution"]["first5"], r["launch_ms_distribution"]["last5"]), vals)
PY
done
