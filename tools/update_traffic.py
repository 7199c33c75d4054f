#!/usr/bin/env python3
"""Record the DRAM bytes per launch of a K1 ncu --set full capture in
profiles/k1_traffic.json, tied to the kernel source it measured (sha1 of the
kernel's .cu and the shared headers, bench.kernel_source_sha): bench.py
reports roofline.traffic only while that source is unchanged.

  python tools/update_traffic.py REPORT.ncu-rep 512x512x512/tb2 "profiles/r02_....md (ncu --set full, gpurun TAG)"
"""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    rep, key, source = sys.argv[1:4]
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units, row = rows[0], rows[1], rows[2]

    def val(m):
        v, u = float(row[hdr.index(m)].replace(",", "")), units[hdr.index(m)]
        return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ms": 1, "us": 1e-3, "ns": 1e-6}.get(u, 1)

    import bench

    kernel = key.split("/")[1]
    path = os.path.join(ROOT, "profiles", "k1_traffic.json")
    d = json.load(open(path)) if os.path.exists(path) else {}
    d[key] = {"dram_bytes_per_launch": val("dram__bytes_read.sum") + val("dram__bytes_write.sum"),
              "gpu_time_ms": val("gpu__time_duration.sum"), "source": source,
              "source_sha": bench.kernel_source_sha(kernel)}
    if kernel == "tb2":
        d[key]["steps_per_launch"] = 2
    json.dump(d, open(path, "w"), indent=1)
    print(key, d[key])


if __name__ == "__main__":
    main()
