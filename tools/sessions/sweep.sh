#!/bin/bash
# bench.py across grid sizes (kernel-resident value + roofline), one JSON line each.
mkdir -p gpurun_out/sweep
for g in ${GRIDS:-16 128 256 512 1024 1200}; do
  steps=100; [ $g -ge 1024 ] && steps=20
  python bench.py --grid $g --steps $steps --warmup 5 --no-e2e --no-cpu-baseline > gpurun_out/sweep/g$g.json 2>gpurun_out/sweep/g$g.err
  python -c "import json;d=json.load(open('gpurun_out/sweep/g$g.json'));r=d['roofline'];print('$g', '%.4g'%d['value'], 'ms %.4f'%d['ms_per_step'], 'GB/s %.0f'%r['achieved'], 'frac %.3f'%r['frac'], 'median_launch %.4f'%r['launch_ms_distribution']['median'])"
done
