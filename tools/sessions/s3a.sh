python tools/tb2_gap_probe.py 512
OUT=gpurun_out/seg2; mkdir -p $OUT
for ns in 1 2 3 4 5 6; do
  SOMIER_TB2_NSEG=$ns timeout 300 python bench.py --kernel tb2 --steps 100 --warmup 6 --no-e2e --no-cpu-baseline > $OUT/ns$ns.json 2>$OUT/ns$ns.err
  python -c "import json;d=json.load(open('$OUT/ns$ns.json'));r=d['roofline'];print('nseg $ns', '%.4g'%d['value'], 'ms %.4f'%d['ms_per_step'], 'med %.4f'%r['launch_ms_distribution']['median'], d['clocks']['sm_mhz'], d['clocks']['reasons'])" 2>&1 | tail -1
done
