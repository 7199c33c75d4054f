OUT=gpurun_out/seg3; mkdir -p $OUT
run() { # grid nseg
  SOMIER_TB2_NSEG=$2 timeout 300 python bench.py --grid $1 --kernel tb2 --steps ${3:-100} --warmup 6 --no-e2e --no-cpu-baseline > $OUT/g$1_ns$2.json 2>$OUT/g$1_ns$2.err
  python -c "import json;d=json.load(open('$OUT/g$1_ns$2.json'));r=d['roofline'];print('grid $1 nseg $2', '%.4g'%d['value'], 'ms %.4f'%d['ms_per_step'], 'med %.4f'%r['launch_ms_distribution']['median'], d['clocks']['sm_mhz'], d['clocks']['reasons'])" 2>&1 | tail -1
}
for ns in 4 6 3 5 8; do run 256 $ns 200; done
for ns in 6 12 4 8; do run 768 $ns; done
for ns in 7 16 4 10 1; do run 1024 $ns 50; done
for ns in 1 4 8 19; do run 1200 $ns 30; done
