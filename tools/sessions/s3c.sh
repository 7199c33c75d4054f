OUT=gpurun_out/cross; mkdir -p $OUT
run() { # grid kernel steps
  timeout 300 python bench.py --grid $1 --kernel $2 --steps $3 --warmup 6 --no-e2e --no-cpu-baseline > $OUT/g$1_$2.json 2>$OUT/g$1_$2.err
  python -c "import json;d=json.load(open('$OUT/g$1_$2.json'));print('grid $1 $2', '%.4g'%d['value'], 'ms %.5f'%d['ms_per_step'])" 2>&1 | tail -1
}
for g in 64 96 128 160 192 224 256; do for k in tb2 march2; do run $g $k 1000; done; done
