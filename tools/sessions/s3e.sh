# per-GPU slab of the 512^3 strong-scaling runs at N = 8 / 4 / 2 (66 / 130 / 257 planes incl. faces)
OUT=gpurun_out/slab; mkdir -p $OUT
run() { # n0 kernel nseg steps
  SOMIER_TB2_NSEG=$3 timeout 300 python bench.py --grid $1 512 512 --kernel $2 --steps $4 --warmup 6 --no-e2e --no-cpu-baseline > $OUT/g$1_$2_$3.json 2>$OUT/g$1_$2_$3.err
  python -c "import json;d=json.load(open('$OUT/g$1_$2_$3.json'));print('n0 $1 $2 nseg $3', '%.4g'%d['value'], 'ms %.5f'%d['ms_per_step'])" 2>&1 | tail -1
}
for rep in 1 2; do
run 66 tb2 0 400; run 66 tb2 1 400; run 66 tb2 2 400; run 66 tb2 3 400; run 66 tb2 4 400; run 66 march2 0 400
run 130 tb2 0 200; run 130 tb2 2 200; run 130 tb2 3 200; run 130 march2 0 200
done
run 257 tb2 0 200; run 257 march2 0 200
