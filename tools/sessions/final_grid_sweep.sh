# bench.py (AUTO kernel) at every BASELINE grid size, final code
OUT=gpurun_out/final_sweep; mkdir -p $OUT
for g in 128 160 192 256 384 512 768 1024 1200; do
  st=100; [ $g -le 256 ] && st=400; [ $g -ge 1024 ] && st=30
  timeout 600 python bench.py --grid $g --steps $st --warmup 6 --no-e2e --no-cpu-baseline > $OUT/g$g.json 2> $OUT/g$g.err
  python -c "import json;d=json.load(open('$OUT/g$g.json'));print($g, d['config']['kernel'], '%.4g'%d['value'], '%.4f'%d['ms_per_step'], '%.3f'%d['roofline']['frac'], d['clocks']['sm_mhz'])"
done
