#!/bin/bash
# Round-2 characterisation on one B200: the AUTO kernel over grid sizes, and the
# per-rank slabs of the 512^3 / 1024^3 strong-scaling layouts (one chunk each).
# Usage (under gpurun): bash tools/sweep_r02.sh TAG
OUT=gpurun_out/$1; mkdir -p $OUT
for n in 128 192 256 384 512 768 1024; do
  steps=$(( n <= 192 ? 400 : (n <= 384 ? 100 : (n <= 512 ? 60 : 20)) ))
  timeout 600 python bench.py --grid $n --steps $steps --warmup 6 --no-e2e --no-cpu-baseline --sustained-s 0 \
      > $OUT/g_$n.json 2> $OUT/g_$n.err
  python -c "import json;d=json.load(open('$OUT/g_$n.json'));print(json.dumps({'n':$n,'kernel':d['config']['kernel'],'value':d['value'],'ms_per_step':d['ms_per_step'],'frac':d['roofline']['frac'],'sm_mhz':d['clocks']['sm_mhz'],'reasons':d['clocks']['reasons']}))" | tee -a $OUT/grid.jsonl
done
# per-rank slab of N-way strong scaling: n0 = ceil((n-2)/N) + 2 planes of the n x n cross-section
for spec in "512 2" "512 4" "512 8" "1024 8"; do
  set -- $spec; n=$1; N=$2; p=$(( (n - 2 + N - 1) / N + 2 ))
  timeout 600 python bench.py --grid $p $n $n --steps 100 --warmup 6 --no-e2e --no-cpu-baseline --sustained-s 0 \
      > $OUT/s_${n}_$N.json 2> $OUT/s_${n}_$N.err
  python -c "import json;d=json.load(open('$OUT/s_${n}_$N.json'));print(json.dumps({'grid':$n,'N':$N,'slab_planes':$p-2,'kernel':d['config']['kernel'],'value':d['value'],'ms_per_step':d['ms_per_step']}))" | tee -a $OUT/slabs.jsonl
done
timeout 900 python tools/logical_scale.py 1024 10 > $OUT/logical_1024.jsonl 2>&1; tail -1 $OUT/logical_1024.jsonl
