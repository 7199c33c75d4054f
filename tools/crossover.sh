#!/bin/bash
# TB2 vs MARCH2 throughput over grid sizes (the AUTO threshold's evidence).
# Usage (under gpurun): bash tools/crossover.sh TAG "128 160 192 256 384 512"
OUT=gpurun_out/$1; mkdir -p $OUT
for n in $2; do
  steps=$(( n <= 192 ? 400 : (n <= 384 ? 100 : 40) ))
  for k in tb2 march2; do
    timeout 300 python bench.py --grid $n --kernel $k --steps $steps --warmup 6 --no-e2e --no-cpu-baseline \
        --sustained-s 0 > $OUT/x_${n}_$k.json 2> $OUT/x_${n}_$k.err
    python -c "import json;d=json.load(open('$OUT/x_${n}_$k.json'));print(json.dumps({'n':$n,'kernel':'$k','value':d['value'],'ms_per_step':d['ms_per_step'],'clocks':d['clocks']['sm_mhz'],'reasons':d['clocks']['reasons']}))" | tee -a $OUT/crossover.jsonl
  done
done
