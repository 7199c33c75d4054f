#!/bin/bash
# Exercise bench.py's N>1 path on a 1-GPU box (--share-gpu: both ranks on cuda:0,
# IPC within the device, gloo plumbing) and the big single-GPU configs.
OUT=gpurun_out/${1:-multi}
mkdir -p $OUT
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node=2 --master-addr=127.0.0.1 --master-port=29533 \
  bench.py --gpus 2 --steps 20 --warmup 3 --grid 256 --share-gpu --no-cpu-baseline > $OUT/bench_n2_share.json 2> $OUT/bench_n2_share.err
echo "n2 share rc=$?"; cat $OUT/bench_n2_share.json | cut -c1-400; tail -3 $OUT/bench_n2_share.err
timeout 600 python bench.py --grid 1024 --steps 20 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $OUT/bench_1024.json 2> $OUT/bench_1024.err
echo "1024 rc=$?"; python -c "import json;d=json.load(open('$OUT/bench_1024.json'));print('1024:', '%.4g'%d['value'], d['ms_per_step'], d['roofline']['frac'], d['roofline']['launch_ms_distribution'])"
timeout 900 python bench.py --grid 1200 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/bench_1200.json 2> $OUT/bench_1200.err
echo "1200 rc=$?"; python -c "import json;d=json.load(open('$OUT/bench_1200.json'));print('1200:', '%.4g'%d['value'], d['ms_per_step'], d['roofline']['frac'])"; tail -2 $OUT/bench_1200.err
timeout 300 python bench.py --grid 128 --steps 100 --warmup 5 --no-cpu-baseline --no-e2e > $OUT/bench_128.json 2> $OUT/bench_128.err
python -c "import json;d=json.load(open('$OUT/bench_128.json'));print('128:', '%.4g'%d['value'], d['ms_per_step'], d['roofline']['frac'])"
timeout 300 python bench.py --grid 256 --steps 100 --warmup 5 --no-cpu-baseline --no-e2e > $OUT/bench_256.json 2> $OUT/bench_256.err
python -c "import json;d=json.load(open('$OUT/bench_256.json'));print('256:', '%.4g'%d['value'], d['ms_per_step'], d['roofline']['frac'])"
