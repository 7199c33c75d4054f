#!/bin/bash
# Bench contract checks on one GPU: the bench tests, the default N=1 line with
# --verify, the N=2 (two ranks sharing cuda:0) line at 512^3 with --verify.
# Usage (under gpurun): bash tools/gpu_bench_check.sh TAG
OUT=gpurun_out/${1:-bench_check}; mkdir -p $OUT
timeout 900 python -m pytest tests/test_bench.py -x -q > $OUT/pytest_bench.log 2>&1; echo "pytest bench rc=$?"; tail -3 $OUT/pytest_bench.log
timeout 900 python bench.py --verify > $OUT/bench1.json 2> $OUT/bench1.err; echo "bench N=1 rc=$?"; tail -c 600 $OUT/bench1.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node=2 --master-addr=127.0.0.1 --master-port=29571 \
    bench.py --gpus 2 --share-gpu --verify --e2e-steps 4 > $OUT/bench2.json 2> $OUT/bench2.err; echo "bench N=2 rc=$?"; tail -c 600 $OUT/bench2.err
