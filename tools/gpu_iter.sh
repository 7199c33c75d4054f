#!/bin/bash
# Fast iteration on K1: quick parity subset, short bench, one ncu --set full capture.
TAG=${1:-iter}
OUT=gpurun_out/$TAG
mkdir -p $OUT
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "not 128cube" > $OUT/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest.log
timeout 300 python bench.py --steps 50 --warmup 5 --no-e2e --no-cpu-baseline ${BENCH_ARGS} > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"
python -c "import json;d=json.load(open('$OUT/bench.json'));print('value %.4g ms/step %.4f frac %.4f clocks %s' % (d['value'], d['ms_per_step'], d['roofline']['frac'], d['clocks']))" 2>&1 | tail -1
if [ "${SKIP_NCU:-0}" != "1" ]; then
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k1_ -s 4 -c 1 -o $OUT/k1_full \
    python bench.py --steps 6 --warmup 3 --no-e2e --no-cpu-baseline ${BENCH_ARGS} > $OUT/ncu_full.log 2>&1; echo "ncu full rc=$?"
fi
