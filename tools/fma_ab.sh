set -x
mkdir -p gpurun_out/fma
timeout 900 python -m pytest tests/test_gpu_fma.py tests/test_gpu_parity.py -x -q > gpurun_out/fma/pytest.log 2>&1
tail -5 gpurun_out/fma/pytest.log
for r in 1 2; do
 for m in exact fma; do
  timeout 300 python bench.py --steps 100 --warmup 6 --math $m --no-e2e --no-cpu-baseline --sustained-s 0 2>/dev/null | tail -1 >> gpurun_out/fma/bench.jsonl
 done
done
