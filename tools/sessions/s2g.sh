OUT=gpurun_out/s2g; mkdir -p $OUT
python __graft_entry__.py smoke > $OUT/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 $OUT/smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -30 $OUT/pytest_gpu.log | grep -v "^\.\.\." | tail -25
timeout 300 python bench.py --no-e2e --no-cpu-baseline > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"; python -c "import json;d=json.load(open('$OUT/bench.json'));print(d['value'],d['config']['kernel'],d['roofline']['frac'])"
