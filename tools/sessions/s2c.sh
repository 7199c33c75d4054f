OUT=gpurun_out/s2c; mkdir -p $OUT
./tools/microbench/fp64_rate > $OUT/fp64_rate.txt 2>&1; tail -1 $OUT/fp64_rate.txt
python __graft_entry__.py smoke > $OUT/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 $OUT/smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $OUT/pytest_gpu.log
timeout 600 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"; head -c 1500 $OUT/bench.json; echo
for g in 128 256 1024; do for k in auto march2; do
 timeout 300 python bench.py --grid $g --kernel $k --no-e2e --no-cpu-baseline $( [ $g = 1024 ] && echo --steps 20 ) > $OUT/g$g.$k.json 2>$OUT/g$g.$k.err
 python -c "import json;d=json.load(open('$OUT/g$g.$k.json'));print($g,'$k',d['config']['kernel'],'%.4g'%d['value'],'%.4f'%d['ms_per_step'],d['clocks']['sm_mhz'])" 2>&1 | tail -1
done; done
