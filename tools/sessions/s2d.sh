OUT=gpurun_out/s2d; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_graphs.py -x -q > $OUT/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest.log
bash tools/ab_tb2.sh s2d/ab main v3
timeout 600 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"; head -c 2500 $OUT/bench.json; echo; tail -2 $OUT/bench.err
for g in 128 256 1024; do for k in auto march2; do
 timeout 300 python bench.py --grid $g --kernel $k --no-e2e --no-cpu-baseline $( [ $g = 1024 ] && echo --steps 20 ) > $OUT/g$g.$k.json 2>$OUT/g$g.$k.err
 python -c "import json;d=json.load(open('$OUT/g$g.$k.json'));print($g,'$k',d['config']['kernel'],'%.4g'%d['value'],'%.4f'%d['ms_per_step'],d['clocks']['sm_mhz'])" 2>&1 | tail -1
done; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k1_ -s 3 -c 1 -o $OUT/full \
    python bench.py --steps 6 --warmup 4 --no-e2e --no-cpu-baseline > $OUT/ncu_full.log 2>&1; echo "ncu full rc=$?"
