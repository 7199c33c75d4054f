OUT=gpurun_out/r01_v9b; mkdir -p $OUT
python tools/tb2_gap_probe.py 512 > $OUT/gap.txt 2>&1; cat $OUT/gap.txt | tail -9
for rep in 1 2; do
timeout 600 python bench.py > $OUT/bench.$rep.json 2> $OUT/bench.$rep.err; echo "bench rc=$?"
python -c "import json;d=json.load(open('$OUT/bench.$rep.json'));r=d['roofline'];print('default', '%.4g'%d['value'], 'ms %.4f'%d['ms_per_step'], 'med %.4f'%r['launch_ms_distribution']['median'], d['clocks']['sm_mhz'], d['clocks']['reasons'])"
SOMIER_TB2_NSEG=1 timeout 300 python bench.py --steps 100 --warmup 6 --no-e2e --no-cpu-baseline > $OUT/ns1.$rep.json 2>$OUT/ns1.$rep.err
python -c "import json;d=json.load(open('$OUT/ns1.$rep.json'));r=d['roofline'];print('nseg1', '%.4g'%d['value'], 'ms %.4f'%d['ms_per_step'], 'med %.4f'%r['launch_ms_distribution']['median'], d['clocks']['sm_mhz'], d['clocks']['reasons'])"
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file $OUT/launches.csv \
    python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/ncu_list_bench.log 2>&1; echo "ncu list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k1_ -s 2 -c 1 -o $OUT/k1_full \
    python bench.py --steps 6 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/ncu_full.log 2>&1; echo "ncu full rc=$?"
