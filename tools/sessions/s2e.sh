OUT=gpurun_out/s2e; mkdir -p $OUT
for g in 128 192 256 384 512 768 1024; do for k in auto march2; do
 timeout 300 python bench.py --grid $g --kernel $k --no-e2e --no-cpu-baseline $( [ $g -ge 768 ] && echo --steps 30 ) > $OUT/g$g.$k.json 2>$OUT/g$g.$k.err
 python -c "import json;d=json.load(open('$OUT/g$g.$k.json'));print($g,'$k',d['config']['kernel'],'%.4g'%d['value'],'%.4f'%d['ms_per_step'],d['clocks']['sm_mhz'],d['clocks']['reasons'])" 2>&1 | tail -1
done; done
