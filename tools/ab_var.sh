#!/bin/bash
# A/B of variant builds (libsomier_<tag>.so, "main" = default lib) on one box:
# TB2 parity subset per variant, then alternating benches.
# Usage (under gpurun): bash tools/ab_var.sh OUTTAG tagA tagB ...
OUT=gpurun_out/$1; shift; mkdir -p $OUT
for tag in "$@"; do
  lib=$PWD/paper_conf_ipps_torresft22_b200/libsomier_$tag.so; [ "$tag" = main ] && lib=$PWD/paper_conf_ipps_torresft22_b200/libsomier.so
  SOMIER_LIB=$lib timeout 600 python -m pytest tests/test_gpu_parity.py -x -q ${PARITY_K:+-k "$PARITY_K"} > $OUT/pytest_$tag.log 2>&1; echo "pytest $tag rc=$?"; tail -1 $OUT/pytest_$tag.log
done
for rep in 1 2; do
for tag in "$@"; do
  lib=$PWD/paper_conf_ipps_torresft22_b200/libsomier_$tag.so; [ "$tag" = main ] && lib=$PWD/paper_conf_ipps_torresft22_b200/libsomier.so
  SOMIER_LIB=$lib timeout 300 python bench.py --kernel ${KERNEL:-tb2} --steps 100 --warmup 6 --no-e2e --no-cpu-baseline ${VBENCH} > $OUT/$tag.$rep.json 2>$OUT/$tag.$rep.err
  python -c "import json;d=json.load(open('$OUT/$tag.$rep.json'));r=d['roofline'];print('$tag', '%.4g'%d['value'], 'ms %.4f'%d['ms_per_step'], 'first5 %.4f last5 %.4f'%(r['launch_ms_distribution']['first5'], r['launch_ms_distribution']['last5']), d['clocks']['sm_mhz'], d['clocks']['reasons'])" 2>&1 | tail -1
done; done
for tag in $NCU_TAGS; do
  lib=$PWD/paper_conf_ipps_torresft22_b200/libsomier_$tag.so; [ "$tag" = main ] && lib=$PWD/paper_conf_ipps_torresft22_b200/libsomier.so
  SOMIER_LIB=$lib timeout 600 ncu --set full --clock-control none --import-source on -k regex:k1_ -s 3 -c 1 -o $OUT/full_$tag \
    python bench.py --kernel ${KERNEL:-tb2} --steps 6 --warmup 4 --no-e2e --no-cpu-baseline > $OUT/ncu_$tag.log 2>&1; echo "ncu $tag rc=$?"
done
