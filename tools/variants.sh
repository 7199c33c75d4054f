#!/bin/bash
# Build K1 variants (here, no GPU) and time them on the GPU box:
#   bash tools/variants.sh build "tagA:-DK1_MIN_BLOCKS=2 -DK1_UNROLL=2" "tagB:..."
#   bash tools/variants.sh run tagA tagB          (under gpurun)
MODE=$1; shift
if [ "$MODE" = build ]; then
  for spec in "$@"; do
    tag=${spec%%:*}; defs=${spec#*:}
    SOMIER_BUILD_TAG=$tag SOMIER_NVCC_DEFS="$defs" python paper_conf_ipps_torresft22_b200/build.py -v 2>&1 | grep -A2 k1_march | grep -E "registers|spill" | tail -2
  done
else
  mkdir -p gpurun_out/variants
  for tag in "$@"; do
    SOMIER_LIB=$PWD/paper_conf_ipps_torresft22_b200/libsomier_$tag.so timeout 300 python bench.py --steps 100 --warmup 5 --no-e2e --no-cpu-baseline ${VBENCH} > gpurun_out/variants/$tag.json 2>gpurun_out/variants/$tag.err
    python -c "import json;d=json.load(open('gpurun_out/variants/$tag.json'));r=d['roofline'];print('$tag', '%.4g'%d['value'], 'ms %.4f'%d['ms_per_step'], 'first5 %.4f last5 %.4f'%(r['launch_ms_distribution']['first5'], r['launch_ms_distribution']['last5']))" 2>&1 | tail -1
  done
fi
