#!/bin/bash
# A/B of programmatic dependent launch between K1 steps (SOMIER_NO_PDL=1 disables it).
for rep in 1 2; do for g in ${GRIDS:-128 256 512}; do for pdl in 0 1; do
  if [ $pdl = 1 ]; then unset SOMIER_NO_PDL; else export SOMIER_NO_PDL=1; fi
  python bench.py --grid $g --no-e2e --no-cpu-baseline > gpurun_out/pdl.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/pdl.json'));r=d['roofline'];print('$g r$rep pdl=$pdl', '%.4g'%d['value'], 'ms %.4f'%d['ms_per_step'], 'frac %.3f'%r['frac'])"
done; done; done
unset SOMIER_NO_PDL
