#!/bin/bash
# e2e (host-streamed, somier_stream_run) vs the streamed chunk size, 512^3.
for c in 16 32 64 128; do
  python bench.py --no-cpu-baseline --steps 10 --warmup 3 --stream-chunk $c > gpurun_out/e2e_c$c.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/e2e_c$c.json'));e=d['e2e'];print('chunk $c', '%.4g'%e['value'], 'frac %.3f'%e['roofline']['frac'], 'bidir %.1f'%e['roofline']['peak_gbs_bidir_measured'])"
done
