#!/bin/bash
# e2e variants (diagnostics): copy-stream sets x host stream buffers per set
timeout 300 python tools/e2e_probe.py c3_hacc
for L in 2 3; do for H in 1 2; do
  CUSZP_E2E_LANES=$L CUSZP_E2E_HBUF=$H timeout 600 python bench.py --no-cpu-baseline --no-secondary --no-variants --no-datasets --steps 10 > gpurun_out/bench_e2e_l${L}h${H}.json 2>gpurun_out/bench_e2e_l${L}h${H}.err
  python -c "
import json; d=json.load(open('gpurun_out/bench_e2e_l${L}h${H}.json')); e=d['e2e']; print('lanes $L hbuf $H', round(e['value'],2), 'bound', e['link_bound_gbs'], 'link', e['link_gbs_per_direction'])"
done; done
