#!/bin/bash
# e2e with / without binding the bench process to the GPU's NUMA node (interleaved runs)
nvidia-smi topo -m 2>&1 | head -4; lscpu | grep -i "numa\|^CPU(s)"
for i in 1 2 3; do for N in 0 1; do
  CUSZP_E2E_NUMA=$N timeout 600 python bench.py --no-cpu-baseline --no-secondary --no-variants --no-datasets --steps 10 > gpurun_out/e2e_numa_${N}_$i.json 2>/dev/null
  python -c "
import json; e=json.loads(open('gpurun_out/e2e_numa_${N}_$i.json').read().strip().splitlines()[-1])['e2e']; print('numa=$N run $i', round(e['value'],2), 'bound', e['link_bound_gbs'], e['host_placement'])"
done; done
