for L in 1 2 3; do CUSZP_E2E_LANES=$L timeout 600 python bench.py --no-cpu-baseline --no-secondary --no-variants --steps 10 > gpurun_out/bench_e2e_l$L.json 2>gpurun_out/bench_e2e_l$L.err; python -c "
import json; d=json.load(open('gpurun_out/bench_e2e_l$L.json')); print($L, d['e2e']['value'], d['e2e']['link_bound_gbs'], d['value'])"; done
