#!/bin/bash
# one GPU round (run through gpurun): tests, scan trace, bench, ncu
# usage: tools/gpu_check.sh [quick]   (quick: skip slow tests and the ncu pass)
set -x
if [ "$1" == "quick" ]; then K="not slow"; else K=""; fi
timeout 900 python -m pytest tests -m gpu -x -q -k "$K" 2>&1 | tail -15
timeout 300 python tools/trace_scan.py 2>&1 | tail -30
python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -3 gpurun_out/bench.err
if [ "$1" != "quick" ]; then
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"compress_kernel|decompress_kernel|range_kernel" -s 9 -c 3 -o gpurun_out/prof python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-large > gpurun_out/ncu_full.log 2>&1; tail -2 gpurun_out/ncu_full.log
fi
