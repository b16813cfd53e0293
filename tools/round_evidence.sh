#!/bin/bash
# Round-end evidence on one B200 (run through gpurun): bench line, ncu launch
# list of a short bench run, one ncu --set full capture of the three kernels
# (job 2 of the bench = Hurricane U at REL 1e-3).
set -x
TAG=${1:-r01}
python bench.py > gpurun_out/bench_${TAG}.json 2> gpurun_out/bench_${TAG}.err; tail -2 gpurun_out/bench_${TAG}.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --no-large > gpurun_out/ncu_launch_${TAG}.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"range_kernel|compress_kernel|decompress_kernel" -s 3 -c 3 -o gpurun_out/prof_${TAG} python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-large > gpurun_out/ncu_full_${TAG}.log 2>&1
tail -2 gpurun_out/ncu_full_${TAG}.log
