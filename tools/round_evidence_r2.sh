#!/bin/bash
# Round-2 evidence on one B200 (run through gpurun): the default bench line
# (c3 HACC headline + secondary configs), the ncu launch list of a short
# headline run, and one ncu --set full capture of the headline step's three
# kernels (range, compress, decompress on the 1.12 GB field).
set -x
TAG=${1:-r2}
python bench.py > gpurun_out/bench_${TAG}.json 2> gpurun_out/bench_${TAG}.err; tail -2 gpurun_out/bench_${TAG}.err
Q="--no-e2e --no-cpu-baseline --no-secondary --no-variants --no-datasets"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}.csv python bench.py --steps 2 --warmup 1 $Q > gpurun_out/ncu_launch_${TAG}.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"range_kernel|compress_kernel|decompress_kernel" -s 9 -c 3 -o gpurun_out/prof_${TAG} python bench.py --steps 1 --warmup 1 $Q > gpurun_out/ncu_full_${TAG}.log 2>&1
tail -2 gpurun_out/ncu_full_${TAG}.log
