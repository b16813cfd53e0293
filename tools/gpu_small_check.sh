#!/bin/bash
# L = 8 / 16: parity (block-length tests, grid sweep, stress build), then A/B timings
timeout 900 python -m pytest tests/test_gpu_blocklen.py tests/test_gpu_stress.py -x -q -k "8 or 16 or interleaved or sweep or stress_build" 2>&1 | tail -5
bash tools/gpu_ab_smallL.sh "$@"
