#!/bin/bash
# L = 8 / 16 A/B (compress / decompress kernels) on Hurricane U and HACC
for L in 8 16; do for cfg in "c2_hurricane --field U --rel 1e-3" "c3_hacc --rel 1e-3"; do
  echo "== L=$L $cfg"; timeout 300 python tools/ab.py "$@" --L $L --rounds 7 --config $cfg 2>&1 | grep -v "Warning\|SMs 148" | tail -$#
done; done
