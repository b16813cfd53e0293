#!/bin/bash
# compress/decompress A/B of build_variants (L = 32 on c3 / c2 / c4, L = 8 on c3)
for cfg in "c3_hacc --rel 1e-3" "c2_hurricane --field U --rel 1e-3" "c2_hurricane --field TC --rel 1e-4" "c4_nyx --rel 1e-4"; do
  echo "== $cfg"; timeout 300 python tools/ab.py "$@" --rounds 7 --config $cfg 2>&1 | grep -v "Warning\|SMs 148" | tail -$#
done
echo "== L=8 c3"; timeout 300 python tools/ab.py "$@" --L 8 --rounds 5 --config c3_hacc --rel 1e-3 2>&1 | grep -v "Warning\|SMs 148" | tail -$#
