#!/bin/bash
# A/B timings only (no tests): c2 fields (U / QCLOUD / TC) + c3
for cfg in "c2_hurricane --field U --rel 1e-3" "c2_hurricane --field QCLOUD --rel 1e-2" "c2_hurricane --field TC --rel 1e-4" "c3_hacc --rel 1e-3"; do
  echo "== $cfg"; timeout 300 python tools/ab.py "$@" --rounds 9 --config $cfg 2>&1 | grep -v "Warning\|SMs 148" | tail -$#
done
