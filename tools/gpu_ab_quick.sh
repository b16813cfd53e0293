#!/bin/bash
# A/B timings only (no tests) of build_variants/*.so given as args, c3 + c2 TC
for cfg in "c3_hacc --rel 1e-3" "c2_hurricane --field TC --rel 1e-4"; do
  echo "== $cfg"; timeout 300 python tools/ab.py "$@" --rounds 7 --config $cfg 2>&1 | grep -v "Warning\|SMs 148" | tail -$#
done
