#!/bin/bash
# quick GPU iteration: parity (not slow) + A/B timings of build_variants/*.so given as args
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -4
for cfg in "c3_hacc --rel 1e-3" "c4_nyx --rel 1e-4" "c2_hurricane --field U --rel 1e-3" "c2_hurricane --field TC --rel 1e-4"; do
  echo "== $cfg"; timeout 300 python tools/ab.py "$@" --rounds 7 --config $cfg 2>&1 | grep -v Warning | tail -$(( $# + 2 ))
done
