#!/bin/bash
# A/B timings only (no tests): c3 / c4 at REL 1e-2 (small F), c4 1e-3, c5 RTM set 1e-3
for cfg in "c3_hacc --rel 1e-2" "c4_nyx --rel 1e-2" "c4_nyx --rel 1e-3" "c5_rtm --rel 1e-3" "c3_hacc --rel 1e-3"; do
  echo "== $cfg"; timeout 300 python tools/ab.py "$@" --rounds 7 --config $cfg 2>&1 | grep -v "Warning\|SMs 148" | tail -$#
done
