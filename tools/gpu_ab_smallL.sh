for L in 8 16; do for cfg in "c2_hurricane --field U --rel 1e-3" "c3_hacc --rel 1e-3" "c2_hurricane --field TC --rel 1e-4"; do
  echo "== L=$L $cfg"; timeout 300 python tools/ab.py ${LIBS:-build_variants/new.so build_variants/old3.so} --L $L --rounds 7 --config $cfg 2>&1 | grep -v Warning | tail -3
done; done
