#!/usr/bin/env bash
# K1 against its own copy-only ceiling (same kernel, CRC compiled out: timing only)
set -u
for v in paper_conf_asplos_strati0k25_b200 build/va_nocrc paper_conf_asplos_strati0k25_b200 build/va_nocrc; do
  echo "== $v"
  for c in "c2 --cb 16777216" "c3"; do PCC_LIB=$v/libpccheck.so python tools/k1_bench.py --config $c --reps 6; done
done
