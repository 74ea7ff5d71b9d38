#!/usr/bin/env bash
# A/B K1 variants (build/va*/libpccheck.so) against the default build
set -u
for v in paper_conf_asplos_strati0k25_b200 build/va*; do
  echo "== $v"
  PCC_LIB=$v/libpccheck.so python tools/k1_bench.py --config c2 --cb 16777216 --reps 8
  PCC_LIB=$v/libpccheck.so python tools/k1_bench.py --config c3 --reps 4
  [ -n "${AB_UNPACK:-}" ] && PCC_LIB=$v/libpccheck.so python tools/k1_bench.py --config c2 --cb 16777216 --reps 6 --unpack
done
