#!/usr/bin/env bash
# kRun A/B: parity of each variant's K1/K2 against the oracle, then K1/K2 timings
set -u
for v in paper_conf_asplos_strati0k25_b200 build/va_run*; do
  echo "== $v"
  PCC_LIB=$v/libpccheck.so timeout 600 python -m pytest tests/test_kernels_gpu.py -q -x -p no:cacheprovider 2>&1 | tail -1
  for i in 1 2; do
    PCC_LIB=$v/libpccheck.so python tools/k1_bench.py --config c2 --cb 16777216 --reps 8
  done
  PCC_LIB=$v/libpccheck.so python tools/k1_bench.py --config c3 --reps 4
  PCC_LIB=$v/libpccheck.so python tools/k1_bench.py --config c2 --cb 16777216 --reps 6 --unpack
done
