#!/usr/bin/env bash
# A/B the K1 register-pipeline variants (build/v<batch>_<minblocks>/libpccheck.so)
set -u
for v in build/v*/; do
  echo "== $v"
  PCC_LIB=$v/libpccheck.so python tools/k1_bench.py --config c2 --reps 8
  PCC_LIB=$v/libpccheck.so python tools/k1_bench.py --config c2 --reps 8 --unpack; PCC_LIB=$v/libpccheck.so python tools/k1_bench.py --config c3 --reps 4
done
timeout 300 python -m pytest tests/test_kernels_gpu.py -q -x -p no:cacheprovider 2>&1 | tail -2
