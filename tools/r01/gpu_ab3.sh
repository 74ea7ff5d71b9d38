#!/usr/bin/env bash
# default vs build/va_*: kernel parity, K1/finalize timings (c2, c3), K2; finalize launch list
set -u
mkdir -p gpurun_out
for v in paper_conf_asplos_strati0k25_b200 build/va_*; do
  echo "== $v"
  PCC_LIB=$v/libpccheck.so timeout 600 python -m pytest tests/test_kernels_gpu.py tests/test_runtime_gpu.py -q -x -p no:cacheprovider 2>&1 | tail -1
  for c in "c2 --cb 16777216" "c2 --cb 16777216" "c3" "c3 --cb 4194304"; do PCC_LIB=$v/libpccheck.so python tools/k1_bench.py --config $c --reps 6; done
  PCC_LIB=$v/libpccheck.so timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$(basename $v).csv \
    python tools/k1_bench.py --config c2 --cb 16777216 --reps 3 > /dev/null 2>&1
  PCC_LIB=$v/libpccheck.so timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_k2_$(basename $v).csv \
    python tools/k1_bench.py --config c2 --cb 16777216 --reps 3 --unpack > /dev/null 2>&1
done
