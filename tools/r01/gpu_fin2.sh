#!/usr/bin/env bash
# two-kernel finalize: all GPU tests, K1/finalize timings, finalize launch list
set -u
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
for c in "c2 --cb 16777216" "c3" "c1 --cb 4194304" "c3 --cb 4194304"; do python tools/k1_bench.py --config $c --reps 6; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/fin_launches.csv \
  python tools/k1_bench.py --config c2 --cb 16777216 --reps 3 > /dev/null 2>&1; echo "ncu rc=$?"
