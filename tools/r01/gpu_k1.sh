#!/usr/bin/env bash
# quick K1/K2 iteration: parity tests + microbench + one ncu capture of each
set -u
OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu.log 2>&1; tail -3 $OUT/pytest_gpu.log
python tools/k1_bench.py --config c2 --reps 6
python tools/k1_bench.py --config c2 --reps 6 --unpack
python tools/k1_bench.py --config c3 --reps 3
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_snapshot -s 2 -c 1 -o $OUT/k1_full -f python tools/k1_bench.py --config c2 --cb 16777216 --reps 4 > $OUT/ncu_full.log 2>&1; echo "ncu rc=$?"
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_snapshot -s 2 -c 1 -o $OUT/k2_full -f python tools/k1_bench.py --config c2 --reps 4 --unpack > $OUT/ncu_full_k2.log 2>&1; echo "ncu k2 rc=$?"
