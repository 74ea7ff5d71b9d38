#!/usr/bin/env bash
# One gpurun call: GPU tests, bench, ncu launch list of the bench, ncu --set full of K1.
set -u
mkdir -p gpurun_out
OUT=gpurun_out
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
tail -3 $OUT/pytest_gpu.log
timeout 600 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"
tail -1 $OUT/bench.json | cut -c1-600
if [ "${NCU:-1}" = "1" ]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $OUT/launches.csv \
      python bench.py --steps 5 --warmup 3 --no-slowdown --no-cpu-baseline > $OUT/bench_under_ncu.log 2>&1; echo "ncu list rc=$?"
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_snapshot -s 2 -c 1 \
      -o $OUT/k1_full -f python tools/k1_bench.py --config c2 --reps 4 > $OUT/ncu_full.log 2>&1; echo "ncu full rc=$?"
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_snapshot -s 2 -c 1 \
      -o $OUT/k2_full -f python tools/k1_bench.py --config c2 --reps 4 --unpack > $OUT/ncu_full_k2.log 2>&1; echo "ncu k2 rc=$?"
fi
python tools/k1_bench.py --config c2 --reps 6
python tools/k1_bench.py --config c2 --reps 6 --unpack
