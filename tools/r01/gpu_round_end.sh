#!/usr/bin/env bash
# Everything the round-end driver checks, plus the evidence: GPU tests, smoke, default bench,
# the bench's ncu launch list and one ncu --set full capture of K1 in the bench configuration.
set -u
OUT=gpurun_out; mkdir -p $OUT
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $OUT/launches.csv \
    python bench.py --steps 5 --warmup 3 --no-slowdown --no-cpu-baseline > $OUT/bench_under_ncu.log 2>&1; echo "ncu list rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_snapshot -s 2 -c 1 \
    -o $OUT/k1_full -f python tools/k1_bench.py --config c2 --cb 16777216 --reps 4 > $OUT/ncu_full.log 2>&1; echo "ncu full rc=$?"
