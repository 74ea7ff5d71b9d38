#!/usr/bin/env bash
# Bench lines for the larger BASELINE configs at the current code (1 x B200): C3 OPT-1.3B with
# N = 4 in flight, C4 BLOOM-7b1 and C5 OPT-2.7B as rank 0 of 8 (the 1/8 slice each rank packs).
set -u
OUT=gpurun_out; mkdir -p $OUT
timeout 900 python bench.py --config c3 --inflight 4 --steps 6 --no-cpu-baseline > $OUT/bench_c3.json 2> $OUT/bench_c3.err; echo "bench c3 rc=$?"
timeout 900 python bench.py --config c4 --emulate-world 8 --steps 6 --no-cpu-baseline > $OUT/bench_c4.json 2> $OUT/bench_c4.err; echo "bench c4 rc=$?"
timeout 600 python bench.py --config c5 --emulate-world 8 --steps 10 --no-cpu-baseline --no-slowdown > $OUT/bench_c5.json 2> $OUT/bench_c5.err; echo "bench c5 rc=$?"
