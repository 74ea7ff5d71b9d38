#!/usr/bin/env bash
# Round evidence refresh: round-end checks (GPU tests, smoke, default bench, launch list, ncu K1)
# + ncu K2 + the C3 / C4-slice bench lines + the reference arm line.
set -u
mkdir -p gpurun_out
bash tools/gpu_round_end.sh
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_snapshot -s 2 -c 1 \
    -o gpurun_out/k2_full -f python tools/k1_bench.py --config c2 --cb 16777216 --reps 4 --unpack > gpurun_out/ncu_full_k2.log 2>&1; echo "ncu k2 rc=$?"
timeout 900 python bench.py --config c3 --inflight 4 --steps 6 --no-cpu-baseline > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err; echo "bench c3 rc=$?"
timeout 900 python bench.py --config c4 --emulate-world 8 --steps 6 --no-cpu-baseline > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err; echo "bench c4 rc=$?"
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; echo "bench ref rc=$?"
timeout 900 python bench.py --config bert --steps 10 --no-cpu-baseline > gpurun_out/bench_bert.json 2> gpurun_out/bench_bert.err; echo "bench bert rc=$?"
