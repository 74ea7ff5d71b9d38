#!/usr/bin/env bash
# bench lines with the training slowdown of every model config: C2 VGG-16, BERT-large, C3 OPT-1.3B, C4 BLOOM-7B slice
set -u
mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/bench_c2m.json 2> gpurun_out/bench_c2m.err; echo c2 rc=$?
timeout 900 python bench.py --config bert --steps 10 --no-cpu-baseline > gpurun_out/bench_bertm.json 2> gpurun_out/bench_bertm.err; echo bert rc=$?
timeout 1200 python bench.py --config c3 --inflight 4 --steps 6 > gpurun_out/bench_c3m.json 2> gpurun_out/bench_c3m.err; echo c3 rc=$?
timeout 1200 python bench.py --config c4 --emulate-world 8 --steps 6 --no-cpu-baseline > gpurun_out/bench_c4m.json 2> gpurun_out/bench_c4m.err; echo c4 rc=$?
