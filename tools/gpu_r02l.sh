#!/usr/bin/env bash
# v7: new kernel tests, eager-launch penalty probe, the default bench line, K1 --set full on C3 and C2 (16 MiB), bench launch list
set -u
mkdir -p gpurun_out
o=gpurun_out/r02l.log; : > $o
timeout -s KILL 900 python -m pytest tests/test_kernels_gpu.py -m gpu -q -p no:cacheprovider >> $o 2>&1; echo "kernels rc=$?" >> $o
timeout -s KILL 600 python tools/exp/launch_probe2.py > gpurun_out/r02l_launch_probe2.jsonl 2>&1; echo "probe rc=$?" >> $o
timeout -s KILL 1500 python bench.py > gpurun_out/r02l_bench_c3.json 2> gpurun_out/r02l_bench_c3.err; echo "bench rc=$?" >> $o
timeout -s KILL 900 ncu --set full --import-source on --clock-control none -k regex:k_snap_tma --launch-skip 2 -c 1 -o gpurun_out/r02l_k1_c3 \
  python tools/k1_bench.py --config c3 --reps 3 > gpurun_out/r02l_ncu_c3.log 2>&1; echo "ncu c3 rc=$?" >> $o
timeout -s KILL 600 ncu --set full --import-source on --clock-control none -k regex:k_snap_tma --launch-skip 2 -c 1 -o gpurun_out/r02l_k1_c2_16m \
  python tools/k1_bench.py --config c2 --cb 16777216 --reps 3 > gpurun_out/r02l_ncu_c2.log 2>&1; echo "ncu c2 rc=$?" >> $o
timeout -s KILL 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_snap|k_fold|k_chunk" -c 300 --csv \
  --log-file gpurun_out/r02l_launches.csv python bench.py --steps 5 --warmup 3 --no-slowdown --no-cpu-baseline \
  > gpurun_out/r02l_bench_under_ncu.log 2>&1; echo "ncu launches rc=$?" >> $o
cat $o
