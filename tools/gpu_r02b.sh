#!/usr/bin/env bash
# round 2, second box call: the default bench (C3) with PCIe tx/rx sampled by nvidia-smi dmon,
# the reference arm, the ncu launch list of a short bench, one ncu --set full capture of K1 on
# the C3 state, the TMA-ring staging probe and the K1 compile-time variants.
set -u
mkdir -p gpurun_out
( nvidia-smi dmon -s t -d 1 > gpurun_out/r02b_dmon_pcie.txt 2>&1 & echo $! > /tmp/dmon.pid )
timeout 1500 python bench.py > gpurun_out/r02b_bench.json 2> gpurun_out/r02b_bench.err
echo "bench rc=$?"
kill $(cat /tmp/dmon.pid) 2>/dev/null
timeout 600 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/r02b_ref.json 2> gpurun_out/r02b_ref.err
echo "ref rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/r02b_launches.csv python bench.py --steps 3 --warmup 3 --no-slowdown --no-cpu-baseline \
  > gpurun_out/r02b_bench_under_ncu.log 2>&1
echo "ncu launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_snapshot -s 2 -c 1 \
  -o gpurun_out/r02b_k1_c3 python tools/k1_bench.py --config c3 --reps 3 > gpurun_out/r02b_ncu_full.log 2>&1
echo "ncu full rc=$?"
timeout 300 tools/exp/bulk_copy_probe > gpurun_out/r02b_bulk_probe.jsonl 2>&1
echo "bulk probe rc=$?"
timeout 1200 bash tools/gpu_k1_variants.sh > /dev/null 2>&1
echo "variants rc=$?"
tail -c 1500 gpurun_out/r02b_bench.json
