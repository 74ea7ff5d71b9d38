#!/usr/bin/env bash
# the N > 1 bench path on ONE GPU: 2 self-spawned ranks sharing cuda:0 over gloo (--share-gpu),
# C3 1/2 slices, the collective commit, OPT-1.3B under DDP with the checkpoint every 10
set -u
mkdir -p gpurun_out
timeout -s KILL 1500 python bench.py --gpus 2 --share-gpu --collectives torch --steps 5 --warmup 3 \
  --slowdown-iters 40 --slowdown-runs 1 > gpurun_out/r02_share2.json 2> gpurun_out/r02_share2.err
echo "rc=$?"
tail -c 2500 gpurun_out/r02_share2.json; tail -5 gpurun_out/r02_share2.err
timeout 1500 compute-sanitizer --tool memcheck --print-limit 20 python -m pytest tests/test_kernels_gpu.py tests/test_runtime_gpu.py -q -p no:cacheprovider \
    -k "rfc or misaligned or partial or host_mapped or roundtrip or file_matches_oracle or n_in_flight or small_ring or failed_k1" \
    > gpurun_out/r02_sanitizer_memcheck.txt 2>&1; echo "memcheck rc=$?"; tail -3 gpurun_out/r02_sanitizer_memcheck.txt
