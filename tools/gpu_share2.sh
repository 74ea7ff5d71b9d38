#!/usr/bin/env bash
# the N > 1 bench path on ONE GPU: 2 self-spawned ranks sharing cuda:0 over gloo (--share-gpu),
# C3 1/2 slices, the collective commit, OPT-1.3B under DDP with the checkpoint every 10
set -u
mkdir -p gpurun_out
timeout -s KILL 1500 python bench.py --gpus 2 --share-gpu --collectives torch --steps 5 --warmup 3 \
  --slowdown-iters 40 --slowdown-runs 1 > gpurun_out/r02_share2.json 2> gpurun_out/r02_share2.err
echo "rc=$?"
tail -c 2500 gpurun_out/r02_share2.json; tail -5 gpurun_out/r02_share2.err
