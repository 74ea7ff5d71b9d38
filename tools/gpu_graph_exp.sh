#!/usr/bin/env bash
# OPT-1.3B as 2 CUDA graphs, checkpoint every 10: host lead / ring size / N (60 iterations x 1 run)
set -u
mkdir -p gpurun_out
o=gpurun_out/graph_exp.jsonl; : > $o
run() { echo "{\"args\": \"$*\", \"res\": $(timeout -s KILL 400 python tools/slowdown.py opt13 --graphs --iters 60 --runs 1 "$@" 2>/dev/null | tail -1)}" >> $o; }
run --inflight 4
run --inflight 4 --host-lead 2
run --inflight 4 --ring-slices 2
run --inflight 2
run --inflight 4 --ring-slices 2 --host-lead 2
cat $o | cut -c1-600
