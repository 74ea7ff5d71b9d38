#!/usr/bin/env bash
set -u
mkdir -p gpurun_out
o=gpurun_out/graph_exp2.jsonl; : > $o
run() { echo "{\"args\": \"$*\", \"res\": $(timeout -s KILL 400 python tools/slowdown.py opt13 --graphs --iters 60 --runs 1 "$@" 2>/dev/null | tail -1)}" >> $o; }
run --inflight 4 --ring-slices 4
run --inflight 2 --ring-slices 2
echo "{\"args\": \"trace --inflight 4\", \"res\": $(PCC_TRACE=1 timeout -s KILL 400 python tools/slowdown.py opt13 --graphs --iters 40 --runs 1 --inflight 4 2> gpurun_out/graph_trace.txt | tail -1)}" >> $o
grep -E "ckpt|guard|window" gpurun_out/graph_trace.txt | grep -v "persist\|orch:" > gpurun_out/graph_trace_short.txt
cut -c1-300 $o
