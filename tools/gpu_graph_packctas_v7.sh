#!/usr/bin/env bash
# OPT-1.3B as CUDA graphs (the bench's `slowdown` setup: tuner's graph pace, host <= 2 ahead), K1 v7 with its
# grid capped (pack_ctas): does a K1 on fewer SMs interleave better with the training graph? 200 iterations x 2 runs
set -u
mkdir -p gpurun_out
o=gpurun_out/r02t_graph_packctas.jsonl; : > $o
run() { echo "{\"args\": \"$*\", \"res\": $(timeout -s KILL 900 python tools/slowdown.py opt13 --graphs --iters 200 --runs 2 --inflight 4 --host-lead 2 --no-upfront --pace auto --link-gbs 57 "$@" 2>/dev/null | tail -1)}" >> $o; }
run --pack-ctas 0
run --pack-ctas 74
run --pack-ctas 37
run --pack-ctas 16
python - <<'PY'
import json
for l in open('gpurun_out/r02t_graph_packctas.jsonl'):
    d=json.loads(l); r=d['res']
    print(d['args'], '| slow %.2f%%'%r['slowdown_pct'], r.get('slowdown_pct_runs'), '| k1', round(r['contended']['k1_busy_ms'],2), '| pos', [round(x,1) for x in r['extra_ms_by_pos']])
PY
