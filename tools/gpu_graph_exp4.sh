#!/usr/bin/env bash
set -u
mkdir -p gpurun_out
o=gpurun_out/graph_exp4.jsonl; : > $o
run() { echo "{\"args\": \"$*\", \"res\": $(timeout -s KILL 600 python tools/slowdown.py opt13 --graphs --iters 200 --runs 1 --inflight 4 "$@" 2>/dev/null | tail -1)}" >> $o; }
run
run --pack-ctas 74
run --pack-ctas 111
run --pack-ctas 37
python - <<'PY'
import json
for l in open('gpurun_out/graph_exp4.jsonl'):
    d=json.loads(l); r=d['res']
    print(d['args'], '| slow %.2f%%'%r['slowdown_pct'], '| k1', r['contended']['k1_busy_ms'], '| snap', r['contended']['snapshot_ms'], '| pos', [round(x,1) for x in r['extra_ms_by_pos']])
PY
