#!/usr/bin/env bash
set -u
mkdir -p gpurun_out
o=gpurun_out/graph_exp5.jsonl; : > $o
run() { echo "{\"args\": \"$*\", \"res\": $(timeout -s KILL 600 python tools/slowdown.py opt13 --graphs --iters 200 --runs 1 --inflight 4 "$@" 2>/dev/null | tail -1)}" >> $o; }
run --host-lead 2 --no-upfront
run --host-lead 2 --no-upfront --pace 30
run --host-lead 2 --no-upfront --pace 40
run --host-lead 2 --no-upfront --pace 30 --quantum-kib 4096
run --host-lead 2
python - <<'PY'
import json
for l in open('gpurun_out/graph_exp5.jsonl'):
    d=json.loads(l); r=d['res']
    print(d['args'], '| slow %.2f%%'%r['slowdown_pct'], '| k1', r['contended']['k1_busy_ms'], '| snap', r['contended']['snapshot_ms'], 'deliv', r.get('pace_delivered_frac'), '| pos', [round(x,1) for x in r['extra_ms_by_pos']])
PY
