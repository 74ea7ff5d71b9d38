#!/usr/bin/env bash
# graph-mode D2H pace x quantum on ONE box (OPT-1.3B, 200 iterations x 1 run each, host <= 2 ahead)
set -u
mkdir -p gpurun_out
o=gpurun_out/graph_exp6.jsonl; : > $o
run() { echo "{\"args\": \"$*\", \"res\": $(timeout -s KILL 600 python tools/slowdown.py opt13 --graphs --iters 200 --runs 1 --inflight 4 --host-lead 2 --no-upfront "$@" 2>/dev/null | tail -1)}" >> $o; }
for q in 512 1024 4096; do for p in 35 45; do run --pace $p --quantum-kib $q; done; done
run --pace 0
run --pace 40 --quantum-kib 512
python - <<'PY'
import json
for l in open('gpurun_out/graph_exp6.jsonl'):
    d=json.loads(l); r=d['res']
    print(d['args'][-30:], '| slow %.2f%%'%r['slowdown_pct'], '| snap', round(r['contended']['snapshot_ms']), 'deliv', r.get('pace_delivered_frac'), '| pos', [round(x,1) for x in r['extra_ms_by_pos']])
PY
