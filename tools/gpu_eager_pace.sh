#!/usr/bin/env bash
# eager OPT-1.3B with the (now rate-delivering) pacer: pace x quantum (200 iterations x 1 run each)
set -u
mkdir -p gpurun_out
o=gpurun_out/eager_pace.jsonl; : > $o
run() { echo "{\"args\": \"$*\", \"res\": $(timeout -s KILL 600 python tools/slowdown.py opt13 --iters 200 --runs 1 --inflight 4 "$@" 2>/dev/null | tail -1)}" >> $o; }
run --pace 0
run --pace 40 --quantum-kib 1024
run --pace 50 --quantum-kib 1024
run --pace 40 --quantum-kib 256
run --pace 50 --quantum-kib 4096
python - <<'PY'
import json
for l in open('gpurun_out/eager_pace.jsonl'):
    d=json.loads(l); r=d['res']
    print(d['args'][-30:], '| slow %.2f%%'%r['slowdown_pct'], '| snap', round(r['contended']['snapshot_ms']), 'deliv', r.get('pace_delivered_frac'), '| pos', [round(x,1) for x in r['extra_ms_by_pos']])
PY
