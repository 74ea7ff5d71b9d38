#!/usr/bin/env bash
# eager OPT-1.3B, K1 v7: finer pace x copy-size grid around the tuner's eager point (200 iterations x 1 run each)
set -u
mkdir -p gpurun_out
o=gpurun_out/r02p_eager_pace2.jsonl; : > $o
run() { echo "{\"args\": \"$*\", \"res\": $(timeout -s KILL 600 python tools/slowdown.py opt13 --iters 200 --runs 1 --inflight 4 "$@" 2>/dev/null | tail -1)}" >> $o; }
for q in 1024 2048 4096; do
  for p in 36 40 44; do run --pace $p --quantum-kib $q; done
done
run --pace 40 --quantum-kib 512
run --pace 40 --quantum-kib 8192
python - <<'PY'
import json
for l in open('gpurun_out/r02p_eager_pace2.jsonl'):
    d=json.loads(l); r=d['res']
    print(d['args'][-30:], '| slow %.2f%%'%r['slowdown_pct'], '| snap', round(r['contended']['snapshot_ms']), 'deliv', r.get('pace_delivered_frac'), '| pos', [round(x,1) for x in r['extra_ms_by_pos']])
PY
