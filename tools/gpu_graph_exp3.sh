#!/usr/bin/env bash
set -u
mkdir -p gpurun_out
timeout -s KILL 600 python -m pytest tests/test_runtime_gpu.py -q -p no:cacheprovider > gpurun_out/r02d_runtime.log 2>&1; echo "runtime tests rc=$?"; tail -3 gpurun_out/r02d_runtime.log
o=gpurun_out/graph_exp3.jsonl; : > $o
run() { echo "{\"args\": \"$*\", \"res\": $(timeout -s KILL 400 python tools/slowdown.py opt13 --graphs --iters 60 --runs 1 "$@" 2>/dev/null | tail -1)}" >> $o; }
run --inflight 4
run --inflight 4 --host-lead 2
run --inflight 2
python - <<'PY'
import json
for l in open('gpurun_out/graph_exp3.jsonl'):
    d=json.loads(l); r=d['res']
    print(d['args'], '| slow %.2f%%'%r['slowdown_pct'], '| guard', r.get('host_guard_ms'), r.get('host_guard_ms_max'), '| call', r['host_ckpt_call_ms'], r['host_ckpt_call_ms_max'], '| snap', r['contended']['snapshot_ms'], '| pos', [round(x,1) for x in r['extra_ms_by_pos']])
PY
