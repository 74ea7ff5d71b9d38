#!/usr/bin/env bash
# K1's stream priority (PCC_PACK_PRIO: high = default, low) vs OPT-1.3B training slowdown, graphs (bench `slowdown` setup) and eager
set -u
mkdir -p gpurun_out
o=gpurun_out/r02y_packprio.jsonl; : > $o
run() { p=$1; shift; echo "{\"prio\": \"$p\", \"args\": \"$*\", \"res\": $(PCC_PACK_PRIO=$p timeout -s KILL 900 python tools/slowdown.py opt13 --iters 200 --runs 2 --inflight 4 --pace auto --link-gbs 57 "$@" 2>/dev/null | tail -1)}" >> $o; }
for p in high low high low; do run $p --graphs --host-lead 2 --no-upfront; done
for p in high low; do run $p; done
python - <<'PY'
import json
for l in open('gpurun_out/r02y_packprio.jsonl'):
    d=json.loads(l); r=d['res']
    print(d['prio'], d['args'][:30], '| slow %.2f%%'%r['slowdown_pct'], r.get('slowdown_pct_runs'), '| k1', round(r['contended']['k1_busy_ms'],2), 'pack', round(r['contended']['pack_span_ms'],2), '| pos', [round(x,1) for x in r['extra_ms_by_pos']], 'guard', r.get('host_guard_ms_max'))
PY
