#!/usr/bin/env bash
# same-box A/B: K1 window rule half ring (current) vs quarter ring (build/quarter), OPT-1.3B graphs (bench setup) and eager
set -u
mkdir -p gpurun_out
o=gpurun_out/r02wab.jsonl; : > $o
run() { v=$1; shift; lib=""; [ $v = quarter ] && lib=build/quarter/libpccheck.so; echo "{\"v\": \"$v\", \"args\": \"$*\", \"res\": $(PCC_LIB=$lib timeout -s KILL 900 python tools/slowdown.py opt13 --iters 200 --runs 2 --inflight 4 --pace auto --link-gbs 57 "$@" 2>/dev/null | tail -1)}" >> $o; }
for v in half quarter half quarter; do run $v --graphs --host-lead 2 --no-upfront; done
for v in half quarter; do run $v; done
python - <<'PY'
import json
for l in open('gpurun_out/r02wab.jsonl'):
    d=json.loads(l); r=d['res']
    print(d['v'], d['args'][:20], '| slow %.2f%%'%r['slowdown_pct'], [round(x,2) for x in r['slowdown_pct_runs']], '| k1', round(r['contended']['k1_busy_ms'],2), 'pack', round(r['contended']['pack_span_ms'],2), '| pos', [round(x,1) for x in r['extra_ms_by_pos']])
PY
