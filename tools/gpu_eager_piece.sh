#!/usr/bin/env bash
# eager OPT-1.3B, unpaced D2H in small pieces (PCC_D2H_PIECE_MIB) x queue drain interval (PCC_D2H_DRAIN_MIB),
# vs the default 64 MiB pieces and the tuner's pace (200 iterations x 1 run each)
set -u
mkdir -p gpurun_out
o=gpurun_out/r02e2_eager_piece.jsonl; : > $o
run() { tag=$1; shift; echo "{\"tag\": \"$tag\", \"res\": $(env "$@" timeout -s KILL 600 python tools/slowdown.py opt13 --iters 200 --runs 1 --inflight 4 --pace 0 2>/dev/null | tail -1)}" >> $o; }
run piece64_drain128 PCC_D2H_PIECE_MIB=64 PCC_D2H_DRAIN_MIB=128
run piece1_drain128 PCC_D2H_PIECE_MIB=1 PCC_D2H_DRAIN_MIB=128
run piece1_drain16 PCC_D2H_PIECE_MIB=1 PCC_D2H_DRAIN_MIB=16
run piece1_drain4 PCC_D2H_PIECE_MIB=1 PCC_D2H_DRAIN_MIB=4
run piece4_drain32 PCC_D2H_PIECE_MIB=4 PCC_D2H_DRAIN_MIB=32
run piece2_drain16 PCC_D2H_PIECE_MIB=2 PCC_D2H_DRAIN_MIB=16
echo "{\"tag\": \"paced_auto\", \"res\": $(timeout -s KILL 600 python tools/slowdown.py opt13 --iters 200 --runs 1 --inflight 4 --pace auto --link-gbs 57 2>/dev/null | tail -1)}" >> $o
python - <<'PY'
import json
for l in open('gpurun_out/r02e2_eager_piece.jsonl'):
    d=json.loads(l); r=d['res']
    print(d['tag'], '| slow %.2f%%'%r['slowdown_pct'], '| snap', round(r['contended']['snapshot_ms']), 'gbs', round(r['contended']['gbs'],1), '| pos', [round(x,1) for x in r['extra_ms_by_pos']])
PY
