#!/usr/bin/env bash
# K1 time in the back-to-back bench vs the D2H copy loop settings (same box)
set -u
for cfg in "64 100000 0" "8 4 8" "64 100000 0" "8 4 8" "16 4 8" "32 4 4"; do
  set -- $cfg
  PCC_D2H_PIECE_MIB=$1 PCC_D2H_DEPTH=$2 PCC_D2H_DRAIN=$3 timeout 600 python bench.py --no-slowdown --no-cpu-baseline --steps 20 2>/dev/null | tail -1 | \
    python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('piece $1 depth $2 drain $3:', round(d['value'],2), 'K1', round(r['k1_ms_per_checkpoint'],3), round(r['frac'],3), 'idle', round(d['snapshot_idle']['ms'],2))"
done
