#!/usr/bin/env bash
# D2H loop settings: C2 bench K1/value and OPT-1.3B unpaced slowdown
set -u
for cfg in "64 100000 0" "8 4 8" "8 100000 8" "64 100000 2"; do
  set -- $cfg
  export PCC_D2H_PIECE_MIB=$1 PCC_D2H_DEPTH=$2 PCC_D2H_DRAIN=$3
  timeout 600 python bench.py --no-slowdown --no-cpu-baseline --steps 20 2>/dev/null | tail -1 | \
    python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('piece $1 depth $2 drain $3:', round(d['value'],2), 'K1', round(r['k1_ms_per_checkpoint'],3), round(r['frac'],3), 'idle', round(d['snapshot_idle']['ms'],2))"
  timeout 900 python - <<'PY'
import os, sys
sys.path.insert(0, os.getcwd())
import paper_conf_asplos_strati0k25_b200 as pcc
from tools.slowdown import hf_slowdown
r = hf_slowdown(pcc, "opt13", iters=30)
print("   opt13 unpaced", round(r["slowdown_pct"], 2), "its", [round(x) for x in r["iter_ms_ckpt_run"][8:14]], flush=True)
PY
done
