#!/usr/bin/env bash
# bounded D2H queue A/B: (piece MiB, depth) -> C2 bench value / idle snapshot, OPT-1.3B and VGG-16 unpaced slowdown
set -u
for pd in "8 4 8" "8 4 32" "16 4 8" "8 4 0"; do
  set -- $pd
  export PCC_D2H_PIECE_MIB=$1 PCC_D2H_DEPTH=$2 PCC_D2H_DRAIN=$3
  timeout 600 python bench.py --no-slowdown --no-cpu-baseline --steps 20 2>/dev/null | tail -1 | \
    python -c "import json,sys; d=json.loads(sys.stdin.read()); print('piece', $1, 'depth', $2, 'drain', $3, 'c2', round(d['value'],2), round(d['link_roofline']['frac'],3), 'idle', round(d['snapshot_idle']['ms'],2), 'e2e', round(d['e2e']['value'],1))"
  timeout 900 python - <<'PY'
import json, os, sys
sys.path.insert(0, os.getcwd())
import paper_conf_asplos_strati0k25_b200 as pcc
from tools.slowdown import hf_slowdown, vgg16_slowdown
r = hf_slowdown(pcc, "opt13", iters=40)
v = vgg16_slowdown(pcc, iters=60, every=10)
print("   opt13 unpaced", round(r["slowdown_pct"], 2), "snap", round(r["contended"]["snapshot_ms"], 1),
      "its", [round(x) for x in r["iter_ms_ckpt_run"][8:13]], "| vgg unpaced", round(v["slowdown_pct"], 2),
      "snap", round(v["contended"]["snapshot_ms"], 1), flush=True)
PY
done
