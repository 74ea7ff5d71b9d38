set -u
OUT=gpurun_out; mkdir -p $OUT
DIAG_GRAPHS=1 DIAG_ONLY=0,2,3,7 timeout 600 python tools/slowdown_diag.py >> $OUT/diag2.jsonl 2>&1
PCC_PACK_PRIO=low DIAG_GRAPHS=1 DIAG_ONLY=0,3,7 timeout 600 python tools/slowdown_diag.py >> $OUT/diag2.jsonl 2>&1
PCC_D2H_GBS=30 PCC_D2H_QUANTUM_MIB=2 DIAG_GRAPHS=1 DIAG_ONLY=0,3 timeout 600 python tools/slowdown_diag.py >> $OUT/diag2.jsonl 2>&1
PCC_D2H_GBS=30 PCC_D2H_QUANTUM_MIB=1 DIAG_GRAPHS=0 DIAG_ONLY=0 timeout 600 python tools/slowdown_diag.py >> $OUT/diag2.jsonl 2>&1
python - <<'PY'
import json
for l in open("gpurun_out/diag2.jsonl"):
    if not l.startswith("{"): print(l.strip()[:200]); continue
    d=json.loads(l)
    print(d["variant"], d["pack_prio"], d["pace"], "slow %.2f%%"%d["slowdown_pct"], "base %.2f"%d["iter_ms_no_ckpt"], d["extra_ms_by_pos"][:4])
PY
