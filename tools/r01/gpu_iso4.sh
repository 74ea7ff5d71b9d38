set -u
OUT=gpurun_out; mkdir -p $OUT
timeout 600 python -m pytest tests/test_runtime_gpu.py -q -x -k "paced or file_matches" -p no:cacheprovider 2>&1 | tail -3
for q in 0.5 0.25 2; do
  PCC_D2H_QUANTUM_MIB=$q ISO_KINDS=none,ckpt timeout 600 python tools/slowdown_iso.py 2>&1 | grep ckpt >> $OUT/iso4.jsonl
done
PCC_D2H_GBS=30 PCC_D2H_QUANTUM_MIB=0.5 DIAG_ONLY=0,3 timeout 600 python tools/slowdown_diag.py >> $OUT/diag4.jsonl 2>&1
PCC_D2H_GBS=30 PCC_D2H_QUANTUM_MIB=0.5 DIAG_GRAPHS=1 DIAG_ONLY=0,3 timeout 600 python tools/slowdown_diag.py >> $OUT/diag4.jsonl 2>&1
PCC_PACK_PRIO=low PCC_D2H_GBS=30 PCC_D2H_QUANTUM_MIB=0.5 DIAG_ONLY=0,3 timeout 600 python tools/slowdown_diag.py >> $OUT/diag4.jsonl 2>&1
cut -c1-250 $OUT/iso4.jsonl
python - <<'PY'
import json
for l in open("gpurun_out/diag4.jsonl"):
    if not l.startswith("{"): print(l.strip()[:200]); continue
    d=json.loads(l)
    print(d["variant"].get("pack_ctas"), d["graphs"], d["pack_prio"], d["d2h_gbs"], d["d2h_quantum"], "slow %.2f%%"%d["slowdown_pct"], "base %.2f"%d["iter_ms_no_ckpt"], [round(x,2) for x in d["extra_ms_by_pos"][:4]])
PY
python - <<'PY' > gpurun_out/bloom4.jsonl 2>&1
import json, sys
sys.path.insert(0, ".")
import paper_conf_asplos_strati0k25_b200 as pcc
from tools.slowdown import bloom_slowdown
for kw in (dict(), dict(d2h_gbs=30.0, d2h_quantum=512 << 10)):
    print(json.dumps(bloom_slowdown(pcc, world=8, iters=40, every=10, **kw)), flush=True)
PY
cut -c1-600 gpurun_out/bloom4.jsonl
