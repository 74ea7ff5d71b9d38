set -u
mkdir -p gpurun_out
OUT=gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $OUT/pytest_gpu.log
timeout 600 python tools/slowdown_diag.py > $OUT/diag_hi.jsonl 2>&1; echo "diag rc=$?"
PCC_PACK_PRIO=low DIAG_ONLY=0,2 timeout 600 python tools/slowdown_diag.py > $OUT/diag_lo.jsonl 2>&1; echo "diag lo rc=$?"
PCC_PACK_PRIO=default DIAG_ONLY=0 timeout 600 python tools/slowdown_diag.py > $OUT/diag_def.jsonl 2>&1; echo "diag def rc=$?"
