set -u
python - <<'PY'
import torch
for nb in (1106860352, 15789098512):
    a = torch.empty(nb, dtype=torch.uint8, device="cuda"); b = torch.empty_like(a)
    best = 1e9
    for i in range(6):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); b.copy_(a); e1.record(); e1.synchronize()
        if i: best = min(best, e0.elapsed_time(e1))
    print({"torch_copy_bytes": nb, "ms": best, "gbs_rw": 2 * nb / best / 1e6})
    del a, b
PY
bash tools/gpu_ab.sh 2>&1 | grep -v Warn | sed 's/"finalize_ms.*k1_gbs_algorithmic"/ gbs/'
