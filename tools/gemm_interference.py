"""DESIGN §11 item 4: does the checkpoint's D2H burst slow GPU-bound work that has no host
launch pressure?  A bf16 GEMM loop (64 x 8192^3 per 'iteration', ~40 ms, 64 launches) with a
checkpoint of a 15.0 GB synthetic state every 10 iterations, against the same loop without.
GEMMs slowed as much as OPT-1.3B's eager step -> GPU-side interference; not slowed -> the
eager step's host path."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_asplos_strati0k25_b200 as pcc  # noqa: E402

dev = torch.device("cuda", 0)
g = torch.Generator(device=dev).manual_seed(0)
state = [torch.randint(-2**31, 2**31 - 1, (64 << 20,), dtype=torch.int32, device=dev, generator=g)
         for _ in range(56)]  # 56 x 256 MiB = 15.0 GB
a = torch.randn(8192, 8192, device=dev, dtype=torch.bfloat16)
b = torch.randn(8192, 8192, device=dev, dtype=torch.bfloat16)
c = torch.empty(8192, 8192, device=dev, dtype=torch.bfloat16)
stream = torch.cuda.current_stream()


def step():
    for _ in range(64):
        torch.matmul(a, b, out=c)


path = f"/dev/shm/pcc_gemm_{os.getpid()}.pcc"
ck = pcc.PCCheck(path, chunk_bytes=64 << 20, max_inflight=2, flags=pcc.MAPFILE, staging_bytes=8 * (64 << 20),
                 device=0)
ck.register(state)


def loop(n, checkpoint, it0):
    evs = [torch.cuda.Event(enable_timing=True) for _ in range(n + 1)]
    evs[0].record(stream)
    hs = []
    for i in range(1, n + 1):
        step()
        if checkpoint and i % 10 == 0:
            hs.append(ck.checkpoint(it0 + i, stream))
        evs[i].record(stream)
    evs[-1].synchronize()
    for h in hs:
        ck.wait(h)
    return [evs[i - 1].elapsed_time(evs[i]) for i in range(1, n + 1)]


loop(5, False, 0)
loop(12, True, 100)  # warm the library path
base = loop(40, False, 0)
withck = loop(40, True, 1000)
ck.drain()
ck.close()
os.unlink(path)
mb, mc = sum(base) / len(base), sum(withck) / len(withck)
print(json.dumps({"iter_ms_no_ckpt": mb, "iter_ms_ckpt": mc, "slowdown_pct": 100 * (mc / mb - 1),
                  "tflops_no_ckpt": 64 * 2 * 8192**3 / (mb * 1e-3) / 1e12,
                  "iters_ms_ckpt": [round(x, 2) for x in withck[:20]],
                  "state_bytes": 56 * (256 << 20)}))
