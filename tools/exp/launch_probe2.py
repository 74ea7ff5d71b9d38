"""Where does the eager launch penalty under a D2H burst come from (OPT-1.3B eager)?
Alone and under two kinds of 8 GiB device -> pinned-host burst, measures
  cpu_ms      a pure-Python CPU loop (no CUDA at all): host memory / CPU contention
  host_ms     host time of 3000 eager x.add_ launches (perf_counter around the Python loop)
  gpu_ms      device time of the same 3000 kernels (CUDA events)
Bursts: "ce"    = torch copy_ device -> pinned in 64 MiB pieces (copy engine);
        "sm"    = one asynchronous pcc_checkpoint in ZEROCOPY | MAPFILE mode: K1 (v7) bulk-stores the
                  8 GiB straight into the registered /dev/shm file mapping from the SMs
                  (Variant A's path), all SMs;
        "sm16"  = the same with K1's grid capped at 16 CTAs (pack_ctas).
Not part of the product path.""" 
import json
import os
import sys
import threading
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import paper_conf_asplos_strati0k25_b200 as pcc  # noqa: E402

dev = torch.device("cuda", 0)
x = torch.zeros(1024, device=dev)
N = 8 << 30
src = torch.randint(0, 255, (N,), dtype=torch.uint8, device=dev)
dst = torch.empty(N, dtype=torch.uint8, pin_memory=True)
side = torch.cuda.Stream()
main = torch.cuda.current_stream()
CB = 64 << 20
chunks = [src[i:i + CB] for i in range(0, N, CB)]
crc = torch.zeros(len(chunks), dtype=torch.int32, device=dev)
dig = torch.zeros(1, dtype=torch.int32, device=dev)


def cpu_work():
    t = time.perf_counter()
    d = {}
    for i in range(200000):
        d[i & 1023] = [i, i + 1]
    return (time.perf_counter() - t) * 1e3


def launches(n=3000):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(main)
    t = time.perf_counter()
    for _ in range(n):
        x.add_(1.0)
    host = (time.perf_counter() - t) * 1e3
    e1.record(main)
    e1.synchronize()
    return host, e0.elapsed_time(e1)


CKS = {}


def zc(kind):
    if kind not in CKS:
        path = f"/dev/shm/launch_probe2_{kind}_{os.getpid()}.pcc"
        ck = pcc.PCCheck(path, chunk_bytes=CB, max_inflight=1, flags=pcc.MAPFILE | pcc.ZEROCOPY,
                         pack_ctas=16 if kind == "sm16" else 0)
        ck.register(chunks)
        CKS[kind] = (ck, path, [0])
    return CKS[kind]


def burst(kind):
    if kind == "ce":
        with torch.cuda.stream(side):
            for off in range(0, N, CB):
                dst[off:off + CB].copy_(src[off:off + CB], non_blocking=True)
        return None
    ck, _, it = zc(kind)
    it[0] += 1
    return ck.checkpoint(it[0], stream=side)


def measure(kind):
    out = {"burst": kind}
    h = None
    if kind != "none":
        for _ in range(2):  # warm the burst path
            hh = burst(kind)
            if hh is not None:
                CKS[kind][0].wait(hh)
        side.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(side)
        t_call = time.perf_counter()
        h = burst(kind)
        out["call_ms"] = (time.perf_counter() - t_call) * 1e3
        e1.record(side)
    cpu = [cpu_work() for _ in range(3)]
    ln = [launches() for _ in range(3)]
    if kind == "ce":
        done_before = e1.query()
        e1.synchronize()
        ms = e0.elapsed_time(e1)
        out.update(burst_ms=ms, burst_gbs=N / (ms * 1e-3) / 1e9, burst_still_running_at_end=not done_before)
    elif kind != "none":
        ck = CKS[kind][0]
        done_before = pcc.STATE_NAMES[ck.poll(h)]
        ck.wait(h)
        inf = ck.info(h)
        out.update(k1_ms=inf.get("k1_busy_ms", inf.get("pack_ms")), burst_info={k: v for k, v in inf.items() if k.endswith("_ms")},
                   burst_done_at_end=done_before)
    out.update(cpu_ms=cpu, host_ms=[h for h, _ in ln], gpu_ms=[g for _, g in ln],
               us_per_launch_host=[h / 3 for h, _ in ln], us_per_launch_gpu=[g / 3 for _, g in ln])
    return out


for _ in range(3):
    launches()
    cpu_work()
try:
    for kind in ("none", "ce", "sm", "sm16", "none"):
        print(json.dumps(measure(kind)))
        sys.stdout.flush()
finally:
    for ck, path, _ in CKS.values():
        ck.close()
        os.unlink(path)
