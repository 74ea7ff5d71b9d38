"""DESIGN §11 item 4: do small-kernel launches slow down while a bulk D2H saturates PCIe?
Times 3000 tiny elementwise kernels (CUDA events, one stream) alone, then while another stream
copies 8 GiB device -> pinned host in 64 MiB pieces (the library's D2H shape); the same 3000
kernels replayed as one CUDA graph (argv[1] == "graph")."""
import json
import sys

import torch

dev = torch.device("cuda", 0)
x = torch.zeros(1024, device=dev)
src = torch.empty(8 << 30, dtype=torch.uint8, device=dev)
dst = torch.empty(8 << 30, dtype=torch.uint8, pin_memory=True)
side = torch.cuda.Stream()
main = torch.cuda.current_stream()


use_graph = len(sys.argv) > 1 and sys.argv[1] == "graph"
if use_graph:
    g = torch.cuda.CUDAGraph()
    cap = torch.cuda.Stream()
    cap.wait_stream(main)
    with torch.cuda.stream(cap):
        x.add_(1.0)
        with torch.cuda.graph(g, stream=cap):
            for _ in range(3000):
                x.add_(1.0)
    main.wait_stream(cap)


def launches(n=3000):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(main)
    if use_graph:
        g.replay()
    else:
        for _ in range(n):
            x.add_(1.0)
    e1.record(main)
    e1.synchronize()
    return e0.elapsed_time(e1)


def burst():
    piece = 64 << 20
    with torch.cuda.stream(side):
        for off in range(0, src.numel(), piece):
            dst[off:off + piece].copy_(src[off:off + piece], non_blocking=True)


for _ in range(3):
    launches()
alone = sorted(launches() for _ in range(5))[2]
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(side)
burst()
e1.record(side)
under = [launches() for _ in range(4)]  # within the ~150 ms burst
e1.synchronize()
burst_ms = e0.elapsed_time(e1)
print(json.dumps({"graph": use_graph, "launches": 3000, "ms_alone": alone, "ms_under_burst": under, "us_per_launch_alone": alone / 3,
                  "us_per_launch_under": [u / 3 for u in under], "burst_ms": burst_ms,
                  "burst_gbs": (8 << 30) / (burst_ms * 1e-3) / 1e9}))
