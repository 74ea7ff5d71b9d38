"""Eager launch cost under a D2H issued as a CUDA graph of many small back-to-back copies
(no host cadence needed), vs one stream of 64 MiB / 1 MiB copies.  Hypothesis: the
GPU's eager launch reads from host memory cannot pass the posted D2H writes queued ahead of them,
so smaller copies (a shallower queue) should cost launches less.  Measures, for each D2H shape,
the device time per tiny eager kernel (3000 x.add_) during the transfer and the transfer's rate.
Not part of the product path."""
import json
import sys

import torch

N = 4 << 30
src = torch.randint(0, 255, (N,), dtype=torch.uint8, device="cuda")
dst = torch.empty(N, dtype=torch.uint8, pin_memory=True)
x = torch.zeros(1024, device="cuda")
main = torch.cuda.current_stream()
side = torch.cuda.Stream()


def launches(n=3000):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(main)
    for _ in range(n):
        x.add_(1.0)
    e1.record(main)
    e1.synchronize()
    return e0.elapsed_time(e1) / n * 1e3  # us per kernel


def make_graph(piece):
    g = torch.cuda.CUDAGraph()
    side.wait_stream(main)
    with torch.cuda.stream(side):
        with torch.cuda.graph(g, stream=side):
            for o in range(0, N, piece):
                dst[o:o + piece].copy_(src[o:o + piece], non_blocking=True)
    torch.cuda.synchronize()
    return g


def measure(kind, piece):
    g = make_graph(piece) if kind == "graph" else None
    for _ in range(2):
        launches(300)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(side)
    if g is not None:
        with torch.cuda.stream(side):
            g.replay()
    else:
        with torch.cuda.stream(side):
            for o in range(0, N, piece):
                dst[o:o + piece].copy_(src[o:o + piece], non_blocking=True)
    e1.record(side)
    us = [launches(1000) for _ in range(3)]  # ~15-30 ms each, inside the ~80 ms transfer
    done = e1.query()
    e1.synchronize()
    ms = e0.elapsed_time(e1)
    return {"kind": kind, "piece_kib": piece >> 10, "us_per_launch_during": us, "transfer_done_before_end": done,
            "d2h_ms": ms, "d2h_gbs": N / (ms * 1e-3) / 1e9}


print(json.dumps({"kind": "alone", "us_per_launch": [launches(1000) for _ in range(3)]}), flush=True)
for kind, piece in (("stream", 64 << 20), ("stream", 1 << 20), ("graph", 1 << 20), ("graph", 256 << 10),
                    ("graph", 64 << 10)):
    try:
        print(json.dumps(measure(kind, piece)), flush=True)
    except Exception as ex:  # noqa: BLE001
        print(json.dumps({"kind": kind, "piece_kib": piece >> 10, "error": repr(ex)[:200]}), flush=True)
print(json.dumps({"kind": "alone", "us_per_launch": [launches(1000) for _ in range(3)]}), flush=True)
