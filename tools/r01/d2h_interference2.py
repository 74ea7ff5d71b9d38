"""A tiny D2H (.item()) on the default stream while a background thread streams 8 GiB D2H in
8 MiB pieces with at most `depth` pieces queued (events), or paced with gaps."""
import threading
import time

import torch

n = 8 << 30
piece = 8 << 20
d = torch.empty(n, dtype=torch.uint8, device="cuda")
h = torch.empty(n, dtype=torch.uint8).pin_memory()
x = torch.ones(1, device="cuda")
side = torch.cuda.Stream()


def streamer(depth, gap_us, done):
    q = []
    with torch.cuda.stream(side):
        for i in range(n // piece):
            while len(q) >= depth:
                q.pop(0).synchronize()
            if gap_us:
                time.sleep(gap_us * 1e-6)
            h[i * piece:(i + 1) * piece].copy_(d[i * piece:(i + 1) * piece], non_blocking=True)
            e = torch.cuda.Event()
            e.record(side)
            q.append(e)
    side.synchronize()
    done.append(time.perf_counter())


for depth, gap in ((1 << 30, 0), (4, 0), (2, 0), (1, 0), (4, 100)):
    torch.cuda.synchronize()
    done = []
    t0 = time.perf_counter()
    th = threading.Thread(target=streamer, args=(depth, gap, done))
    th.start()
    time.sleep(0.05)
    samples = []
    for _ in range(5):
        t = time.perf_counter()
        x.item()
        samples.append((time.perf_counter() - t) * 1e3)
        time.sleep(0.01)
    th.join()
    print(f"depth {depth} gap {gap} us: .item() ms {[round(s, 2) for s in samples]}, bulk {8 / (done[0] - t0):.1f} GiB/s",
          flush=True)
