"""Does a bulk D2H on a side stream delay a tiny D2H (.item()) on the default stream?"""
import time

import torch

n = 8 << 30
d = torch.empty(n, dtype=torch.uint8, device="cuda")
h = torch.empty(n, dtype=torch.uint8).pin_memory()
x = torch.ones(1, device="cuda")
side = torch.cuda.Stream()


def item_ms():
    t = time.perf_counter()
    x.item()
    return (time.perf_counter() - t) * 1e3


def bulk(pieces):
    step = n // pieces
    with torch.cuda.stream(side):
        for i in range(pieces):
            h[i * step:(i + 1) * step].copy_(d[i * step:(i + 1) * step], non_blocking=True)


torch.cuda.synchronize()
print("idle .item() ms", round(item_ms(), 3))
for pieces in (1, 128, 1024):
    torch.cuda.synchronize()
    bulk(pieces)
    time.sleep(0.01)
    ms = item_ms()
    t = time.perf_counter()
    side.synchronize()
    rest = (time.perf_counter() - t) * 1e3
    print(f"bulk 8 GiB in {pieces} copies: .item() ms {ms:.3f}, bulk remaining after it {rest:.1f} ms", flush=True)
# a tiny H2D too
torch.cuda.synchronize()
bulk(1)
time.sleep(0.01)
t = time.perf_counter()
y = torch.tensor([3.0]).cuda()
torch.cuda.current_stream().synchronize()
print("tiny H2D during bulk D2H ms", round((time.perf_counter() - t) * 1e3, 3))
side.synchronize()
