"""Pinned H2D and D2H at the same time: what does the box's PCIe path carry per direction?
bench.py's bidir_peak_gbs (one 1 GiB copy each way, max of the two elapsed times) reports ~26 GB/s
per direction while the e2e line itself moves ~41 GB/s each way; this measures it the way e2e
runs (many 64 MiB copies per direction on separate streams, each direction timed on its own
stream over the window where both run), plus each direction alone.  Not part of the product path."""
import json

import torch

N = 8 << 30
P = 64 << 20
dev_a = torch.empty(N, dtype=torch.uint8, device="cuda")
dev_b = torch.empty(N, dtype=torch.uint8, device="cuda")
host_a = torch.empty(N, dtype=torch.uint8).pin_memory()
host_b = torch.empty(N, dtype=torch.uint8).pin_memory()
s_up, s_dn = torch.cuda.Stream(), torch.cuda.Stream()


def run(up, dn, piece=P):
    torch.cuda.synchronize()
    ev = {k: torch.cuda.Event(enable_timing=True) for k in ("u0", "u1", "d0", "d1")}
    start = torch.cuda.Event(enable_timing=True)
    start.record(torch.cuda.current_stream())
    s_up.wait_event(start)
    s_dn.wait_event(start)
    if up:
        ev["u0"].record(s_up)
        with torch.cuda.stream(s_up):
            for o in range(0, N, piece):
                dev_a[o:o + piece].copy_(host_a[o:o + piece], non_blocking=True)
        ev["u1"].record(s_up)
    if dn:
        ev["d0"].record(s_dn)
        with torch.cuda.stream(s_dn):
            for o in range(0, N, piece):
                host_b[o:o + piece].copy_(dev_b[o:o + piece], non_blocking=True)
        ev["d1"].record(s_dn)
    torch.cuda.synchronize()
    out = {}
    if up:
        out["h2d_gbs"] = N / (ev["u0"].elapsed_time(ev["u1"]) * 1e-3) / 1e9
    if dn:
        out["d2h_gbs"] = N / (ev["d0"].elapsed_time(ev["d1"]) * 1e-3) / 1e9
    return out


for up, dn in ((1, 0), (0, 1), (1, 1), (1, 1)):
    run(up, dn)
    r = run(up, dn)
    r.update(up=up, down=dn, bytes_per_direction=N, piece=P)
    print(json.dumps(r))
big = run(1, 1, piece=1 << 30)
big.update(up=1, down=1, piece=1 << 30, note="1 GiB pieces")
print(json.dumps(big))
