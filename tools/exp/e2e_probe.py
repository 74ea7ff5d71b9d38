"""Where does bench.py's e2e step (upload the whole C3 state from pinned host memory, then
checkpoint it) spend its time?  Replicates the e2e loop (N = 4, 2-slice HBM ring, 64 MiB chunks,
MAPFILE on /dev/shm) with CUDA events around each step's upload on the training stream and the
library's per-checkpoint host timestamps (t_call, t_packed, t_landed, t_committed).  Not part of
the product path."""
import json
import os
import statistics
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import paper_conf_asplos_strati0k25_b200 as pcc  # noqa: E402
from synth import config_tensors, make_state  # noqa: E402

specs = config_tensors("c3")
state = make_state(specs, "cuda", seed=0, it=0)
cb = 64 << 20
nbytes = sum(s.nbytes for s in specs)
host = [torch.empty_like(t, device="cpu").pin_memory() for t in state]
for h, t in zip(host, state):
    h.copy_(t)
stream = torch.cuda.current_stream()
mode = sys.argv[1] if len(sys.argv) > 1 else "mapfile"  # mapfile | nullsink (a reused pinned pool)
path = None if mode == "nullsink" else f"/dev/shm/e2e_probe_{os.getpid()}.pcc"
slice_est = pcc.k_layout(state, 256, cb)[2] * cb
out = {}
try:
    with pcc.PCCheck(path, chunk_bytes=cb, max_inflight=4, flags=pcc.NULLSINK if mode == "nullsink" else pcc.MAPFILE,
                     staging_bytes=8 * cb,
                     ring_bytes=2 * slice_est) as ck:
        ck.register(state)
        for variant in (mode + ",drain=" + os.environ.get("PCC_D2H_DRAIN_MIB", "128"),):
            it0 = 100
            ev = []
            hs = []
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            e_all0 = torch.cuda.Event(enable_timing=True)
            e_all0.record(stream)
            for k in range(8):
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
                for t, h in zip(state, host):
                    t.copy_(h, non_blocking=True)
                b.record(stream)
                ev.append((a, b))
                hs.append(ck.checkpoint(it0 + k, stream))
                ck.guard(stream)
            for h in hs:
                ck.wait(h)
            e_all1 = torch.cuda.Event(enable_timing=True)
            e_all1.record(stream)
            e_all1.synchronize()
            infos = [ck.info(h) for h in hs]
            up = [a.elapsed_time(b) for a, b in ev]
            gap = [ev[i][0].elapsed_time(ev[i + 1][0]) for i in range(len(ev) - 1)]  # step period on the stream
            t_call = [i["t_call_us"] for i in infos]
            out[variant] = {
                "total_ms": e_all0.elapsed_time(e_all1), "e2e_gbs": 8 * nbytes / (e_all0.elapsed_time(e_all1) * 1e-3) / 1e9,
                "upload_ms": up, "upload_gbs_median": nbytes / (statistics.median(up) * 1e-3) / 1e9,
                "step_period_ms": gap,
                "snapshot_ms": [i["snapshot_ms"] for i in infos], "k1_busy_ms": [i["k1_busy_ms"] for i in infos],
                "pack_ms": [i["pack_ms"] for i in infos],
                "landed_minus_call_ms": [(i["t_landed_us"] - i["t_call_us"]) / 1e3 for i in infos],
                "call_spacing_ms": [(t_call[i + 1] - t_call[i]) / 1e3 for i in range(len(t_call) - 1)],
            }
            print(json.dumps({variant: out[variant]}), flush=True)
finally:
    if path and os.path.exists(path):
        os.unlink(path)
