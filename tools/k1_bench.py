"""K1 / K2 alone on a config's state, for ncu and quick timing.

    python tools/k1_bench.py [--config c2] [--reps 5] [--unpack]
pack: K1 timed by the runtime's CUDA events (pcc_checkpoint, NULL sink, checkpoints waited one
by one) -> pack_ms; algorithmic bytes = read the slice's state + write its packed chunks.
unpack: pcc_k_unpack on a packed image (includes its host-side setup).
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c2")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--cb", type=int, default=64 << 20)
    ap.add_argument("--unpack", action="store_true")
    a = ap.parse_args()
    import torch
    import paper_conf_asplos_strati0k25_b200 as pcc
    from synth import config_tensors, make_state
    specs = config_tensors(a.config)
    ts = make_state(specs, "cuda", seed=0, it=0)
    state = sum(s.nbytes for s in specs)
    off, end, c = pcc.k_layout(ts, 256, a.cb)
    if not a.unpack:
        with pcc.PCCheck(None, chunk_bytes=a.cb, max_inflight=2, flags=pcc.NULLSINK, staging_bytes=4 * a.cb) as ck:
            ck.register(ts)
            ms, fin = [], []
            for it in range(1, a.reps + 1):
                h = ck.checkpoint(it)
                ck.wait(h)
                inf = ck.info(h)
                ms.append(inf["pack_ms"])
                fin.append(inf["finalize_ms"])
        k1 = statistics.median(ms[1:] if len(ms) > 1 else ms)
        b = state + c * a.cb
        print(json.dumps({"config": a.config, "op": "pack", "chunks": c, "k1_ms": k1, "finalize_ms": statistics.median(fin),
                          "k1_gbs_algorithmic": b / (k1 * 1e-3) / 1e9, "state_gbs": state / (k1 * 1e-3) / 1e9}))
        return
    img = torch.empty(c * a.cb, dtype=torch.uint8, device="cuda")
    crc = torch.zeros(c, dtype=torch.int32, device="cuda")
    aux = torch.zeros(c + 8, dtype=torch.int32, device="cuda")
    pcc.k_pack(ts, img.data_ptr(), crc.data_ptr(), aux.data_ptr(), 256, a.cb)
    times = []
    for i in range(a.reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        pcc.k_unpack(ts, img.data_ptr(), crc.data_ptr(), aux.data_ptr(), aux[c:].data_ptr(), aux[c + 1:].data_ptr(),
                     256, a.cb)
        e1.record()
        e1.synchronize()
        times.append(e0.elapsed_time(e1))
    ms = statistics.median(times)
    print(json.dumps({"config": a.config, "op": "unpack", "chunks": c, "ms_incl_setup": ms,
                      "gbs_incl_setup": (state + c * a.cb) / (ms * 1e-3) / 1e9}))


if __name__ == "__main__":
    main()
