"""K1 / K2 alone on a config's state (pccheck_kernels.h), for ncu and quick timing.

    python tools/k1_bench.py [--config c2] [--reps 5] [--unpack]
Prints one JSON line: achieved GB/s (algorithmic bytes = read state + write image) per launch.
"""
import argparse
import json
import os
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
    off, end, c = pcc.k_layout(ts, 256, a.cb)
    img = torch.empty(c * a.cb, dtype=torch.uint8, device="cuda")
    crc = torch.zeros(c, dtype=torch.int32, device="cuda")
    aux = torch.zeros(c + 8, dtype=torch.int32, device="cuda")
    times = []
    for i in range(a.reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        if a.unpack and i > 0:
            pcc.k_unpack(ts, img.data_ptr(), crc.data_ptr(), aux.data_ptr(), aux[c:].data_ptr(),
                         aux[c + 1:].data_ptr(), 256, a.cb)
        else:
            pcc.k_pack(ts, img.data_ptr(), crc.data_ptr(), aux.data_ptr(), 256, a.cb)
        e1.record()
        e1.synchronize()
        times.append(e0.elapsed_time(e1))
    ms = min(times[1:]) if len(times) > 1 else times[0]
    b = 2 * c * a.cb
    print(json.dumps({"config": a.config, "op": "unpack" if a.unpack else "pack", "chunks": c,
                      "ms_incl_setup": ms, "gbs_incl_setup": b / (ms * 1e-3) / 1e9}))


if __name__ == "__main__":
    main()
