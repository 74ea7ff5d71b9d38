"""Sensitivity sweeps on one B200 (the paper's Fig 11-14).

    python tools/sweeps.py [--quick] > gpurun_out/sweeps.jsonl
One JSON line per point:
  fig12  VGG-16 training slowdown vs N (concurrent checkpoints) and checkpoint interval
  fig13  snapshot+persist GB/s vs writer threads p (PWRITE mode, O_DIRECT file on /dev/shm and
         on the local disk)
  fig14  snapshot+persist GB/s vs chunk size b and DRAM staging slots c = M/b
  fig11  time to checkpoint vs state size (C1, C2, C3, C5 shapes)
  variant  Variant B (HBM ring + copy engine) vs A (SM stores into host memory) vs null sink
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def emit(d):
    print(json.dumps(d), flush=True)


def snapshot_rate(pcc, torch, ts, path, cb, flags, n_ckpt=4, n_inflight=2, writer_threads=4, staging_bytes=0):
    with pcc.PCCheck(path, chunk_bytes=cb, max_inflight=n_inflight, flags=flags, writer_threads=writer_threads,
                     staging_bytes=staging_bytes) as ck:
        ck.register(ts)
        ck.wait(ck.checkpoint(1))
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        hs = [ck.checkpoint(2 + i) for i in range(n_ckpt)]
        for h in hs:
            ck.wait(h)
        dt = time.perf_counter() - t0
        inf = ck.info(hs[-1])
    if path and os.path.exists(path):
        os.unlink(path)
    state = sum(t.numel() * t.element_size() for t in ts)
    return {"gbs": state * n_ckpt / dt / 1e9, "ms_per_ckpt": dt / n_ckpt * 1e3, "k1_ms": inf["k1_busy_ms"],
            "gate_ms": inf["pack_ms"]}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--only", default="")
    a = ap.parse_args()
    import torch
    import paper_conf_asplos_strati0k25_b200 as pcc
    from synth import config_tensors, make_state
    from tools.slowdown import vgg16_slowdown
    shm = "/dev/shm"
    disk = os.environ.get("GRAFT_REPO_ROOT", "/tmp")
    only = set(a.only.split(",")) if a.only else None

    if not only or "fig12" in only:
        from bench import d2h_peak_gbs
        link = d2h_peak_gbs(torch)  # the tuner's link rate, measured here as bench.py does
        for every in ([1, 2, 5, 10] if not a.quick else [1, 10]):
            for n in [1, 2, 4]:
                for pace in ("auto", 0.0):  # the tuner's eager pace, and unpaced
                    r = vgg16_slowdown(pcc, iters=200 if not a.quick else 60, every=every, runs=1, n_inflight=n,
                                       d2h_gbs=pace, link_gbs=link)
                    emit({"sweep": "fig12", "every": every, "N": n, "pace": pace, "d2h_gbs": r.get("d2h_gbs"),
                          "slowdown_pct": r["slowdown_pct"], "iter_ms_no_ckpt": r["iter_ms_no_ckpt"],
                          "iter_ms_ckpt": r["iter_ms_ckpt"], "p99_ms": r["p99_ms"],
                          "pace_delivered_frac": r.get("pace_delivered_frac")})

    specs = config_tensors("c2")
    ts = make_state(specs, "cuda", seed=0, it=0)
    if not only or "fig13" in only:
        for where in (shm, disk):
            for p in [1, 2, 4, 8]:
                path = os.path.join(where, f"pcc_sweep_{os.getpid()}.pcc")
                r = snapshot_rate(pcc, torch, ts, path, 64 << 20, pcc.ODIRECT | pcc.FSYNC, writer_threads=p,
                                  staging_bytes=16 * (64 << 20))
                emit({"sweep": "fig13", "target": "tmpfs" if where == shm else "disk", "p": p, **r})
    if not only or "fig14" in only:
        for cb_mib in [4, 16, 64, 256]:
            for slots in [2, 8, 32]:
                cb = cb_mib << 20
                path = os.path.join(shm, f"pcc_sweep_{os.getpid()}.pcc")
                r = snapshot_rate(pcc, torch, ts, path, cb, pcc.ODIRECT, writer_threads=4, staging_bytes=slots * cb)
                emit({"sweep": "fig14", "chunk_mib": cb_mib, "staging_slots": slots, **r})
            path = os.path.join(shm, f"pcc_sweep_{os.getpid()}.pcc")
            r = snapshot_rate(pcc, torch, ts, path, cb_mib << 20, pcc.MAPFILE)
            emit({"sweep": "fig14", "chunk_mib": cb_mib, "staging_slots": "file mapping", **r})
    if not only or "variant" in only:
        for name, flags in (("B: HBM ring + CE into file mapping", pcc.MAPFILE),
                            ("A: K1 stores into file mapping", pcc.MAPFILE | pcc.ZEROCOPY),
                            ("B: HBM ring + CE, null sink", pcc.NULLSINK)):
            path = None if flags == pcc.NULLSINK else os.path.join(shm, f"pcc_sweep_{os.getpid()}.pcc")
            r = snapshot_rate(pcc, torch, ts, path, 64 << 20, flags)
            emit({"sweep": "variant", "variant": name, **r})
    del ts
    torch.cuda.empty_cache()
    if not only or "fig11" in only:
        for cfg in (["c1", "c2", "c3"] if a.quick else ["c1", "c2", "c3", "c5"]):
            specs = config_tensors(cfg)
            ts = make_state(specs, "cuda", seed=0, it=0)
            cb = 4 << 20 if cfg == "c1" else 64 << 20
            path = os.path.join(shm, f"pcc_sweep_{os.getpid()}.pcc")
            r = snapshot_rate(pcc, torch, ts, path, cb, pcc.MAPFILE, n_ckpt=3, n_inflight=1)
            emit({"sweep": "fig11", "config": cfg, "state_gb": sum(s.nbytes for s in specs) / 1e9, **r})
            del ts
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
