#!/usr/bin/env python
"""bench.py — snapshot GB/s of the PCcheck path on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c3] [--impl reference]

A step is one whole checkpoint through pccheck.h — every row of SURVEY §8(a): the U-gate,
Listing 1 lines 3-11, K1 (gather-pack + CRC32C into the HBM ring), the finalize kernels
(chunk CRCs + slice digest), copy-engine D2H straight into the registered DRAM-file mapping
(/dev/shm: the box has no NVMe), header COMPLETE, the CAS commit and the pointer record,
plus (N > 1) the NCCL allreduce(MIN) global commit.  K checkpoints are issued back to back
with N in flight and the clock stops when the last one committed.

Default workload: BASELINE configs[2] — OPT-1.3B fp32 params + Adam (15.79 GB, 1552 tensors),
64 MiB chunks, 4 in flight: the largest configuration that fits one GPU (configs[3]/[4] need
2-8 GPUs; --config c4 / --gpus N runs them).

value = state bytes of the whole job / time (box GB/s; per GPU = value / n_gpus).
e2e   = the same with the state re-uploaded from pinned host memory every step.
--gpus N without torchrun: the bench starts N local rank processes itself (one per GPU) and
fails loudly when fewer than N GPUs are visible.  Rank 0 prints ONE JSON line.
--impl reference times the CPU oracle (oracle/) instead.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "snapshot GB/s per GPU & box at 1/2/4/8 B200; % iter slowdown @ ckpt every 10 iters"
WORKLOADS = {
    "c1": "synthetic 64 MiB fp32 state in 97 mixed-size tensors, 4 MiB chunks, 2 in-flight checkpoints, DRAM-file target",
    "c2": "VGG-16 fp32 params + SGD momentum (1.107 GB), 16 MiB chunks, 2 in-flight checkpoints, DRAM-file target",
    "c3": "OPT-1.3B fp32 params + Adam (15.79 GB, 1552 tensors), 64 MiB chunks, 4 in-flight checkpoints, "
          "DRAM-file target (/dev/shm: the box has no NVMe SSD)",
    "c4": "BLOOM-7b1 bf16 params + fp32 master + Adam (98.97 GB), 64 MiB chunks, 1/world slice per rank",
    "bert": "BERT-large QA fp32 params + Adam (PAPER Table 3's 4 GB checkpoint), 64 MiB chunks, 2 in-flight "
            "checkpoints, DRAM-file target",
}


def env_int(k, d):
    try:
        return int(os.environ.get(k, d))
    except ValueError:
        return d


class ClockSampler:
    """nvidia-smi clocks + throttle reasons DURING the timed region (B200_PROFILING.md)."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, device):
        self.device = device
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.device), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "50"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for l in self.lines:
            p = [x.strip() for x in l.split(",")]
            if len(p) < 8:
                continue
            try:
                sm.append(float(p[1]))
                mx.append(float(p[2]))
            except ValueError:
                continue
            for n, v in zip(names, p[4:8]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


def d2h_peak_gbs(torch, nbytes=1 << 30):
    """Pinned cudaMemcpy D2H peak, measured live (the link roofline denominator)."""
    d = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    h = torch.empty(nbytes, dtype=torch.uint8).pin_memory()
    s = torch.cuda.Stream()
    best = 1e9
    with torch.cuda.stream(s):
        for i in range(11):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            h.copy_(d, non_blocking=True)
            b.record(s)
            b.synchronize()
            if i >= 1:
                best = min(best, a.elapsed_time(b))
    del d, h
    return nbytes / (best * 1e-3) / 1e9


def bidir_peak_gbs(torch, nbytes=2 << 30, piece=64 << 20):
    """Pinned H2D and D2H running at once, the way the e2e line moves data (a stream of 64 MiB
    copies each way on two streams), each direction timed on its own stream: (h2d, d2h) GB/s,
    best of 2.  The e2e line moves the slice up AND the checkpoint down every step, so the slower
    of these, not the one-way peak, bounds it.  (Measured on the box: 46.5 up + 49.8 down with
    both running, 55.4 / 56.4 alone; tools/exp/bidir_probe.py.  The round-2 version timed one
    1 GiB copy each way from a common start and reported ~26 GB/s, below what e2e itself moved.)"""
    d1 = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    d2 = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    h1 = torch.empty(nbytes, dtype=torch.uint8).pin_memory()
    h2 = torch.empty(nbytes, dtype=torch.uint8).pin_memory()
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    best_up = best_dn = 0.0
    for i in range(3):
        torch.cuda.synchronize()
        start = torch.cuda.Event()
        start.record(torch.cuda.current_stream())
        e = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
        s1.wait_event(start)
        s2.wait_event(start)
        e[0].record(s1)
        e[2].record(s2)
        with torch.cuda.stream(s1):
            for o in range(0, nbytes, piece):
                d1[o:o + piece].copy_(h1[o:o + piece], non_blocking=True)
        with torch.cuda.stream(s2):
            for o in range(0, nbytes, piece):
                h2[o:o + piece].copy_(d2[o:o + piece], non_blocking=True)
        e[1].record(s1)
        e[3].record(s2)
        torch.cuda.synchronize()
        if i >= 1:
            best_up = max(best_up, nbytes / (e[0].elapsed_time(e[1]) * 1e-3) / 1e9)
            best_dn = max(best_dn, nbytes / (e[2].elapsed_time(e[3]) * 1e-3) / 1e9)
    del d1, d2, h1, h2
    return best_up, best_dn


def cpu_baseline(specs, state, cb, budget_bytes=4 << 30, threads=1):
    """The oracle as it stands (plain C: byte-loop pack + byte-at-a-time CRC32C) on a bounded
    sample of the same image: its first chunks up to `budget_bytes` (the whole image when it is
    smaller), then the per-chunk CRCs.  Each oracle is handed only the tensors overlapping its
    chunk range (their bytes copied to the host by torch, untimed).  threads > 1: that many host
    threads over disjoint chunk ranges, each an independent oracle (K independent
    oracles; ctypes drops the GIL)."""
    import oracle
    from concurrent.futures import ThreadPoolExecutor
    from synth import host_bytes
    nb = [s.nbytes for s in specs]
    off, end, c = oracle.layout(nb, 256, cb)
    k = max(1, min(c, budget_bytes // cb))
    parts = [(i * k // threads, (i + 1) * k // threads) for i in range(threads)]
    parts = [(a, b) for a, b in parts if b > a]
    hi_all = k * cb
    hb = {i: host_bytes(state[i]) for i in range(len(nb)) if nb[i] and int(off[i]) < hi_all}

    def run(ab):
        lo, hi = ab[0] * cb, ab[1] * cb
        mine = {i: hb[i] for i in hb if int(off[i]) < hi and int(off[i]) + nb[i] > lo}
        img = oracle.pack_chunks_sparse(nb, mine, 256, cb, ab[0], ab[1] - ab[0])
        oracle.chunk_crcs(img, cb)

    t0 = time.perf_counter()
    with ThreadPoolExecutor(len(parts)) as ex:
        list(ex.map(run, parts))
    dt = time.perf_counter() - t0
    return {"value": k * cb / dt / 1e9, "unit": "GB/s", "cores": len(parts), "kind": "oracle",
            "sample": f"pack + CRC32C of chunks 0..{k - 1} of {c} ({cb >> 20} MiB) of the same image "
                      f"({k * cb / 1e9:.3f} GB{' = the whole image' if k == c else ' prefix'}, {dt:.1f} s, plain C, "
                      f"{len(parts)} thread(s) over disjoint chunk ranges)",
            "cpu": _cpu_model(), "nproc": os.cpu_count()}


def _cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def load_traffic(name):
    p = os.path.join(ROOT, "profiles", "k1_traffic.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return d.get(name)
    except Exception:
        return None


def default_inflight(cfg):
    """N (Table 2: 2-4): 4 for OPT-1.3B (configs[2] says so), 2 elsewhere."""
    return 4 if cfg == "c3" else 2


def spawn_local_ranks(args):
    """`python bench.py --gpus N` outside torchrun: start N rank processes on this node (one per
    GPU, RANK / LOCAL_RANK / WORLD_SIZE / MASTER_* in their environment), wait for all, return
    the worst exit code.  Rank 0 prints the JSON line."""
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    procs = []
    for r in range(args.gpus):
        env = dict(os.environ, RANK=str(r), LOCAL_RANK=str(r), WORLD_SIZE=str(args.gpus), LOCAL_WORLD_SIZE=str(args.gpus),
                   MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        procs.append(subprocess.Popen([sys.executable, os.path.abspath(__file__)] + sys.argv[1:], env=env))
    rcs = [p.wait() for p in procs]
    return max(rcs, key=abs) if any(rcs) else 0


def default_chunk_bytes(args):
    """chunk size b (R2): 4 MiB for the 64 MiB state; 16 MiB for VGG-16 (fig14 sweep: best of
    4/16/64/256 MiB — less zero padding in the last chunk); 64 MiB for the 10-100 GB states"""
    if args.chunk_mib:
        return args.chunk_mib << 20
    return {"c1": 4 << 20, "c2": 16 << 20}.get(args.config, 64 << 20)


def run_reference(args, rank, world):
    """--impl reference: the CPU oracle on the same workload, bounded sample per step (the next
    ~128 MiB of chunks of the image per step); only the tensors a step's chunks overlap are
    materialised (same seeded generator as the native arm, on the host)."""
    if rank != 0:
        return
    import torch
    import oracle as O  # the reference arm: the one other place bench.py runs oracle/
    from synth import config_tensors, fill_tensor, torch_dtype
    specs = config_tensors(args.config)
    cb = default_chunk_bytes(args)
    nb = [s.nbytes for s in specs]
    off, end, c = O.layout(nb, 256, cb)
    per_step = max(1, min(c, (128 << 20) // cb))
    cache = {}

    def host(i):  # tensor i as the native arm's make_state(seed=0, it=0) fills it, on the host
        if i not in cache:
            t = torch.empty(specs[i].shape, dtype=torch_dtype(specs[i].dtype))
            fill_tensor(t, specs[i], 0, 0, i)
            cache[i] = t.reshape(-1).view(torch.uint8).numpy() if t.dim() else t.reshape(1).view(torch.uint8).numpy()
        return cache[i]

    times = []
    j = 0
    for step in range(args.warmup + args.steps):
        a = j % c
        k = min(per_step, c - a)
        lo, hi = a * cb, (a + k) * cb
        idx = [i for i in range(len(nb)) if int(off[i]) < hi and int(off[i]) + nb[i] > lo and nb[i]]
        for i in list(cache):
            if i not in idx:
                del cache[i]
        mine = {i: host(i) for i in idx}
        t0 = time.perf_counter()
        img = O.pack_chunks_sparse(nb, mine, 256, cb, a, k)
        O.chunk_crcs(img, cb)
        dt = time.perf_counter() - t0
        if step >= args.warmup:
            times.append((img.nbytes, dt))
        j += k
    tot_b = sum(b for b, _ in times)
    tot_t = sum(t for _, t in times)
    v = tot_b / tot_t / 1e9
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "GB/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": tot_t / len(times) * 1e3,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u8",
            "data": "synthetic (seeded bit patterns shaped like the model state)",
            "config": {"workload": WORKLOADS.get(args.config, args.config), "config": args.config,
                       "chunk_bytes": cb},
            "cpu_baseline": {"value": v, "unit": "GB/s", "cores": 1, "kind": "oracle",
                             "sample": f"per step: pack + CRC32C of the next {per_step} {cb >> 20} MiB chunks of the image "
                                       f"(1 thread, plain C; the tensors they overlap materialised untimed)"},
            "e2e": {"value": v, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def run_slowdowns(args, pcc, rank, world, coll, uid, peak_link, emu, torch, dist):
    """The slowdown variants of the config's model (see the comment at the call site)."""
    from tools import slowdown as S
    kw = dict(iters=args.slowdown_iters, runs=args.slowdown_runs, every=10)
    auto = dict(d2h_gbs="auto", link_gbs=peak_link)
    plans = []
    if args.config == "c2":
        if world > 1:
            ckw = dict(coll) if coll else {"nccl_unique_id": None}
            for name, extra in (("slowdown", auto), ("slowdown_unpaced", {})):
                def fn(extra=extra):
                    if not coll:  # a fresh NCCL unique id per communicator, broadcast by torch
                        obj = [pcc.nccl_unique_id() if rank == 0 else None]
                        dist.broadcast_object_list(obj, src=0)
                        ckw["nccl_unique_id"] = obj[0]
                    return S.vgg16_slowdown(pcc, rank=rank, world=world, ck_kwargs=ckw, **kw, **extra)
                plans.append((name, fn))
        else:
            plans = [("slowdown", lambda: S.vgg16_slowdown(pcc, graphs=True, host_lead=2, **kw, **auto)),
                     ("slowdown_eager", lambda: S.vgg16_slowdown(pcc, **kw, **auto)),
                     ("slowdown_unpaced", lambda: S.vgg16_slowdown(pcc, **kw))]
    elif args.config == "c3" and world > 1:  # OPT-1.3B under DDP, every rank its 1/world slice
        ckw = dict(coll) if coll else {"nccl_unique_id": None}
        for name, extra in (("slowdown", auto), ("slowdown_unpaced", {})):
            def fn(extra=extra):
                if not coll:
                    obj = [pcc.nccl_unique_id() if rank == 0 else None]
                    dist.broadcast_object_list(obj, src=0)
                    ckw["nccl_unique_id"] = obj[0]
                return S.hf_slowdown(pcc, "opt13", n_inflight=args.inflight, rank=rank, world=world, ck_kwargs=ckw,
                                     **kw, **extra)
            plans.append((name, fn))
    elif args.config == "c3" and world == 1:
        o = dict(n_inflight=args.inflight, **kw)
        plans = [  # graphs + the tuner's graph pace, host <= 2 replays ahead (a loop that reads its loss)
                 ("slowdown", lambda: S.hf_slowdown(pcc, "opt13", graphs=True, host_lead=2, **o, **auto)),
                 # graphs, host unthrottled (runs into a full launch queue): PCC_D2H_UPFRONT, unpaced
                 ("slowdown_graphs_unthrottled", lambda: S.hf_slowdown(pcc, "opt13", graphs=True, **o)),
                 ("slowdown_eager", lambda: S.hf_slowdown(pcc, "opt13", **o, **auto)),
                 ("slowdown_unpaced", lambda: S.hf_slowdown(pcc, "opt13", **o))]
    elif args.config == "bert" and world == 1:
        plans = [("slowdown", lambda: S.hf_slowdown(pcc, "bert", **kw, **auto)),
                 ("slowdown_unpaced", lambda: S.hf_slowdown(pcc, "bert", **kw))]
    elif args.config == "c4" and world == 1:
        plans = [("slowdown", lambda: S.bloom_slowdown(pcc, world=emu or 8, **kw, **auto)),
                 ("slowdown_unpaced", lambda: S.bloom_slowdown(pcc, world=emu or 8, **kw))]
    out = {}
    for name, fn in plans:
        err = 0
        try:
            r = fn()
        except Exception as ex:  # noqa: BLE001
            r, err = {"error": repr(ex)[:300]}, 1
        torch.cuda.empty_cache()
        if world > 1:  # the max over ranks
            t = torch.tensor([r.get("slowdown_pct") or 0.0, float(err)], device="cpu" if args.share_gpu else "cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            r["slowdown_pct_rank"] = r.get("slowdown_pct")
            r["slowdown_pct"] = float(t[0]) if not float(t[1]) else None
        out[name] = r
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="c3")
    ap.add_argument("--impl", default="native", choices=["native", "reference"])
    ap.add_argument("--inflight", type=int, default=0, help="N checkpoints in flight (0 = per-config default)")
    ap.add_argument("--chunk-mib", type=int, default=0, help="chunk size b in MiB (0 = per-config default)")
    ap.add_argument("--ring-slices", type=int, default=2, help="HBM ring = this many slices")
    ap.add_argument("--d2h-gbs", type=float, default=0.0, help="pace the D2H copies (GB/s; 0 = full link)")
    ap.add_argument("--d2h-quantum-kib", type=int, default=0, help="bytes per D2H copy in KiB (0 = chunk groups)")
    ap.add_argument("--no-slowdown", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--mode", default="mapfile", choices=["mapfile", "zerocopy", "nullsink", "pwrite"])
    ap.add_argument("--share-gpu", action="store_true", help=argparse.SUPPRESS)  # test hook (see main)
    ap.add_argument("--collectives", default="nccl", choices=["torch", "nccl"],
                    help="N>1: the library's own NCCL communicator (default) or torch.distributed callbacks")
    ap.add_argument("--slowdown-iters", type=int, default=200, help="measured iterations per run (SURVEY §8(d): 200)")
    ap.add_argument("--slowdown-runs", type=int, default=3, help="runs (PAPER L308: 3)")
    ap.add_argument("--emulate-world", type=int, default=0,
                    help="1 GPU plays rank 0 of this world size alone (PCC_NOCOMM): per-GPU share of a DP job")
    args = ap.parse_args()
    args.inflight = args.inflight or default_inflight(args.config)
    if args.impl == "reference":
        run_reference(args, env_int("RANK", 0), env_int("WORLD_SIZE", 1))
        return
    if "RANK" not in os.environ and args.gpus > 1:  # not under torchrun: start the ranks ourselves
        sys.exit(spawn_local_ranks(args))
    rank, world = env_int("RANK", 0), env_int("WORLD_SIZE", 1)
    local = env_int("LOCAL_RANK", 0)
    if world != args.gpus:
        sys.exit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}: refusing to report a "
                 f"{world}-rank run as {args.gpus} GPUs")
    args.warmup = max(3, args.warmup)

    import torch
    import torch.distributed as dist
    if args.share_gpu:  # test hook: every rank on cuda:0, gloo transport (NCCL refuses duplicate GPUs)
        local = 0
    elif torch.cuda.device_count() < world:
        sys.exit(f"bench.py: {world} ranks need {world} GPUs, {torch.cuda.device_count()} visible")
    torch.cuda.set_device(local)
    if world > 1:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        if args.share_gpu:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    import paper_conf_asplos_strati0k25_b200 as pcc
    from synth import config_tensors, make_state

    specs = config_tensors(args.config)
    cb = default_chunk_bytes(args)
    state = make_state(specs, "cuda", seed=0, it=0)
    state_bytes = sum(s.nbytes for s in specs)
    uid = None
    coll = {}
    if world > 1 and args.collectives == "nccl":  # the library's own NCCL communicator
        obj = [pcc.nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        uid = obj[0]
    elif world > 1:  # torch.distributed as the library's transport (gloo with --share-gpu)
        if not args.share_gpu:
            sys.exit("bench.py: --collectives torch needs --share-gpu (gloo); use the native NCCL default")
        coll = pcc.torch_collectives(dist)
    from paper_conf_asplos_strati0k25_b200 import k_layout
    n_est = k_layout([(1 << 20, s.nbytes, s.code) for s in specs], 256, cb)[2]
    slice_est = -(-n_est // world) * cb
    emu = args.emulate_world if world == 1 and args.emulate_world > 1 else 0
    if emu:
        slice_est = -(-n_est // emu) * cb
    flags = {"mapfile": pcc.MAPFILE, "zerocopy": pcc.MAPFILE | pcc.ZEROCOPY, "nullsink": pcc.NULLSINK,
             "pwrite": pcc.ODIRECT}[args.mode] | (pcc.NOCOMM if emu else 0)
    shm = "/dev/shm" if os.path.isdir("/dev/shm") else "/tmp"
    path = None if args.mode == "nullsink" else os.path.join(shm, f"pcc_bench_{os.getpid()}_r{rank}.pcc")
    ck = pcc.PCCheck(path, chunk_bytes=cb, max_inflight=args.inflight, flags=flags, device=local, rank=rank,
                     world=emu or world, nccl_unique_id=uid, **coll, staging_bytes=8 * cb, ring_bytes=args.ring_slices * slice_est,
                     d2h_gbs=args.d2h_gbs, d2h_quantum=args.d2h_quantum_kib << 10)
    ck.register(state)
    geo = ck.geometry()
    slice_bytes = geo["count"] * cb
    # state bytes inside this rank's chunk range (R3: GB/s counts state bytes, not pads)
    offs, _, _ = pcc.k_layout([(1 << 20, s.nbytes, s.code) for s in specs], 256, cb)
    lo, hi = geo["first"] * cb, (geo["first"] + geo["count"]) * cb
    rank_state_bytes = sum(max(0, min(o + s.nbytes, hi) - max(o, lo)) for o, s in zip(offs, specs))
    if emu:  # one GPU playing one rank: the job is this rank's share
        state_bytes = rank_state_bytes
    stream = torch.cuda.current_stream()

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    it = 0

    def one_ckpt():
        nonlocal it
        it += 1
        h = ck.checkpoint(it, stream)
        ck.guard(stream)
        if world > 1:
            ck.commit()
        return h

    clocks = ClockSampler(local)  # started before the warm-up so it samples the whole timed region
    clocks.start()
    time.sleep(0.5)
    # ---- warm-up
    warm = []
    for _ in range(args.warmup):
        h = one_ckpt()
        ck.wait(h)
        warm.append(ck.info(h))
    # one checkpoint at a time with nothing else running (SURVEY §8(d) "idle"): K1 start -> last
    # chunk landed, GPU clock; the first warm-up checkpoint also pays first-touch costs
    idle_ms = statistics.median(i["snapshot_ms"] for i in warm[1:] or warm)
    if world > 1:
        ck.commit()
    barrier()

    # ---- timed region: K checkpoints, N in flight
    launches0 = ck.kernel_launches()
    barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    e0.record(stream)
    hs = [one_ckpt() for _ in range(args.steps)]
    for h in hs:
        ck.wait(h)
    if world > 1:
        ck.commit()
    e1.record(stream)
    e1.synchronize()
    wall = time.perf_counter() - t0
    dev_ms = e0.elapsed_time(e1)
    launches = ck.kernel_launches() - launches0
    clk = clocks.stop()
    infos = [ck.info(h) for h in hs]
    pack_ms = statistics.mean(i["pack_ms"] for i in infos)  # U-gate span (incl. ring waits between launches)
    k1_ms = statistics.mean(i["k1_busy_ms"] for i in infos)  # K1's own launches, summed per checkpoint
    fin_ms = statistics.mean(i["finalize_ms"] for i in infos)
    lat_ms = statistics.median((i["t_committed_us"] - i["t_call_us"]) / 1e3 for i in infos)
    t = torch.tensor([dev_ms], device="cpu" if args.share_gpu else "cuda")
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_total = float(t.item())
    value = state_bytes * args.steps / (ms_total * 1e-3) / 1e9  # whole job (every rank packs its 1/W slice)

    # ---- e2e: the state comes from pinned host memory every step (H2D inside the timed region)
    # the inputs of this rank's share: every tensor overlapping its chunk range (all of them at W=1)
    offs_all, _, _ = pcc.k_layout([(1 << 20, s.nbytes, s.code) for s in specs], 256, cb)
    lo_b, hi_b = geo["first"] * cb, (geo["first"] + geo["count"]) * cb
    upload = [i for i, (o, s) in enumerate(zip(offs_all, specs)) if o < hi_b and o + s.nbytes > lo_b]
    h2d_bytes = sum(specs[i].nbytes for i in upload)
    host_state = {i: torch.empty_like(state[i], device="cpu").pin_memory() for i in upload}
    for i, h_ in host_state.items():
        h_.copy_(state[i])
    barrier()
    e2 = torch.cuda.Event(enable_timing=True)
    e3 = torch.cuda.Event(enable_timing=True)
    e2.record(stream)
    hs2 = []
    e2e_steps = args.steps  # the same step count as `value`
    for _ in range(e2e_steps):
        for i, h_ in host_state.items():
            state[i].copy_(h_, non_blocking=True)
        hs2.append(one_ckpt())
    crc_bytes = 0
    for h in hs2:
        ck.wait(h)
        crc_bytes += 4 * (geo["count"] + 1)
        ck.info(h, with_crc=True)  # the step's result read (CRC table + digest)
    if world > 1:
        ck.commit()
    e3.record(stream)
    e3.synchronize()
    t2 = torch.tensor([e2.elapsed_time(e3)], device="cpu" if args.share_gpu else "cuda")
    if world > 1:
        dist.all_reduce(t2, op=dist.ReduceOp.MAX)
    e2e_value = state_bytes * e2e_steps / (float(t2.item()) * 1e-3) / 1e9

    # restore (L287 + K2 verify): the newest checkpoint back into the registered tensors
    restore = None
    if args.mode != "nullsink" and world == 1:
        barrier()
        t0r = time.perf_counter()
        rit, rbad = ck.restore()
        torch.cuda.synchronize()
        rdt = time.perf_counter() - t0r
        rs = ck.restore_stats()
        restore = {"iter": rit, "ms": rdt * 1e3, "gbs": state_bytes / rdt / 1e9, "bad_chunks": len(rbad),
                   "path": "file mapping -> H2D into the HBM ring -> K2 verify+scatter",
                   # SURVEY §8(d) breakdown (pcc_restore_stats; storage read is the copy engine's
                   # read of the mapped file, inside h2d, in MAPFILE mode)
                   "breakdown_ms": {k: rs[k] for k in ("read_ms", "h2d_ms", "k2_ms", "finalize_ms", "fanout_ms",
                                                       "total_ms")},
                   "h2d_gbs": rs["bytes"] / (rs["h2d_ms"] * 1e-3) / 1e9 if rs["h2d_ms"] else None,
                   # K2 reads the staged slice and writes the state bytes back: bytes + state bytes
                   "k2_gbs": (rs["bytes"] + state_bytes) / (rs["k2_ms"] * 1e-3) / 1e9 if rs["k2_ms"] else None}
    barrier()  # W > 1: every GPU probes its link at the same time (the peak at the same concurrency)
    peak_link = d2h_peak_gbs(torch)
    peak_bidir = bidir_peak_gbs(torch)
    peak_box = peak_link
    if world > 1:  # the concurrent aggregate of all ranks' D2H peaks (SURVEY §8(d) "box level")
        tb = torch.tensor([peak_link], device="cpu" if args.share_gpu else "cuda", dtype=torch.float64)
        dist.all_reduce(tb)
        peak_box = float(tb.item())
    ck.close()
    if path and os.path.exists(path):
        os.unlink(path)

    # the oracle as it stands on the host cores, on the same image (before the slowdown runs free
    # the state)
    cpu = cpu_all = None
    if rank == 0 and not args.no_cpu_baseline and args.config in ("c1", "c2", "c3", "bert"):
        cpu = cpu_baseline(specs, state, cb)
        cpu_all = cpu_baseline(specs, state, cb, threads=len(os.sched_getaffinity(0)))

    # training slowdown, checkpoint every 10 iterations (BASELINE metric, second half), on the
    # config's own model with SURVEY §8(d)'s protocol (tools/slowdown.run_protocol: 20 warm-up +
    # --slowdown-iters x --slowdown-runs, p50/p99, final drain):
    #   slowdown           the library as configured for training: the step as 2 CUDA graphs, the
    #                      tuner's graph D2H pace (tuner.choose_pace), host <= 2 replays ahead
    #   slowdown_graphs_unthrottled  (C3) graphs with the host unthrottled: PCC_D2H_UPFRONT
    #   slowdown_eager     eager PyTorch, tuned pace
    #   slowdown_unpaced   eager PyTorch, unpaced (the transfer configuration `value` is measured in)
    #   world > 1: DDP on every rank, each checkpointing its 1/world slice with the collective
    #   commit; the reported slowdown is the max over ranks
    if "state" in locals():
        del state
    if "host_state" in locals():
        del host_state
    torch.cuda.empty_cache()
    slowdowns = {}
    if not args.no_slowdown:
        slowdowns = run_slowdowns(args, pcc, rank, world, coll, uid, peak_link, emu, torch, dist)

    if rank == 0:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            peaks = json.load(f)
        k1_bytes = rank_state_bytes + slice_bytes  # read the slice's state bytes + write the packed slice (R3: pads count)
        if restore and restore.get("k2_gbs"):
            restore["k2_hbm_frac"] = restore["k2_gbs"] / peaks["hbm_gbs"]
        k1_achieved = k1_bytes / (k1_ms * 1e-3) / 1e9
        link_achieved = slice_bytes / (ms_total * 1e-3 / args.steps) / 1e9
        line = {
            "metric": METRIC, "value": value, "unit": "GB/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_total / args.steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "u8",
            "data": "synthetic (seeded bit patterns; shapes of the model's params + optimizer state)",
            "config": {"workload": WORKLOADS.get(args.config, args.config), "config": args.config,
                       "state_bytes": state_bytes, "chunk_bytes": cb, "chunks": geo["n_chunks"],
                       "inflight": args.inflight, "mode": args.mode, "hbm_ring_slices": args.ring_slices,
                       "d2h_gbs": args.d2h_gbs or None, "d2h_quantum_bytes": (args.d2h_quantum_kib << 10) or None,
                       "emulated_rank_of_world": emu or None,
                       "collectives": (args.collectives if world > 1 else None), "parallelism": f"dp{world}",
                       "target": "DRAM file on /dev/shm (tmpfs), mmap + cudaHostRegister" if args.mode != "nullsink"
                       else "null sink", "l2": "inputs larger than L2 (state >> 126 MB)"},
            "per_gpu_gbs": value / world,
            "checkpoint_latency_ms_p50": lat_ms,
            "snapshot_idle": {"ms": idle_ms, "gbs": rank_state_bytes / (idle_ms * 1e-3) / 1e9,
                              "def": "K1 start -> last chunk landed in host memory, CUDA events, one checkpoint "
                                     "in flight, median of the warm-up checkpoints after the first"},
            "roofline": {"bound": "hbm", "kernel": "k_snap_tma<pack> (K1 v7)" if os.environ.get("PCC_KIMPL") != "v6" else "k_snapshot<pack> (K1 v6)", "achieved": k1_achieved,
                         "peak": peaks["hbm_gbs"], "unit": "GB/s", "frac": k1_achieved / peaks["hbm_gbs"],
                         # ncu's DRAM bytes of one W = 1 launch (profiles/k1_traffic.json)
                         "traffic": load_traffic(f"{args.config}_k1" + ("_v6" if os.environ.get("PCC_KIMPL") == "v6" else "")) if world == 1 and not emu else None,
                         "algorithmic_bytes_per_checkpoint": k1_bytes, "k1_ms_per_checkpoint": k1_ms,
                         "k1_launches_per_checkpoint": (launches - 2 * args.steps) / args.steps,  # minus the 2 finalize kernels
                         "pack_span_ms": pack_ms,
                         "peak_source": "MEASURED_PEAKS.json hbm_gbs (burst copy)"},
            "link_roofline": {"bound": "pcie_d2h", "achieved": link_achieved, "peak": peak_link, "unit": "GB/s",
                              "frac": link_achieved / peak_link,
                              "peak_source": "pinned 1 GiB cudaMemcpy D2H, measured in this run (all ranks at once)",
                              "box": {"achieved": value, "peak": peak_box, "frac": value / peak_box,
                                      "def": "whole-job state GB/s vs the sum of the ranks' concurrent D2H peaks"}},
            "finalize_ms": fin_ms,
            "restore": restore,
            "cpu_baseline": cpu,
            "cpu_baseline_all_cores": cpu_all,
            "e2e": {"value": e2e_value, "unit": "GB/s", "h2d_bytes_per_step": h2d_bytes,
                    "d2h_bytes_per_step": slice_bytes + 4 * (geo["count"] + 1),
                    # both directions busy every step: the bound is the concurrent H2D + D2H rate
                    "link_peak_bidir_gbs": {"h2d": peak_bidir[0], "d2h": peak_bidir[1],
                                            "def": "both directions at once, 64 MiB copies each way, per-direction stream time"},
                    "frac_of_bidir": e2e_value / world / min(peak_bidir)},  # per GPU, vs the slower direction
            "gpu_launches": launches,
            "clocks": clk,
            **slowdowns,
            "wall_s_timed": wall,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
