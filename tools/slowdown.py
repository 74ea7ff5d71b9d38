"""Training-iteration slowdown with a checkpoint every `every` iterations vs none
(BASELINE.json metric, second half; SURVEY §8(d) "Definitions").

One measurement protocol (``run_protocol``) for every model: 20 warm-up iterations (with
checkpoints, so first-touch costs are paid), then per run `iters` = 200 iterations without and
200 with a checkpoint every `every`, x `runs` = 3 (3 runs).  Wall time on the
device (CUDA events, synchronised at both ends); p50 / p99 iteration times so the stall spikes at
checkpoint iterations show; the final drain (waiting for the checkpoints still in flight after
the last iteration) is reported separately, not hidden in the loop time.

Per iteration: forward + backward, ``pcc_guard`` (the U-gate of L139: the update must not
overwrite state K1 is still reading), the optimizer step; after the step of every `every`-th
iteration ``pcc_checkpoint(iter)`` (+ the collective ``pcc_commit`` when world > 1).

Models (random init, synthetic inputs):
  vgg16   torchvision VGG-16 fp32, SGD(momentum 0.9), batch 32 x 3x224x224   (PAPER Table 3)
  bert    BERT-large QA fp32, Adam(fused), batch 3 x 384                      (Table 3)
  opt13   OPT-1.3B fp32 params, Adam(fused), bf16 autocast, batch 1 x 2048    (Table 3; C3)
  bloom   BLOOM-7b1 bf16 + fp32 master Adam, micro-batch 1 x 2048, as rank 0 of `world` (C4)
``graphs=True`` captures the step as two CUDA graphs — forward + backward, then the optimizer
step — with the U-gate between them (a training loop that is launch-bound in eager mode pays a
saturating D2H twice over: DESIGN.md §8).
"""
from __future__ import annotations

import os
import statistics
import time


def _iter_time(fn, stream, n=10):
    import torch
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    fn()
    a.record(stream)
    for _ in range(n):
        fn()
    b.record(stream)
    b.synchronize()
    return a.elapsed_time(b) / n * 1e-3


def _slice_bytes(pcc, state, chunk_bytes, rank=0, world=1):
    _, _, c = pcc.k_layout(state, 256, chunk_bytes)
    return (((rank + 1) * c) // world - (rank * c) // world) * chunk_bytes


def _auto_pace(pcc, state, chunk_bytes, every, link_gbs, step_fn, stream, rank=0, world=1, graphs=False):
    from paper_conf_asplos_strati0k25_b200.tuner import choose_pace
    t = _iter_time(step_fn, stream)
    choice = choose_pace(_slice_bytes(pcc, state, chunk_bytes, rank, world), every, t, link_gbs, graphs=graphs)
    choice.update(t_iter_s=t, link_gbs=link_gbs)
    return choice["d2h_gbs"], choice["d2h_quantum"], choice


def _pct(v, q):
    v = sorted(v)
    return v[min(len(v) - 1, int(q * len(v)))] if v else None


def run_protocol(ck, stream, fwd_bwd, update, every=10, iters=200, warmup=20, runs=3, host_lead=None,
                 use_guard=True, commit=False, snap_bytes=None):
    """SURVEY §8(d) slowdown protocol on an open, registered ``ck``.  host_lead=k keeps the host
    at most k iterations ahead of the GPU (a loop that reads its loss every k steps); None lets
    it run ahead freely.  Returns the result dict (slowdown %, per-run values, p50/p99, the
    per-position extra ms, the host time of every pcc_checkpoint call, the drain times and the
    contended snapshot rate)."""
    import torch
    host_ms, infos, drain_ms, guard_ms = [], [], [], []

    def loop(n, checkpoint, it0):
        evs = [torch.cuda.Event(enable_timing=True) for _ in range(n + 1)]
        handles = []
        evs[0].record(stream)
        for i in range(1, n + 1):
            if host_lead and i > host_lead:
                evs[i - host_lead].synchronize()
            fwd_bwd()
            if checkpoint and use_guard:
                tg = time.perf_counter()
                ck.guard(stream)
                if i % every == 1 and i > 1:
                    guard_ms.append((time.perf_counter() - tg) * 1e3)
            update()
            if checkpoint and i % every == 0:
                th = time.perf_counter()
                handles.append(ck.checkpoint(it0 + i, stream))
                if commit:
                    ck.commit()  # collective, the same program point on every rank
                host_ms.append((time.perf_counter() - th) * 1e3)
            evs[i].record(stream)
        evs[n].synchronize()
        t_end = time.perf_counter()
        ck.drain()
        if checkpoint:
            drain_ms.append((time.perf_counter() - t_end) * 1e3)
            # the library keeps the newest 64 terminal records queryable (pcc_info); every = 1
            # runs issue more checkpoints than that per loop
            infos.extend(ck.info(h) for h in handles[-48:])
        if commit and handles:
            ck.commit()
        return evs[0].elapsed_time(evs[n]), [evs[i - 1].elapsed_time(evs[i]) for i in range(1, n + 1)]

    loop(warmup, True, 1)  # warm-up: pays first-touch costs of the file pages, events, graphs
    host_ms.clear()
    infos.clear()
    drain_ms.clear()
    guard_ms.clear()
    base_t, ck_t, its_b, its_c = [], [], [], []
    pos_b, pos_c = [[] for _ in range(every)], [[] for _ in range(every)]
    it0 = 1000
    for _ in range(runs):
        t, its = loop(iters, False, 0)
        base_t.append(t)
        its_b += its
        for i, v in enumerate(its):
            pos_b[(i + 1) % every].append(v)
        t, its = loop(iters, True, it0)
        it0 += 10 * iters
        ck_t.append(t)
        its_c += its
        for i, v in enumerate(its):
            pos_c[(i + 1) % every].append(v)
    b, c = statistics.mean(base_t), statistics.mean(ck_t)
    snap = statistics.median(i["snapshot_ms"] for i in infos) if infos else None
    return {
        "every": every, "iters": iters, "warmup": warmup, "runs": runs, "host_lead": host_lead,
        "iter_ms_no_ckpt": b / iters, "iter_ms_ckpt": c / iters,
        "slowdown_pct": (c / b - 1.0) * 100.0,
        "slowdown_pct_runs": [(x / y - 1.0) * 100.0 for x, y in zip(ck_t, base_t)],
        "p50_ms": [_pct(its_b, 0.5), _pct(its_c, 0.5)], "p99_ms": [_pct(its_b, 0.99), _pct(its_c, 0.99)],
        # mean extra ms of iteration i with i % every == k (k = 0: the iteration that issues the
        # checkpoint after its step; k = 1: the next one, whose update waits at the U-gate)
        "extra_ms_by_pos": [statistics.mean(pc) - statistics.mean(pb) for pb, pc in zip(pos_b, pos_c)],
        "host_ckpt_call_ms": statistics.median(host_ms) if host_ms else None,
        "host_ckpt_call_ms_max": max(host_ms) if host_ms else None,
        # the U-gate call right after a checkpoint: host time (it waits only while the packer
        # thread still holds K1 windows of that checkpoint, i.e. the HBM ring was full)
        "host_guard_ms": statistics.median(guard_ms) if guard_ms else None,
        "host_guard_ms_max": max(guard_ms) if guard_ms else None,
        "drain_ms": statistics.median(drain_ms) if drain_ms else None,
        "iters_ms_ckpt_last_run": [round(x, 2) for x in its_c[-iters:]],
        "contended": None if not infos else {
            "checkpoints": len(infos), "k1_busy_ms": statistics.median(i["k1_busy_ms"] for i in infos),
            "pack_span_ms": statistics.median(i["pack_ms"] for i in infos), "snapshot_ms": snap,
            "gbs": snap_bytes / (snap * 1e-3) / 1e9 if snap_bytes and snap else None, "bytes": snap_bytes,
            "def": "K1 start -> last chunk landed in host memory (CUDA events), median over the checkpoints "
                   "taken while training runs"},
    }


def _open(pcc, state, path, chunk_bytes, n_inflight, flags, d2h_gbs, d2h_quantum, dev, rank=0, world=1,
          ck_kwargs=None, ring_bytes=0, pack_ctas=0):
    shm = "/dev/shm" if os.path.isdir("/dev/shm") else "/tmp"
    path = path or os.path.join(shm, f"pcc_slowdown_{os.getpid()}_{time.monotonic_ns()}.pcc")
    ck = pcc.PCCheck(None if flags == pcc.NULLSINK else path, chunk_bytes=chunk_bytes, max_inflight=n_inflight,
                     flags=pcc.MAPFILE if flags is None else flags, ring_bytes=ring_bytes,
                     staging_bytes=8 * chunk_bytes, d2h_gbs=d2h_gbs or 0.0, d2h_quantum=d2h_quantum or 0,
                     device=dev, rank=rank, world=world, pack_ctas=pack_ctas, **(ck_kwargs or {}))
    ck.register(state)
    return ck, path


def _finish(ck, path, res, **extra):
    ck.drain()
    ck.close()
    if path and os.path.exists(path):
        os.unlink(path)
    res.update(extra)
    g = extra.get("d2h_gbs")
    if g and res.get("contended") and res["contended"].get("gbs"):
        # the pace a checkpoint taken while training actually got (choose_pace's rule needs ~1)
        res["pace_delivered_frac"] = res["contended"]["gbs"] / g
    return res


def _graphs(stream, fwd_bwd, update, warm=3):
    """Captures forward + backward and the update as two CUDA graphs (the U-gate sits between
    the replays).  Warm-up on a side stream first, as CUDA graph capture requires."""
    import torch
    s0 = torch.cuda.Stream()
    s0.wait_stream(stream)
    with torch.cuda.stream(s0):
        for _ in range(warm):
            fwd_bwd()
            update()
    stream.wait_stream(s0)
    g_fb, g_up = torch.cuda.CUDAGraph(), torch.cuda.CUDAGraph()
    with torch.cuda.graph(g_fb):
        fwd_bwd()
    with torch.cuda.graph(g_up):
        update()
    return g_fb.replay, g_up.replay


def vgg16_slowdown(pcc, iters=200, every=10, warmup=20, batch=32, runs=3, path=None, n_inflight=2, flags=None,
                   chunk_bytes=64 << 20, graphs=False, d2h_gbs=0.0, d2h_quantum=0, link_gbs=None, rank=0, world=1,
                   ck_kwargs=None, use_guard=True, host_lead=None):
    """world > 1 (every rank calls this at the same point, torch.distributed initialised): data
    parallelism — DistributedDataParallel, batch `batch` per rank — and each rank checkpoints its
    1/world slice of the replicated state, every checkpoint followed by the collective commit
    (allreduce MIN).  d2h_gbs="auto": the tuner's pace (tuner.choose_pace)."""
    import torch
    import torchvision

    torch.manual_seed(0)
    dev = torch.device("cuda", torch.cuda.current_device())
    model = torchvision.models.vgg16(weights=None).to(dev)
    net = model
    if world > 1:
        net = torch.nn.parallel.DistributedDataParallel(model, device_ids=[dev.index])
    opt = torch.optim.SGD(model.parameters(), lr=1e-3, momentum=0.9)
    x = torch.randn(batch, 3, 224, 224, device=dev)
    y = torch.randint(0, 1000, (batch,), device=dev)
    lossf = torch.nn.CrossEntropyLoss()
    stream = torch.cuda.current_stream()

    def fwd_bwd():
        opt.zero_grad(set_to_none=not graphs)
        lossf(net(x), y).backward()

    for _ in range(2):  # momentum buffers exist after the first step
        fwd_bwd()
        opt.step()
    update = opt.step
    if graphs:
        fwd_bwd, update = _graphs(stream, fwd_bwd, update)
    state = []
    for p in model.parameters():
        state += [p.data, opt.state[p]["momentum_buffer"]]
    pace_choice = None
    if d2h_gbs == "auto":
        d2h_gbs, d2h_quantum, pace_choice = _auto_pace(pcc, state, chunk_bytes, every, link_gbs,
                                                       lambda: (fwd_bwd(), update()), stream, rank, world, graphs)
    if flags is None and graphs and not d2h_gbs:  # an unpaced CUDA-graph loop: PCC_D2H_UPFRONT
        flags = pcc.MAPFILE | pcc.D2H_UPFRONT
    ck, path = _open(pcc, state, path, chunk_bytes, n_inflight, flags, d2h_gbs, d2h_quantum, dev.index, rank, world,
                     ck_kwargs)
    nbytes = sum(t.numel() * t.element_size() for t in state)
    res = run_protocol(ck, stream, fwd_bwd, update, every, iters, warmup, runs, host_lead, use_guard, world > 1,
                       nbytes if world == 1 else _slice_bytes(pcc, state, chunk_bytes, rank, world))
    return _finish(ck, path, res,
                   model="vgg16 fp32 SGD(momentum) batch 32, random init, synthetic inputs"
                   + (", step as 2 CUDA graphs (fwd+bwd | optimizer)" if graphs else ", eager")
                   + (f", DDP over {world} ranks (this rank: {rank}; its 1/{world} slice)" if world > 1 else ""),
                   N=n_inflight, graphs=graphs, guard=use_guard, d2h_gbs=d2h_gbs or None,
                   d2h_quantum=d2h_quantum or None, pace_choice=pace_choice, state_bytes=nbytes, tensors=len(state))


def hf_slowdown(pcc, model="bert", iters=200, every=10, warmup=20, runs=3, path=None, n_inflight=2,
                chunk_bytes=64 << 20, d2h_gbs=0.0, d2h_quantum=0, link_gbs=None, flags=None, ring_bytes=0,
                use_guard=True, graphs=False, host_lead=None, pack_ctas=0, upfront=None, rank=0, world=1,
                ck_kwargs=None):
    """model="bert": BERT-large QA (24 layers, hidden 1024), fp32, batch 3 x 384 tokens, Adam(fused);
    model="opt13": OPT-1.3B, fp32 params, Adam(fused), bf16 autocast, batch 1 x 2048 tokens.
    The checkpointed state is R11's registration of the optimizer (param, exp_avg, exp_avg_sq,
    step per parameter).  graphs=True (opt13): capturable fused Adam, explicit attention mask
    (HF's mask helper reads a flag to the host every forward, which capture forbids), sdpa."""
    import torch
    torch.manual_seed(0)
    dev = torch.device("cuda", torch.cuda.current_device())
    if model == "bert":
        from transformers import BertConfig, BertForQuestionAnswering
        cfg = BertConfig(vocab_size=30522, hidden_size=1024, num_hidden_layers=24, num_attention_heads=16,
                         intermediate_size=4096, max_position_embeddings=512)
        net = BertForQuestionAnswering(cfg).to(dev)
        ids = torch.randint(0, cfg.vocab_size, (3, 384), device=dev)
        starts = torch.randint(0, 384, (3,), device=dev)
        ends = torch.randint(0, 384, (3,), device=dev)

        def loss_fn():
            return model_fwd(input_ids=ids, start_positions=starts, end_positions=ends).loss
        desc = "BERT-large QA fp32, Adam(fused), batch 3 x 384 tokens"
    elif model == "opt13":
        from transformers import OPTConfig, OPTForCausalLM
        cfg = OPTConfig(hidden_size=2048, num_hidden_layers=24, ffn_dim=8192, num_attention_heads=32,
                        vocab_size=50272, max_position_embeddings=2048, word_embed_proj_dim=2048)
        if graphs:
            cfg._attn_implementation = "sdpa"
        net = OPTForCausalLM(cfg).to(dev)
        ids = torch.randint(0, cfg.vocab_size, (1, 2048), device=dev)
        mask = torch.ones(1, 2048, dtype=torch.long, device=dev)

        def loss_fn():
            with torch.autocast("cuda", dtype=torch.bfloat16, cache_enabled=not graphs):
                return model_fwd(input_ids=ids, attention_mask=mask if graphs else None, labels=ids).loss
        desc = "OPT-1.3B fp32 params, Adam(fused), bf16 autocast, batch 1 x 2048 tokens"
    else:
        raise ValueError(model)
    net.train()
    opt = torch.optim.Adam(net.parameters(), lr=1e-5, fused=True, capturable=graphs)
    if world > 1:  # data parallelism: DDP allreduces the gradients, the state stays replicated
        if graphs:
            raise ValueError("world > 1 runs eager (DDP)")
        ddp = torch.nn.parallel.DistributedDataParallel(net, device_ids=[dev.index])
        model_fwd = ddp
    else:
        model_fwd = net
    stream = torch.cuda.current_stream()

    def fwd_bwd():
        opt.zero_grad(set_to_none=not graphs)
        loss_fn().backward()

    for _ in range(2):  # Adam state exists after the first step
        fwd_bwd()
        opt.step()
    update = opt.step
    if graphs:
        fwd_bwd, update = _graphs(stream, fwd_bwd, update)
    state, _ = pcc.state_tensors(opt)
    pace_choice = None
    if d2h_gbs == "auto":
        d2h_gbs, d2h_quantum, pace_choice = _auto_pace(pcc, state, chunk_bytes, every, link_gbs,
                                                       lambda: (fwd_bwd(), update()), stream, rank, world, graphs)
    if upfront is None:  # default: an unpaced CUDA-graph loop enqueues the D2H with K1
        upfront = graphs and not d2h_gbs
    if flags is None and upfront:  # PCC_D2H_UPFRONT (unpaced by construction)
        flags, d2h_gbs, d2h_quantum = pcc.MAPFILE | pcc.D2H_UPFRONT, 0.0, 0
    ck, path = _open(pcc, state, path, chunk_bytes, n_inflight, flags, d2h_gbs, d2h_quantum, dev.index, rank, world,
                     ck_kwargs, ring_bytes=ring_bytes, pack_ctas=pack_ctas)
    nbytes = sum(t.numel() * t.element_size() for t in state)
    res = run_protocol(ck, stream, fwd_bwd, update, every, iters, warmup, runs, host_lead, use_guard, world > 1,
                       nbytes if world == 1 else _slice_bytes(pcc, state, chunk_bytes, rank, world))
    return _finish(ck, path, res, model=desc + ", random init, synthetic inputs"
                   + (", step as 2 CUDA graphs (fwd+bwd | optimizer)" if graphs else ", eager")
                   + (f", DDP over {world} ranks (this rank: {rank}; its 1/{world} slice)" if world > 1 else ""),
                   N=n_inflight, graphs=graphs, guard=use_guard, d2h_gbs=d2h_gbs or None,
                   d2h_quantum=d2h_quantum or None, pace_choice=pace_choice, state_bytes=nbytes, tensors=len(state),
                   ring_bytes=ring_bytes or None, d2h_upfront=bool(flags and flags & pcc.D2H_UPFRONT),
                   pack_ctas=pack_ctas or None)


def bloom_slowdown(pcc, world=8, iters=200, every=10, warmup=20, runs=3, seq=2048, path=None, d2h_gbs=0.0,
                   d2h_quantum=0, link_gbs=None):
    """BLOOM-7b1 (BASELINE configs[3]) on ONE B200 as a proxy for one rank of a world-`world`
    data-parallel job: the per-GPU compute of DP at micro-batch 1 (forward + backward of the
    full model on one 2048-token sequence, then a mixed-precision Adam step), checkpointing
    only this rank's 1/world slice (PCC_NOCOMM) every `every` iterations.  What it cannot
    show: the gradient allreduce of real DP and W ranks contending for host DRAM.
    State per parameter (R11, R12): bf16 param, fp32 master, exp_avg, exp_avg_sq, 0-d fp32 step."""
    import torch
    from transformers import BloomConfig, BloomForCausalLM

    torch.manual_seed(0)
    cfg = BloomConfig(vocab_size=250880, hidden_size=4096, n_layer=30, n_head=32)
    with torch.device("cuda"):
        model = BloomForCausalLM(cfg).to(torch.bfloat16)
    params = list(model.parameters())
    master = [p.detach().float() for p in params]
    exp_avg = [torch.zeros_like(m) for m in master]
    exp_avg_sq = [torch.zeros_like(m) for m in master]
    steps = [torch.zeros((), dtype=torch.float32, device="cuda") for _ in params]
    state = []
    for p, m, a, b, st in zip(params, master, exp_avg, exp_avg_sq, steps):
        state += [p.data, m, a, b, st]
    ids = torch.randint(0, cfg.vocab_size, (1, seq), device="cuda")
    stream = torch.cuda.current_stream()
    lr, b1, b2, eps = 1e-5, 0.9, 0.95, 1e-8

    def fwd_bwd():
        for p in params:
            p.grad = None
        model(input_ids=ids, labels=ids).loss.backward()

    @torch.no_grad()
    def adam_step():  # mixed-precision Adam (no bias correction), one parameter at a time
        for p, m, a, b, st in zip(params, master, exp_avg, exp_avg_sq, steps):
            g = p.grad.float()
            st.add_(1.0)
            a.lerp_(g, 1 - b1)
            b.mul_(b2).addcmul_(g, g, value=1 - b2)
            m.addcdiv_(a, b.sqrt().add_(eps), value=-lr)
            p.copy_(m)

    for _ in range(2):
        fwd_bwd()
        adam_step()
    pace_choice = None
    if d2h_gbs == "auto":
        d2h_gbs, d2h_quantum, pace_choice = _auto_pace(pcc, state, 64 << 20, every, link_gbs,
                                                       lambda: (fwd_bwd(), adam_step()), stream, 0, world)
    ck, path = _open(pcc, state, path, 64 << 20, 2, pcc.MAPFILE | pcc.NOCOMM, d2h_gbs, d2h_quantum, 0, 0, world)
    geo = ck.geometry()
    slice_bytes = geo["count"] * (64 << 20)
    res = run_protocol(ck, stream, fwd_bwd, adam_step, every, iters, warmup, runs, None, True, True, slice_bytes)
    return _finish(ck, path, res,
                   model=f"bloom-7b1 bf16 + fp32 master Adam, micro-batch 1 x {seq} tokens, random init; "
                         f"1 GPU playing rank 0 of world {world} (checkpoints its 1/{world} slice)",
                   slice_chunks=geo["count"], slice_bytes=slice_bytes, d2h_gbs=d2h_gbs or None,
                   d2h_quantum=d2h_quantum or None, pace_choice=pace_choice,
                   state_bytes=sum(t.numel() * t.element_size() for t in state))


if __name__ == "__main__":
    import argparse
    import json
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    ap = argparse.ArgumentParser()
    ap.add_argument("model", choices=["vgg16", "bert", "opt13", "bloom"])
    ap.add_argument("--graphs", action="store_true")
    ap.add_argument("--pace", default="0", help="GB/s, 'auto' (tuner) or 0 (unpaced)")
    ap.add_argument("--iters", type=int, default=200)
    ap.add_argument("--runs", type=int, default=3)
    ap.add_argument("--every", type=int, default=10)
    ap.add_argument("--host-lead", type=int, default=0)
    ap.add_argument("--link-gbs", type=float, default=55.0)
    ap.add_argument("--inflight", type=int, default=2)
    ap.add_argument("--pack-ctas", type=int, default=0)
    ap.add_argument("--no-upfront", action="store_true", help="graphs: keep the orchestrator-issued (pace-able) D2H")
    ap.add_argument("--quantum-kib", type=int, default=512)
    ap.add_argument("--unpaced-quantum-kib", type=int, default=0, help="copy size of an unpaced D2H (0 = whole chunk groups)")
    ap.add_argument("--ring-slices", type=float, default=0, help="HBM ring in slices (0 = one slice)")
    a = ap.parse_args()
    import paper_conf_asplos_strati0k25_b200 as pcc
    pace = a.pace if a.pace == "auto" else float(a.pace)
    kw = dict(iters=a.iters, runs=a.runs, every=a.every, d2h_gbs=pace, link_gbs=a.link_gbs)
    if a.model == "vgg16":
        r = vgg16_slowdown(pcc, graphs=a.graphs, host_lead=a.host_lead or None, **kw)
    elif a.model == "bloom":
        r = bloom_slowdown(pcc, **kw)
    else:
        ring = 0
        if a.ring_slices:
            from synth import config_tensors
            nb = sum(t.nbytes for t in config_tensors({"opt13": "c3", "bert": "bert"}[a.model]))
            ring = int(a.ring_slices * -(-nb // (64 << 20))) * (64 << 20)
        r = hf_slowdown(pcc, a.model, graphs=a.graphs, host_lead=a.host_lead or None, n_inflight=a.inflight,
                        ring_bytes=ring, pack_ctas=a.pack_ctas, upfront=False if a.no_upfront else None,
                        d2h_quantum=(a.quantum_kib << 10) if pace else (a.unpaced_quantum_kib << 10), **kw)
    print(json.dumps(r))
