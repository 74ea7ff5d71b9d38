"""Training-iteration slowdown with a checkpoint every `every` iterations vs none
(BASELINE.json metric, second half).

Random-init torchvision VGG-16, fp32, SGD(momentum=0.9), batch 32 of random 3x224x224
images with random labels (PAPER Table 3: VGG16, batch 32).  The checkpointed state
is every parameter and its momentum buffer (R11).  Per iteration: forward + backward, then
pcc_guard (the U-gate of L139: the update must not overwrite the state K1 is still
reading), then optimizer.step(); after the step of every `every`-th iteration,
pcc_checkpoint(iter).  Both runs use the same model, inputs and iteration count; time is
measured with CUDA events around the whole loop.
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


def _auto_pace(pcc, state, chunk_bytes, every, link_gbs, step_fn, stream, rank=0, world=1):
    from paper_conf_asplos_strati0k25_b200.tuner import choose_pace
    t = _iter_time(step_fn, stream)
    choice = choose_pace(_slice_bytes(pcc, state, chunk_bytes, rank, world), every, t, link_gbs)
    choice.update(t_iter_s=t, link_gbs=link_gbs)
    return choice["d2h_gbs"], choice["d2h_quantum"], choice


def vgg16_slowdown(pcc, iters=60, every=10, warmup=10, batch=32, runs=2, path=None, n_inflight=2, flags=None,
                   chunk_bytes=64 << 20, writer_threads=4, staging_bytes=0, pack_ctas=0, use_guard=True,
                   graphs=False, d2h_gbs=0.0, d2h_quantum=0, link_gbs=None, rank=0, world=1, ck_kwargs=None):
    """graphs=True: the training step runs as two CUDA graphs (forward + backward, then the
    optimizer step) with the U-gate between them; False: eager PyTorch.  d2h_gbs="auto": the
    tuner's D2H pace (tuner.choose_pace) for `every` x the measured iteration time and the
    D2H link peak `link_gbs`.

    world > 1 (every rank calls this at the same point, torch.distributed initialised): data
    parallelism — DistributedDataParallel over the default process group, batch `batch` per rank
    — and the library at (rank, world): each rank checkpoints its 1/world slice of the replicated
    state and every checkpoint is followed by the collective commit (allreduce MIN).
    ck_kwargs: the collectives for PCCheck (allreduce / allgather callbacks or nccl_unique_id)."""
    import torch
    import torchvision

    torch.manual_seed(0)
    dev = torch.device("cuda", torch.cuda.current_device())
    model = torchvision.models.vgg16(weights=None).to(dev)
    net = model
    if world > 1:  # DP: gradients allreduced by DDP, parameters / momenta stay replicated
        net = torch.nn.parallel.DistributedDataParallel(model, device_ids=[dev.index])
    opt = torch.optim.SGD(model.parameters(), lr=1e-3, momentum=0.9)
    x = torch.randn(batch, 3, 224, 224, device=dev)
    y = torch.randint(0, 1000, (batch,), device=dev)
    lossf = torch.nn.CrossEntropyLoss()
    stream = torch.cuda.current_stream()

    def step():
        opt.zero_grad(set_to_none=True)
        lossf(net(x), y).backward()

    for _ in range(2):  # momentum buffers exist after the first step
        step()
        opt.step()
    update = opt.step
    if graphs:
        s0 = torch.cuda.Stream()
        s0.wait_stream(stream)
        with torch.cuda.stream(s0):  # warm-up on a side stream before capture
            for _ in range(3):
                step()
                opt.step()
        stream.wait_stream(s0)
        g_fb, g_up = torch.cuda.CUDAGraph(), torch.cuda.CUDAGraph()
        opt.zero_grad(set_to_none=True)
        with torch.cuda.graph(g_fb):
            lossf(net(x), y).backward()
        with torch.cuda.graph(g_up):
            opt.step()
        step, update = g_fb.replay, g_up.replay
    state = []
    for p in model.parameters():
        state += [p.data, opt.state[p]["momentum_buffer"]]
    pace_choice = None
    if d2h_gbs == "auto":  # the tuner's pace for this interval (iteration time measured here)
        d2h_gbs, d2h_quantum, pace_choice = _auto_pace(pcc, state, chunk_bytes, every, link_gbs,
                                                       lambda: (step(), update()), stream, rank, world)
    shm = "/dev/shm" if os.path.isdir("/dev/shm") else "/tmp"
    path = path or os.path.join(shm, f"pcc_slowdown_{os.getpid()}.pcc")
    ck = pcc.PCCheck(path, chunk_bytes=chunk_bytes, max_inflight=n_inflight,
                     flags=pcc.MAPFILE if flags is None else flags, writer_threads=writer_threads,
                     staging_bytes=staging_bytes, pack_ctas=pack_ctas, d2h_gbs=d2h_gbs, d2h_quantum=d2h_quantum,
                     device=dev.index, rank=rank, world=world, **(ck_kwargs or {}))
    ck.register(state)
    host_ms = []
    infos = []  # the checkpoints taken while training runs (contended)

    def loop(n, checkpoint, it0):
        handles = []
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        per = []
        e0.record(stream)
        last = e0
        for i in range(1, n + 1):
            step()
            if checkpoint and use_guard:
                ck.guard(stream)
            update()
            if checkpoint and i % every == 0:
                th = time.perf_counter()
                handles.append(ck.checkpoint(it0 + i, stream))
                if world > 1:
                    ck.commit()  # collective, same program point on every rank
                host_ms.append((time.perf_counter() - th) * 1e3)
            ev = torch.cuda.Event(enable_timing=True)
            ev.record(stream)
            per.append((last, ev))
            last = ev
        e1.record(stream)
        e1.synchronize()
        total = e0.elapsed_time(e1)
        for h in handles:
            ck.wait(h)
            infos.append(ck.info(h))
        if world > 1 and handles:
            ck.commit()
        its = [a.elapsed_time(b) for a, b in per]  # iteration i+1 at index i
        return total, its

    loop(warmup, False, 0)
    base_t, ck_t, its_b, its_c = [], [], [], []
    pos_b, pos_c = [[] for _ in range(every)], [[] for _ in range(every)]
    it0 = 1000
    for r in range(runs):
        t, its = loop(iters, False, 0)
        base_t.append(t)
        its_b += its
        for i, v in enumerate(its):
            pos_b[(i + 1) % every].append(v)
        t, its = loop(iters, True, it0)
        it0 += 1000
        ck_t.append(t)
        its_c += its
        for i, v in enumerate(its):
            pos_c[(i + 1) % every].append(v)
    ck.drain()
    ck.close()
    if os.path.exists(path):
        os.unlink(path)
    b, c = statistics.mean(base_t), statistics.mean(ck_t)
    pct = lambda v, q: sorted(v)[min(len(v) - 1, int(q * len(v)))]  # noqa: E731
    return {"model": "vgg16 fp32 SGD(momentum) batch 32, random init, synthetic inputs"
                     + (", training step as CUDA graphs" if graphs else ", eager")
                     + (f", DDP over {world} ranks (this rank: {rank}; its 1/{world} slice)" if world > 1 else ""),
            "every": every, "iters": iters, "runs": runs, "N": n_inflight,
            "iter_ms_no_ckpt": b / iters, "iter_ms_ckpt": c / iters,
            "slowdown_pct": (c / b - 1.0) * 100.0,
            # mean extra ms of iteration i % every == k (k = 0: the iteration that issues the
            # checkpoint after its step; k = 1: the next one, which overlaps K1)
            "extra_ms_by_pos": [statistics.mean(pc) - statistics.mean(pb) for pb, pc in zip(pos_b, pos_c)],
            "host_ckpt_call_ms": statistics.median(host_ms) if host_ms else None,
            "pack_ctas": pack_ctas, "guard": use_guard, "graphs": graphs,
            "d2h_gbs": d2h_gbs or None, "d2h_quantum": d2h_quantum or None, "pace_choice": pace_choice,
            "p50_ms": [pct(its_b, 0.5), pct(its_c, 0.5)], "p99_ms": [pct(its_b, 0.99), pct(its_c, 0.99)],
            "state_bytes": sum(t.numel() * t.element_size() for t in state),
            # this rank's bytes: the whole state at W = 1, its slice (padded chunks) at W > 1
            "contended": _contended(infos, sum(t.numel() * t.element_size() for t in state) if world == 1
                                    else _slice_bytes(pcc, state, chunk_bytes, rank, world))}


def _contended(infos, nbytes):
    """the snapshot measured while training runs, medians over the checkpoints, on
    the GPU's clock: K1 alone, the U-gate span, and K1 start -> last chunk landed in host memory
    (paced when a D2H pace is set)."""
    if not infos:
        return None
    snap = statistics.median(i["snapshot_ms"] for i in infos)
    return {"checkpoints": len(infos), "k1_busy_ms": statistics.median(i["k1_busy_ms"] for i in infos),
            "pack_span_ms": statistics.median(i["pack_ms"] for i in infos), "snapshot_ms": snap,
            "gbs": nbytes / (snap * 1e-3) / 1e9, "bytes": nbytes}


def bloom_slowdown(pcc, world=8, iters=40, every=10, warmup=4, seq=2048, runs=1, path=None, d2h_gbs=0.0,
                   d2h_quantum=0, link_gbs=None):
    """BLOOM-7b1 (BASELINE configs[3]) on ONE B200 as a proxy for one rank of a world-`world`
    data-parallel job: the per-GPU compute of DP at micro-batch 1 (forward + backward of the
    full model on one 2048-token sequence, then a mixed-precision Adam step), checkpointing
    only this rank's 1/world slice (PCC_NOCOMM) every `every` iterations.  What it cannot
    show: the gradient allreduce of real DP and W ranks contending for host DRAM.

    State per parameter (R11, R12): bf16 param, fp32 master, fp32 exp_avg, fp32 exp_avg_sq,
    0-d fp32 step — 1825 tensors, 98.97 GB.  Random init, random token ids."""
    import torch
    from transformers import BloomConfig, BloomForCausalLM

    torch.manual_seed(0)
    cfg = BloomConfig(vocab_size=250880, hidden_size=4096, n_layer=30, n_head=32)
    with torch.device("cuda"):
        model = BloomForCausalLM(cfg).to(torch.bfloat16)
    params = [p for p in model.parameters()]
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
    def adam_step():  # mixed-precision Adam (no bias correction), one parameter at a time: no fp32 grad copy
        for p, m, a, b, st in zip(params, master, exp_avg, exp_avg_sq, steps):
            g = p.grad.float()
            st.add_(1.0)
            a.lerp_(g, 1 - b1)
            b.mul_(b2).addcmul_(g, g, value=1 - b2)
            m.addcdiv_(a, b.sqrt().add_(eps), value=-lr)
            p.copy_(m)

    for _ in range(warmup):
        fwd_bwd()
        adam_step()
    pace_choice = None
    if d2h_gbs == "auto":
        d2h_gbs, d2h_quantum, pace_choice = _auto_pace(pcc, state, 64 << 20, every, link_gbs,
                                                       lambda: (fwd_bwd(), adam_step()), stream, 0, world)
    shm = "/dev/shm" if os.path.isdir("/dev/shm") else "/tmp"
    path = path or os.path.join(shm, f"pcc_bloom_{os.getpid()}.pcc")
    ck = pcc.PCCheck(path, chunk_bytes=64 << 20, max_inflight=2, flags=pcc.MAPFILE | pcc.NOCOMM, rank=0, world=world,
                     d2h_gbs=d2h_gbs, d2h_quantum=d2h_quantum)
    ck.register(state)
    geo = ck.geometry()
    infos = []

    def loop(n, checkpoint, it0):
        handles = []
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        per = []
        e0.record(stream)
        last = e0
        for i in range(1, n + 1):
            fwd_bwd()
            if checkpoint:
                ck.guard(stream)  # U-gate (L139): the update must not race K1
            adam_step()
            if checkpoint and i % every == 0:
                handles.append(ck.checkpoint(it0 + i, stream))
                ck.commit()
            ev = torch.cuda.Event(enable_timing=True)
            ev.record(stream)
            per.append((last, ev))
            last = ev
        e1.record(stream)
        e1.synchronize()
        for h in handles:
            ck.wait(h)
            infos.append(ck.info(h))
        return e0.elapsed_time(e1), sorted(a.elapsed_time(b) for a, b in per)

    base_t, ck_t, its_b, its_c = [], [], [], []
    it0 = 1000
    for r in range(runs):
        t, its = loop(iters, False, 0)
        base_t.append(t)
        its_b += its
        t, its = loop(iters, True, it0)
        it0 += 1000
        ck_t.append(t)
        its_c += its
    ck.drain()
    ck.close()
    if os.path.exists(path):
        os.unlink(path)
    b, c = statistics.mean(base_t), statistics.mean(ck_t)
    pct = lambda v, q: sorted(v)[min(len(v) - 1, int(q * len(v)))]  # noqa: E731
    return {"model": f"bloom-7b1 bf16 + fp32 master Adam, micro-batch 1 x {seq} tokens, random init; "
                     f"1 GPU playing rank 0 of world {world} (checkpoints its 1/{world} slice)",
            "every": every, "iters": iters, "runs": runs, "slice_chunks": geo["count"],
            "slice_bytes": geo["count"] * (64 << 20),
            "iter_ms_no_ckpt": b / iters, "iter_ms_ckpt": c / iters, "slowdown_pct": (c / b - 1.0) * 100.0,
            "p50_ms": [pct(its_b, 0.5), pct(its_c, 0.5)], "p99_ms": [pct(its_b, 0.99), pct(its_c, 0.99)],
            "d2h_gbs": d2h_gbs or None, "d2h_quantum": d2h_quantum or None, "pace_choice": pace_choice,
            "state_bytes": sum(t.numel() * t.element_size() for t in state),
            "contended": _contended(infos, geo["count"] * (64 << 20))}


def hf_slowdown(pcc, model="bert", iters=40, every=10, warmup=5, runs=1, path=None, n_inflight=2,
                chunk_bytes=64 << 20, d2h_gbs=0.0, d2h_quantum=0, link_gbs=None, flags=None, ring_bytes=0,
                use_guard=True):
    """The same measurement for two more of north_star's models, random init, synthetic inputs:

    * model="bert": BERT-large with a QA head (BertForQuestionAnswering, 24 layers, hidden 1024),
      fp32, batch 3 (PAPER Table 3) x 384 tokens (SQuAD's usual length; the paper is
      silent), Adam(fused) — the "BERT 4 GB" checkpoint of Table 3;
    * model="opt13": OPT-1.3B (OPTForCausalLM), fp32 params, Adam(fused), bf16
      autocast, batch 1 (Table 3) x 2048 tokens.

    The checkpointed state is R11's registration of the optimizer (`state_tensors`): param,
    exp_avg, exp_avg_sq, step per parameter.  Per iteration: forward + backward, pcc_guard (the
    U-gate of L139), optimizer.step(); every `every`-th iteration, pcc_checkpoint."""
    import torch
    torch.manual_seed(0)
    dev = torch.device("cuda", torch.cuda.current_device())
    if model == "bert":
        from transformers import BertConfig, BertForQuestionAnswering
        cfg = BertConfig(vocab_size=30522, hidden_size=1024, num_hidden_layers=24, num_attention_heads=16,
                         intermediate_size=4096, max_position_embeddings=512)
        net = BertForQuestionAnswering(cfg).to(dev)
        batch, seq, amp = 3, 384, False
        ids = torch.randint(0, cfg.vocab_size, (batch, seq), device=dev)
        starts = torch.randint(0, seq, (batch,), device=dev)
        ends = torch.randint(0, seq, (batch,), device=dev)

        def fwd_bwd():
            net(input_ids=ids, start_positions=starts, end_positions=ends).loss.backward()
        desc = "BERT-large QA fp32, Adam(fused), batch 3 x 384 tokens"
    elif model == "opt13":
        from transformers import OPTConfig, OPTForCausalLM
        cfg = OPTConfig(hidden_size=2048, num_hidden_layers=24, ffn_dim=8192, num_attention_heads=32,
                        vocab_size=50272, max_position_embeddings=2048, word_embed_proj_dim=2048)
        net = OPTForCausalLM(cfg).to(dev)
        batch, seq, amp = 1, 2048, True
        ids = torch.randint(0, cfg.vocab_size, (batch, seq), device=dev)

        def fwd_bwd():
            with torch.autocast("cuda", dtype=torch.bfloat16):
                loss = net(input_ids=ids, labels=ids).loss
            loss.backward()
        desc = "OPT-1.3B fp32 params, Adam(fused), bf16 autocast, batch 1 x 2048 tokens"
    else:
        raise ValueError(model)
    net.train()
    opt = torch.optim.Adam(net.parameters(), lr=1e-5, fused=True)
    stream = torch.cuda.current_stream()

    def step():
        opt.zero_grad(set_to_none=True)
        fwd_bwd()

    for _ in range(2):  # Adam state exists after the first step
        step()
        opt.step()
    state, _ = pcc.state_tensors(opt)
    pace_choice = None
    if d2h_gbs == "auto":
        d2h_gbs, d2h_quantum, pace_choice = _auto_pace(pcc, state, chunk_bytes, every, link_gbs,
                                                       lambda: (step(), opt.step()), stream)
    shm = "/dev/shm" if os.path.isdir("/dev/shm") else "/tmp"
    path = path or os.path.join(shm, f"pcc_slowdown_{model}_{os.getpid()}.pcc")
    ck = pcc.PCCheck(None if flags == pcc.NULLSINK else path, chunk_bytes=chunk_bytes, max_inflight=n_inflight,
                     flags=pcc.MAPFILE if flags is None else flags, ring_bytes=ring_bytes,
                     staging_bytes=8 * chunk_bytes, d2h_gbs=d2h_gbs, d2h_quantum=d2h_quantum, device=dev.index)
    ck.register(state)
    infos = []

    def loop(n, checkpoint, it0):
        handles = []
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        per = []
        e0.record(stream)
        last = e0
        for i in range(1, n + 1):
            step()
            if checkpoint and use_guard:
                ck.guard(stream)
            opt.step()
            if checkpoint and i % every == 0:
                th = time.perf_counter()
                handles.append(ck.checkpoint(it0 + i, stream))
                host_ms.append((time.perf_counter() - th) * 1e3)
            ev = torch.cuda.Event(enable_timing=True)
            ev.record(stream)
            per.append((last, ev))
            last = ev
        e1.record(stream)
        e1.synchronize()
        for h in handles:
            ck.wait(h)
            infos.append(ck.info(h))
        its = [a.elapsed_time(b) for a, b in per]
        if checkpoint:
            by_pos.append(its)
        return e0.elapsed_time(e1), sorted(its)

    host_ms, by_pos = [], []
    loop(warmup, False, 0)
    base_t, ck_t, its_b, its_c = [], [], [], []
    it0 = 1000
    for r in range(runs):
        t, its = loop(iters, False, 0)
        base_t.append(t)
        its_b += its
        t, its = loop(iters, True, it0)
        it0 += 1000
        ck_t.append(t)
        its_c += its
    ck.drain()
    ck.close()
    if os.path.exists(path):
        os.unlink(path)
    b, c = statistics.mean(base_t), statistics.mean(ck_t)
    pct = lambda v, q: sorted(v)[min(len(v) - 1, int(q * len(v)))]  # noqa: E731
    nbytes = sum(t.numel() * t.element_size() for t in state)
    return {"model": desc + ", random init, synthetic inputs, eager", "every": every, "iters": iters, "runs": runs,
            "N": n_inflight, "tensors": len(state), "state_bytes": nbytes,
            "iter_ms_no_ckpt": b / iters, "iter_ms_ckpt": c / iters, "slowdown_pct": (c / b - 1.0) * 100.0,
            "p50_ms": [pct(its_b, 0.5), pct(its_c, 0.5)], "p99_ms": [pct(its_b, 0.99), pct(its_c, 0.99)],
            "d2h_gbs": d2h_gbs or None, "d2h_quantum": d2h_quantum or None, "pace_choice": pace_choice,
            "host_ckpt_call_ms": statistics.median(host_ms) if host_ms else None,
            "host_ckpt_call_ms_max": max(host_ms) if host_ms else None,
            "iter_ms_ckpt_run": by_pos[-1] if by_pos else None,
            "contended": _contended(infos, nbytes)}
