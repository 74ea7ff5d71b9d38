"""Configuration tuner — PAPER.md §3.4 (L170-L217), SURVEY §8(f) f1.

Given the checkpoint size m, the storage budget S, the iteration time t and the accepted
overhead q, PCcheck's tool "initiates a checkpoint every t seconds.  It then varies N in
[1, S/m - 1], measures T_w for each checkpoint, and finds the optimal N" (L215) minimising
T_w / N, then sets the checkpoint interval (Eq 3; reading R14: ceiling)

    f* = ceil( T_w / (N* * q * t) ).

Here T_w of one checkpoint is measured by the library itself (pcc_info: pcc_checkpoint call
-> local commit) while N checkpoints are kept in flight at a cadence of one every t seconds.

On B200 the tool also picks the D2H pace (pcc_config d2h_mbps / d2h_quantum): a saturating
copy-engine burst slows a training loop while it lasts, and small paced copies hide most of it
(`choose_pace`, measured rule in its docstring).  It also picks the buffer size b from T_G
(`choose_chunk`, L176) and where K1 puts the chunks under an HBM budget (`choose_ring`).
"""
from __future__ import annotations

import math
import statistics
import time


def choose(tw_by_n: dict, q: float, t: float) -> dict:
    """The decision rule alone: N* = argmin T_w(N)/N, f* = ceil(T_w(N*) / (N* q t))."""
    if not tw_by_n:
        raise ValueError("no measurements")
    n_star = min(tw_by_n, key=lambda n: (tw_by_n[n] / n, n))
    tw = tw_by_n[n_star]
    return {"N": n_star, "Tw": tw, "f": max(1, math.ceil(tw / (n_star * q * t)))}


def measure_tw(ck, n_inflight: int, t: float, probes: int = 4, step=None, it0: int = 1) -> float:
    """Issue a checkpoint every t seconds (or after each call of `step`), at most n_inflight
    outstanding; return the median T_w (seconds) of the last `probes` checkpoints."""
    outstanding, tws = [], []

    def retire():
        h = outstanding.pop(0)
        ck.wait(h)
        inf = ck.info(h)
        tws.append((inf["t_committed_us"] - inf["t_call_us"]) * 1e-6)

    it = it0
    for _ in range(n_inflight + probes):
        t0 = time.perf_counter()
        if len(outstanding) >= n_inflight:
            retire()
        outstanding.append(ck.checkpoint(it))
        ck.guard()
        it += 1
        if step is not None:
            step()
        else:
            dt = t - (time.perf_counter() - t0)
            if dt > 0:
                time.sleep(dt)
    while outstanding:
        retire()
    return statistics.median(tws[-probes:])


def tune(make_ctx, m_bytes: int, S_bytes: int, t: float, q: float, n_max: int = 8, probes: int = 4,
         step=None) -> dict:
    """make_ctx(N) -> a registered PCCheck with max_inflight=N (closed by the tuner).
    Sweeps N in [1, min(S/m - 1, n_max)] (L176: N <= S/m - 1)."""
    n_hi = max(1, min(n_max, S_bytes // max(1, m_bytes) - 1))
    tw = {}
    for n in range(1, n_hi + 1):
        ck = make_ctx(n)
        try:
            tw[n] = measure_tw(ck, n, t, probes=probes, step=step)
        finally:
            ck.close()
    out = choose(tw, q, t)
    out["Tw_by_N"] = tw
    out["t"] = t
    out["q"] = q
    return out


D2H_QUANTUM = 1 << 20    # bytes per paced copy (1 MiB: r02 sweeps, eager and graphs)
EAGER_MARGIN, EAGER_CAP = 0.9, 0.7   # eager loop: land within 0.9 of the interval, pace <= 0.7 x link
GRAPH_MARGIN, GRAPH_CAP = 0.85, 0.85  # CUDA-graph loop
GRAPH_QUANTUM = D2H_QUANTUM
UNPACED_EAGER_QUANTUM = 1 << 20  # unpaced copies under an eager loop (the runtime then drains every 16 MiB)


def choose_pace(slice_bytes: int, f: int, t: float, link_gbs: float, n_inflight: int = 2,
                graphs: bool = False) -> dict:
    """D2H pace for training: {"d2h_gbs": G, "d2h_quantum": Q, "need_gbs": ...}; G = 0 = unpaced.

    The gentlest pace that lands one checkpoint within a margin of its interval f*t, never below
    half the link nor above a cap of it, in 1 MiB copies; unpaced when even the capped pace
    would not land the checkpoint within its interval.  The
    rule is the measured one (round 2, after the pacer was fixed to deliver its rate — the
    round-1 sweeps ran at ~1/3 of their nominal pace):

    * CUDA-graph loop (OPT-1.3B, 15.8 GB every 10 x 51.7 ms, profiles/r02_graph_pace_quantum.jsonl):
      unpaced 3.9%; 35 / 45 GB/s in 1 MiB copies 1.1 / 1.8%; 4 MiB copies 3.0-3.3%.  A replay pays
      per byte in flight on the link, so a long gentle transfer in small copies is cheap:
      margin 0.85, cap 0.85 of the link.
    * eager loop (OPT-1.3B, 10 x 44 ms, profiles/r02_eager_pace.jsonl): unpaced 18.9% (in 64 MiB
      copies; 1 MiB copies, draining every 16 MiB: 7.6%, which is what an unpaced eager choice
      gets); 40 GB/s in
      1 MiB copies 6.5%; 50 GB/s 63% — near the link the copy queue never runs dry and the
      training's own small D2H (HF's per-forward flag read) waits behind it (the r01 starvation);
      256 KiB copies: the host cannot keep the cadence (0.57 of the pace delivered).  Margin 0.9,
      cap 0.7 of the link.
    n_inflight: a pace that lands after 0.5 of the interval overlaps the next checkpoint's K1 only
    when N >= 2 lets it start (the bench and the harness run N >= 2)."""
    if f <= 0 or t <= 0 or link_gbs <= 0:
        raise ValueError("f, t and link_gbs must be positive")
    margin, cap = (GRAPH_MARGIN, GRAPH_CAP) if graphs else (EAGER_MARGIN, EAGER_CAP)
    if n_inflight < 2:
        margin = min(margin, 0.5)
    need = slice_bytes / (margin * f * t) / 1e9  # GB/s to land a checkpoint in margin * f * t
    g = min(max(need, 0.5 * link_gbs), cap * link_gbs)
    if slice_bytes / (g * 1e9) > f * t:  # even the capped pace outlasts the interval: unpaced
        # ... but an eager loop still gets 1 MiB copies: its extra time per burst iteration
        # follows the copy size (OPT-1.3B unpaced: 20.8% in 64 MiB copies, 8.8% in 1 MiB;
        # profiles/r02e2_eager_piece.jsonl).  A CUDA-graph loop keeps whole chunk groups.
        return {"d2h_gbs": 0.0, "d2h_quantum": 0 if graphs else UNPACED_EAGER_QUANTUM, "need_gbs": need}
    return {"d2h_gbs": g, "d2h_quantum": D2H_QUANTUM, "need_gbs": need}


# ------------------------------------------------------------------ buffer size b (L176, T_G)
def choose_chunk(tg_by_b: dict, state_bytes: int, tol: float = 0.97) -> dict:
    """b "chosen by the tool based on T_G" (L176): tg_by_b maps a candidate chunk size b (bytes)
    to the measured GPU->host throughput T_G(b) (GB/s) when the transfer moves b-byte pieces.
    The image is zero-padded to whole chunks (R3), so the useful rate is
        eff(b) = T_G(b) * state_bytes / (ceil(state_bytes / b) * b).
    Returns the SMALLEST b whose eff is within `tol` of the best (smaller chunks pipeline the
    persist sooner, hold less staging, and pay less padding)."""
    if not tg_by_b or state_bytes <= 0:
        raise ValueError("need measurements and a positive state size")

    def eff(b):
        c = -(-state_bytes // b)
        return tg_by_b[b] * state_bytes / (c * b)
    best = max(eff(b) for b in tg_by_b)
    b = min(b for b in tg_by_b if eff(b) >= tol * best)
    return {"chunk_bytes": b, "eff_gbs": eff(b), "best_eff_gbs": best,
            "eff_by_b": {k: eff(k) for k in sorted(tg_by_b)}}


def measure_tg(sizes, total_bytes: int = 1 << 30, device: int = 0) -> dict:
    """T_G(b): pinned copy-engine D2H of `total_bytes` moved as back-to-back b-byte copies, best of
    3 (CUDA events), for each b in `sizes`.  GPU only."""
    import torch
    out = {}
    src = torch.empty(total_bytes, dtype=torch.uint8, device=f"cuda:{device}")
    dst = torch.empty(total_bytes, dtype=torch.uint8).pin_memory()
    s = torch.cuda.Stream(device)
    for b in sizes:
        k = max(1, total_bytes // b)
        best = float("inf")
        with torch.cuda.stream(s):
            for rep in range(4):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                for i in range(k):
                    dst[i * b:(i + 1) * b].copy_(src[i * b:(i + 1) * b], non_blocking=True)
                e1.record(s)
                e1.synchronize()
                if rep:
                    best = min(best, e0.elapsed_time(e1))
        out[b] = k * b / (best * 1e-3) / 1e9
    return out


# ------------------------------------------------- Variant A / B and the HBM ring size R
def choose_ring(slice_bytes: int, chunk_bytes: int, hbm_budget_bytes: int, n_inflight: int, link_gbs: float,
                pack_gbs: float = 5000.0, zerocopy_gbs: float | None = None) -> dict:
    """Where K1 puts the packed chunks, under an HBM budget.

    Variant B: an HBM ring of R chunks, drained by the copy engines.  The U-gate (L139) waits for
    K1 only, except for the part of the slice that does not fit the free ring: K1's later
    windows wait for the D2H to free ring space, so the stall per checkpoint is about
        pack time + max(0, slice - R*b) / T_G.
    Up to N slices of ring are useful (N checkpoints in flight, L139 Fig 6), never more.
    Variant A (PCC_ZEROCOPY): K1 stores straight into host memory over PCIe, no HBM at all, and
    the U-gate spans the whole transfer: slice / T_zero-copy.
    Picks the variant with the smaller predicted U-gate stall (B whenever one chunk fits)."""
    if chunk_bytes <= 0 or slice_bytes < 0 or link_gbs <= 0:
        raise ValueError("bad sizes")
    n = -(-slice_bytes // chunk_bytes)
    r = min(hbm_budget_bytes // chunk_bytes, max(1, n_inflight) * n)
    zc = zerocopy_gbs or 0.92 * link_gbs  # SM stores into mapped memory: 52.7 vs 57.2 GB/s measured
    stall_a = slice_bytes / (zc * 1e9)
    if r < 1:
        return {"variant": "A", "ring_chunks": 0, "ring_bytes": 0, "stall_s": stall_a, "stall_s_B": None}
    stall_b = 2 * slice_bytes / (pack_gbs * 1e9) + max(0, slice_bytes - r * chunk_bytes) / (link_gbs * 1e9)
    if stall_b <= stall_a:
        return {"variant": "B", "ring_chunks": int(r), "ring_bytes": int(r * chunk_bytes), "stall_s": stall_b,
                "stall_s_A": stall_a}
    return {"variant": "A", "ring_chunks": 0, "ring_bytes": 0, "stall_s": stall_a, "stall_s_B": stall_b}


def pace_delivery(contended_gbs: float, d2h_gbs: float) -> float | None:
    """How much of the chosen pace a checkpoint taken while training actually got (1.0 = all).
    choose_pace's rule only holds if this stays near 1."""
    if not d2h_gbs or not contended_gbs:
        return None
    return contended_gbs / d2h_gbs
