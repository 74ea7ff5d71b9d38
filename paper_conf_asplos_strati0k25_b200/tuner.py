"""Configuration tuner — PAPER.md §3.4 (L170-L217), SURVEY §8(f) f1.

Given the checkpoint size m, the storage budget S, the iteration time t and the accepted
overhead q, PCcheck's tool "initiates a checkpoint every t seconds.  It then varies N in
[1, S/m - 1], measures T_w for each checkpoint, and finds the optimal N" (L215) minimising
T_w / N, then sets the checkpoint interval (Eq 3; reading R14: ceiling)

    f* = ceil( T_w / (N* * q * t) ).

Here T_w of one checkpoint is measured by the library itself (pcc_info: pcc_checkpoint call
-> local commit) while N checkpoints are kept in flight at a cadence of one every t seconds.

On B200 the tool also picks the D2H pace (pcc_config d2h_mbps / d2h_quantum): a saturating
copy-engine burst slows an eager training loop by ~10% while it lasts, small paced copies
leave gaps that hide it (profiles/r01_slowdown_diagnosis.md).  `choose_pace` takes the
gentlest pace that still lands one checkpoint within `margin` of its interval f*t, never below
half the link (below that the measured interference no longer drops) and unpaced when even the
full link is needed.
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


D2H_QUANTUM = 512 << 10  # bytes per paced copy (0.5 MiB: measured best trade, r01 diagnosis)


def choose_pace(slice_bytes: int, f: int, t: float, link_gbs: float, margin: float = 0.5,
                max_margin: float = 0.5, n_inflight: int = 2) -> dict:
    """D2H pace for training: {"d2h_gbs": G, "d2h_quantum": Q}; G = 0 means unpaced.

    The gentlest pace that lands one checkpoint within `margin` of its interval f*t, never below
    half the link (below that the measured cost no longer drops).  When that needs more than
    the link and N >= 2 checkpoints may overlap (Fig 6), the interval may be
    stretched up to `max_margin` before giving up the pace.  Off by default (max_margin =
    margin): measured on OPT-1.3B (15.8 GB every 10 x 44 ms: 72 GB/s at margin 0.5, 40 GB/s at
    0.9) the stretched pace kept the link busy the whole interval and cost 19.8% against 16.7%
    unpaced — there the answer is a longer interval (Eq 3's f*), not a pace."""
    if f <= 0 or t <= 0 or link_gbs <= 0:
        raise ValueError("f, t and link_gbs must be positive")
    need = slice_bytes / (margin * f * t) / 1e9  # GB/s to land a checkpoint in margin * f * t
    g = max(need, 0.5 * link_gbs)
    if g >= link_gbs and n_inflight >= 2 and max_margin > margin:
        g = max(slice_bytes / (max_margin * f * t) / 1e9, 0.5 * link_gbs)
    if g >= link_gbs:
        return {"d2h_gbs": 0.0, "d2h_quantum": 0, "need_gbs": need}
    return {"d2h_gbs": g, "d2h_quantum": D2H_QUANTUM, "need_gbs": need}
