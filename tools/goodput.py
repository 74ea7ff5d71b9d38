"""Goodput under preemptions.

The paper's end metric: useful iterations per unit time of a job that is preempted and
resumes from its newest committed checkpoint.  The real spot trace is not available (OUT);
this simulates a Poisson preemption process at the trace's rate (26 preemptions in 3.5 h,
L81) with this build's MEASURED numbers: iteration time with / without checkpointing, the
time from pcc_checkpoint to commit (T_w) and the restore time l.

    python tools/goodput.py --t 0.01712 --slowdown-pct 1.4 --tw 0.02 --restore 0.021

T_w is the paper's worst-case write time (all N checkpoints in flight, L178): for this link-bound
path about N times the single-checkpoint time.  --slowdown-pct is the interference that
remains when no checkpoint stalls (the measured every-10 slowdown).  Per failure the redone
iterations obey Eq 4 (L291): lost <= f + min(N*f, T_w/t) iterations.
"""
from __future__ import annotations

import argparse
import json
import math
import random


def simulate(t, f, tw, l, rate, horizon, slowdown_pct=0.0, n_inflight=2, restart=0.0, seed=0):
    """Returns dict(useful_iters, goodput_it_s, failures, max_lost_iters).

    Time advances iteration by iteration (duration t*(1+slowdown) when checkpointing).  A
    checkpoint issued after iteration k (k % f == 0) commits tw seconds later; if n_inflight are
    already in flight the training thread waits for the oldest (the paper's stall, L139).  A
    failure at time tau rolls progress back to the newest checkpoint committed before tau and
    costs restart + l seconds."""
    rng = random.Random(seed)
    it_time = t * (1.0 + slowdown_pct / 100.0)
    clock, progress, useful = 0.0, 0, 0
    committed = []  # (commit_time, iteration)
    inflight = []
    next_fail = rng.expovariate(rate) if rate > 0 else math.inf
    failures, max_lost = 0, 0
    while clock < horizon:
        if clock + it_time > next_fail:  # preempted during this iteration
            durable = [it for (ct, it) in committed if ct <= next_fail]
            resume = max(durable) if durable else 0
            max_lost = max(max_lost, progress - resume)
            progress = resume
            committed = [(ct, it) for (ct, it) in committed if ct <= next_fail]
            inflight = []
            clock = next_fail + restart + l
            failures += 1
            next_fail = clock + rng.expovariate(rate)
            continue
        clock += it_time
        progress += 1
        if progress % f == 0:
            inflight = [c for c in inflight if c > clock]
            if len(inflight) >= n_inflight:
                clock = max(clock, sorted(inflight)[len(inflight) - n_inflight])
                inflight = [c for c in inflight if c > clock]
            done = clock + tw
            inflight.append(done)
            committed.append((done, progress))
    useful = progress
    return {"useful_iters": useful, "goodput_it_s": useful / horizon, "failures": failures,
            "max_lost_iters": max_lost}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--t", type=float, required=True, help="iteration time without checkpointing (s)")
    ap.add_argument("--slowdown-pct", type=float, default=0.0)
    ap.add_argument("--tw", type=float, required=True,
                    help="T_w: checkpoint call -> commit (s), at worst case with N in flight (L178)")
    ap.add_argument("--restore", type=float, required=True, help="restore time l (s)")
    ap.add_argument("--rate", type=float, default=26 / (3.5 * 3600), help="preemptions per second (L81)")
    ap.add_argument("--horizon", type=float, default=3.5 * 3600)
    ap.add_argument("--restart", type=float, default=0.0)
    a = ap.parse_args()
    ideal = a.horizon / a.t
    for f in (1, 2, 5, 10, 20, 50, 100):
        r = simulate(a.t, f, a.tw, a.restore, a.rate, a.horizon, a.slowdown_pct, restart=a.restart)
        r.update(f=f, goodput_frac_of_ideal=r["useful_iters"] / ideal)
        print(json.dumps(r))


if __name__ == "__main__":
    main()
