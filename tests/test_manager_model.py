"""Pins for oracle/manager_model.py (O8): Listing 1 under every interleaving, the DP rule,
and the paper's runtime / recovery equations against a discrete-event timeline."""
import itertools
import random

import pytest

from oracle.manager_model import ListingOne, DPRank, runtime2, recovery_bound, f_star


def _all_interleavings(k):
    """Every order of k begins and k persists where persist(i) follows begin(i)."""
    events = [("b", i) for i in range(k)] + [("p", i) for i in range(k)]
    for perm in itertools.permutations(events):
        seen = set()
        ok = True
        for e, i in perm:
            if e == "b":
                if any(j > i for j in seen):  # begins are issued in iteration order
                    ok = False
                    break
                seen.add(i)
            elif i not in seen:
                ok = False
                break
        if ok:
            yield perm


@pytest.mark.parametrize("N", [1, 2, 3])
def test_listing1_invariants_all_interleavings(N):
    k = 3
    n_seen = 0
    for order in set(_all_interleavings(k)):
        m = ListingOne(N)
        cks, in_flight, blocked = {}, [], False
        for e, i in order:
            if e == "b":
                ck = m.begin(10 * (i + 1))
                if ck is None:
                    blocked = True
                    break
                cks[i] = ck
                in_flight.append(ck)
            else:
                ck = cks[i]
                in_flight.remove(ck)
                m.persisted(ck)
            m.check_invariants(in_flight)
        if blocked:
            # begin only blocks with N in flight once a pointer holds a slot (L158, L229);
            # before the first commit all N+1 slots are free
            assert len(in_flight) == N + (1 if m.CHECK_ADDR is None else 0)
            continue
        n_seen += 1
        # the final pointer is the checkpoint with the largest counter
        assert m.CHECK_ADDR.counter == max(c.counter for c in cks.values())
        assert sum(c.state == "LOCAL_COMMIT" for c in cks.values()) >= 1
    assert n_seen >= 3


def test_listing1_random_stress():
    rng = random.Random(0)
    for N in (1, 2, 4):
        m = ListingOne(N)
        in_flight, it = [], 0
        for step in range(3000):
            if in_flight and (rng.random() < 0.5 or len(in_flight) == N):
                ck = in_flight.pop(rng.randrange(len(in_flight)))
                m.persisted(ck)
            else:
                it += 10
                ck = m.begin(it)
                assert ck is not None
                in_flight.append(ck)
            m.check_invariants(in_flight)


def test_dp_rule_keeps_g_on_every_rank():
    """R20: in-order local commits + g = MIN(L_r) + free below g -> every rank holds g."""
    rng = random.Random(1)
    W, N = 4, 2
    for trial in range(30):
        ranks = [DPRank(N) for _ in range(W)]
        inflight = [[] for _ in range(W)]
        it = 0
        g = None
        for step in range(200):
            # all ranks begin the same iteration at the same program point (collective backpressure)
            if all(r.free for r in ranks) and rng.random() < 0.5:
                it += 10
                for r in range(W):
                    inflight[r].append(ranks[r].begin(it))
            for r in range(W):
                if inflight[r] and rng.random() < 0.4:
                    c = inflight[r].pop(rng.randrange(len(inflight[r])))
                    ranks[r].persisted(c)
            Ls = [rk.L for rk in ranks]
            if all(x is not None for x in Ls):
                g = min(Ls)
                for rk in ranks:
                    rk.global_commit(g)
                    assert g in rk.held  # restore needs g on every rank
            for rk in ranks:
                assert len(rk.free) + len(rk.held) + len(rk.pending) == N + 1


def _simulate(A, t, f, N, Tw):
    """Discrete-event timeline of Fig 6: train t per iteration; after every f-th iteration a
    checkpoint starts and takes Tw; a new one waits while N are in flight (L139, L158)."""
    clock, inflight = 0.0, []
    for i in range(1, A + 1):
        clock += t
        if i % f == 0:  # A/f checkpoints, the last one after iteration A (the '+ Tw' term)
            inflight = [e for e in inflight if e > clock]
            if len(inflight) >= N:
                clock = max(clock, sorted(inflight)[len(inflight) - N])
                inflight = [e for e in inflight if e > clock]
            inflight.append(clock + Tw)
    return max(inflight)


@pytest.mark.parametrize("N,Tw", [(1, 50), (2, 50), (4, 50), (2, 5), (4, 300), (3, 120)])
def test_runtime2_matches_timeline(N, Tw):
    A, t, f = 1200, 1.0, 10  # the paper assumes N·f divides A (L184)
    sim = _simulate(A, t, f, N, Tw)
    assert abs(sim - runtime2(A, t, f, N, Tw)) <= N * f * t


def test_recovery_and_fstar():
    assert recovery_bound(5, 1, 10, 2, 50) == 5 + 10 + 20
    assert recovery_bound(5, 1, 10, 4, 30) == 5 + 10 + 30
    assert f_star(50, 2, 1.03, 1.0) == 25  # ceil(50 / 2.06) = ceil(24.27)
