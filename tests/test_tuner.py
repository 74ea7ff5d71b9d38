"""Tuner (PAPER §3.4, Eq 3): the decision rule on CPU against the oracle's Eq 3, and one
live sweep on the GPU."""
import os

import pytest

from oracle.manager_model import f_star


def test_choose_matches_eq3():
    from paper_conf_asplos_strati0k25_b200.tuner import choose
    tw = {1: 2.0, 2: 2.6, 3: 4.5, 4: 6.4}  # contention grows with N (L201)
    out = choose(tw, q=1.03, t=0.1)
    assert out["N"] == 2 and out["Tw"] == 2.6  # Tw/N = 2.0, 1.3, 1.5, 1.6 -> N* = 2
    assert out["f"] == f_star(2.6, 2, 1.03, 0.1) == 13
    assert choose({1: 0.01}, q=1.0, t=1.0)["f"] == 1


def test_choose_pace():
    from paper_conf_asplos_strati0k25_b200.tuner import D2H_QUANTUM, choose_pace
    # VGG-16: 1.1 GB every 10 x 17 ms needs 12.9 GB/s at margin 0.5 -> floor of half the link
    p = choose_pace(1_107_296_256, 10, 0.0171, 57.0)
    assert p["d2h_gbs"] == 28.5 and p["d2h_quantum"] == D2H_QUANTUM
    assert abs(p["need_gbs"] - 1_107_296_256 / (0.5 * 10 * 0.0171) / 1e9) < 1e-9
    # a tighter interval raises the pace above the floor
    p = choose_pace(1_107_296_256, 4, 0.0171, 57.0)
    assert 28.5 < p["d2h_gbs"] < 57.0 and p["d2h_gbs"] == pytest.approx(p["need_gbs"])
    # checkpointing every iteration needs more than the link: unpaced
    assert choose_pace(1_107_296_256, 1, 0.0171, 57.0) == {"d2h_gbs": 0.0, "d2h_quantum": 0,
                                                            "need_gbs": pytest.approx(129.5, rel=1e-3)}
    # OPT-1.3B (15.8 GB every 10 x 43.8 ms): 72 GB/s at margin 0.5 exceeds the link -> unpaced by
    # default; the optional stretch (max_margin 0.9, N >= 2) gives 40 GB/s; never with N = 1
    p = choose_pace(15_789_098_512, 10, 0.0438, 57.0)
    assert p["need_gbs"] == pytest.approx(72.1, rel=1e-2) and p["d2h_gbs"] == 0.0
    p = choose_pace(15_789_098_512, 10, 0.0438, 57.0, max_margin=0.9)
    assert p["d2h_gbs"] == pytest.approx(15_789_098_512 / (0.9 * 10 * 0.0438) / 1e9) and p["d2h_quantum"] == D2H_QUANTUM
    assert choose_pace(15_789_098_512, 10, 0.0438, 57.0, max_margin=0.9, n_inflight=1)["d2h_gbs"] == 0.0
    with pytest.raises(ValueError):
        choose_pace(1, 0, 1.0, 1.0)


@pytest.mark.gpu
@pytest.mark.timeout(300)
def test_tune_live_c1():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_asplos_strati0k25_b200 as pcc
    from paper_conf_asplos_strati0k25_b200.tuner import tune
    from synth import config_tensors, make_state
    specs = config_tensors("c1")
    ts = make_state(specs, "cuda", seed=0, it=0)
    d = "/dev/shm" if os.path.isdir("/dev/shm") else "/tmp"
    paths = []

    def make_ctx(n):
        p = os.path.join(d, f"pcc_tune_{os.getpid()}_{n}.pcc")
        paths.append(p)
        ck = pcc.PCCheck(p, chunk_bytes=4 << 20, max_inflight=n, flags=pcc.MAPFILE)
        ck.register(ts)
        return ck

    m = 17 * (4 << 20)
    out = tune(make_ctx, m, 5 * m, t=0.002, q=1.03, n_max=4, probes=3)
    for p in paths:
        if os.path.exists(p):
            os.unlink(p)
    assert set(out["Tw_by_N"]) == {1, 2, 3, 4}
    assert all(v > 0 for v in out["Tw_by_N"].values())
    assert 1 <= out["N"] <= 4 and out["f"] >= 1
