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
    # VGG-16: 1.1 GB every 10 x 17 ms needs 7.2 GB/s at margin 0.9 -> floor of half the link
    p = choose_pace(1_107_296_256, 10, 0.0171, 57.0)
    assert p["d2h_gbs"] == 28.5 and p["d2h_quantum"] == D2H_QUANTUM == 1 << 20
    assert p["need_gbs"] == pytest.approx(1_107_296_256 / (0.9 * 10 * 0.0171) / 1e9)
    # a tighter interval raises the pace above the floor, up to 0.7 of the link (eager)
    p = choose_pace(1_107_296_256, 2, 0.0171, 57.0)
    assert 28.5 < p["d2h_gbs"] <= 0.7 * 57.0 and p["d2h_gbs"] == pytest.approx(min(p["need_gbs"], 0.7 * 57.0))
    # even the capped pace outlasts the interval (every iteration): unpaced
    p = choose_pace(1_107_296_256, 1, 0.0171, 57.0)
    assert p["d2h_gbs"] == 0.0 and p["d2h_quantum"] == 1 << 20  # unpaced, but in 1 MiB copies (eager)
    # OPT-1.3B eager (15.8 GB every 10 x 44 ms) needs 39.9 GB/s at margin 0.9: on a 57.1 GB/s link
    # that is under the cap; on a 56.0 GB/s link it is capped at 39.2 GB/s, which still lands in
    # 403 ms < 440 ms
    p = choose_pace(15_789_098_512, 10, 0.044, 57.1)
    assert p["d2h_gbs"] == pytest.approx(p["need_gbs"]) == pytest.approx(39.87, rel=1e-3)
    p = choose_pace(15_789_098_512, 10, 0.044, 56.0)
    assert p["d2h_gbs"] == pytest.approx(0.7 * 56.0) and p["d2h_quantum"] == 1 << 20
    # ... with a 50 GB/s link the capped 35 GB/s would need 451 ms > 440 ms: unpaced
    assert choose_pace(15_789_098_512, 10, 0.044, 50.0)["d2h_gbs"] == 0.0
    # N = 1: the margin drops to half the interval (need 71.8 GB/s), so the pace is the cap
    p = choose_pace(15_789_098_512, 10, 0.044, 57.0, n_inflight=1)
    assert p["need_gbs"] == pytest.approx(15_789_098_512 / (0.5 * 10 * 0.044) / 1e9) and p["d2h_gbs"] == pytest.approx(39.9)
    with pytest.raises(ValueError):
        choose_pace(1, 0, 1.0, 1.0)
    # a CUDA-graph loop: margin and cap 0.85 (OPT-1.3B at 51.7 ms -> ~35.9 GB/s)
    p = choose_pace(15_789_098_512, 10, 0.0517, 56.7, graphs=True)
    assert p["d2h_gbs"] == pytest.approx(15_789_098_512 / (0.85 * 10 * 0.0517) / 1e9) and p["d2h_quantum"] == 1 << 20
    assert 28.35 < p["d2h_gbs"] < 0.85 * 56.7
    p = choose_pace(15_789_098_512, 4, 0.0517, 56.7, graphs=True)  # would outlast the interval
    assert p["d2h_gbs"] == 0.0 and p["d2h_quantum"] == 0  # graphs keep whole chunk groups


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


def test_choose_chunk_tg_and_padding():
    """b from T_G (L176): a faster link rate wins, but zero padding (R3) counts against big b."""
    from paper_conf_asplos_strati0k25_b200.tuner import choose_chunk
    MiB = 1 << 20
    tg = {4 * MiB: 50.0, 16 * MiB: 55.0, 64 * MiB: 56.0, 256 * MiB: 56.0}
    # VGG-16's 1.107 GB state: 64 MiB pads the last chunk by 3.0%, 16 MiB by 0.04%
    out = choose_chunk(tg, 1_106_860_352)
    assert out["chunk_bytes"] == 16 * MiB
    assert out["eff_by_b"][64 * MiB] == pytest.approx(56.0 * 1_106_860_352 / (17 * 64 * MiB))
    # a state of exactly 16 x 64 MiB: no padding anywhere, 64 MiB's faster link wins over 16 MiB
    out = choose_chunk(tg, 16 * 64 * MiB, tol=0.995)
    assert out["chunk_bytes"] == 64 * MiB
    # tolerance: the smallest b within 3% of the best
    assert choose_chunk({1: 97.0, 2: 100.0}, 2)["chunk_bytes"] == 1
    with pytest.raises(ValueError):
        choose_chunk({}, 1)


def test_choose_ring_variants():
    from paper_conf_asplos_strati0k25_b200.tuner import choose_ring
    GB, MiB = 10 ** 9, 1 << 20
    s = 12_348_030_976  # BLOOM-7b1 rank slice at W = 8 (185 x 64 MiB)
    # plenty of HBM: the whole slice (x N in flight, capped at N slices)
    r = choose_ring(s, 64 * MiB, 40 * GB, 2, 55.0)
    assert r["variant"] == "B" and r["ring_chunks"] == 2 * 184 and r["stall_s"] < 0.01
    # a 4 GB budget: windowed ring, stall = pack + the part beyond the ring over the link
    r = choose_ring(s, 64 * MiB, 4 * GB, 2, 55.0)
    assert r["variant"] == "B" and r["ring_chunks"] == 59
    assert r["stall_s"] == pytest.approx(2 * s / 5e12 + (s - 59 * 64 * MiB) / 55e9)
    assert r["stall_s"] < r["stall_s_A"]
    # no HBM to spare: Variant A (K1 stores into host memory, the U-gate spans the transfer)
    r = choose_ring(s, 64 * MiB, 32 * MiB, 2, 55.0)
    assert r["variant"] == "A" and r["ring_bytes"] == 0 and r["stall_s"] == pytest.approx(s / (0.92 * 55e9))


def test_pace_delivery():
    from paper_conf_asplos_strati0k25_b200.tuner import pace_delivery
    assert pace_delivery(27.0, 28.5) == pytest.approx(0.947, rel=1e-3)
    assert pace_delivery(0.0, 28.5) is None and pace_delivery(27.0, 0.0) is None
