"""Differential fuzzing of the on-storage format parsers ("commit-format parser fuzzing").

A rank file with three committed checkpoints is written by the library's commit engine
(pccheck_host.h), then hypothesis flips bytes in its metadata (the two pointer records of
FORMAT.md and the N+1 slot headers) or truncates it.  Two parsers that share no code must then
take the same decision (FORMAT.md O5-O7, readings R7, R10, R18):
  * the oracle's restore (oracle/pcc_oracle.c, verify + fallback), and
  * the library's pointer query (pcc_latest) and restore agreement (pcc_host_restore_plan,
    W = 1), whose slice verification (K2 on a GPU) is stood in for by the ground truth: the
    slot's data bytes equal the packed image of that iter (K2's CRC check approximates this
    with a 2^-32 miss rate; only truncation changes data bytes here).
Neither may crash, and a mutated file must never restore an iter that was not committed.
"""
import os
import shutil

import numpy as np
import pytest
from hypothesis import HealthCheck, given, settings, strategies as st

import oracle

pcc = pytest.importorskip("paper_conf_asplos_strati0k25_b200")

CB = 4096
SIZES = [5000, 17, 12000, 0, 40000, 3]
N = 2
ITERS = (10, 20, 30, 40)


def _state(seed):
    rng = np.random.default_rng(seed)
    return [rng.integers(0, 256, n, dtype=np.uint8) for n in SIZES]


@pytest.fixture(scope="module")
def pristine(tmp_path_factory):
    d = tmp_path_factory.mktemp("fuzz")
    path = str(d / "p.pcc")
    off, end, c = oracle.layout(SIZES, 256, CB)
    lcrc = oracle.layout_crc(SIZES, [0] * len(SIZES), 256, CB)
    e = pcc.HostEngine(path, CB, N, 0, 1, c, len(SIZES), 256, lcrc)
    for it in ITERS:
        counter, slot = e.begin(it)
        e.filling(counter)
        img = oracle.pack(_state(it), 256, CB)
        with open(path, "r+b") as f:
            f.seek(e.data_offset(slot))
            f.write(img.tobytes())
        e.complete(counter, [int(x) for x in oracle.chunk_crcs(img, CB)], oracle.crc32c(img))
    e.close()
    regions = [(0, 8192)] + [(oracle.slot_offset(s, c, CB), oracle.header_bytes(c)) for s in range(N + 1)]
    return path, c, lcrc, regions


def _library_restore(path, c, lcrc, fallback):
    e = pcc.HostEngine(path, CB, N, 0, 1, c, len(SIZES), 256, lcrc)  # (re)extends a truncated file

    def verify(it, slot):
        want = oracle.pack(_state(it), 256, CB).tobytes() if it in ITERS else None
        with open(path, "rb") as f:
            f.seek(e.data_offset(slot))
            return want is not None and f.read(c * CB) == want
    try:
        return 0, e.restore_plan(lambda v, is_max: v, verify, fallback=fallback)
    except pcc.PCCError as err:
        return err.code, None
    finally:
        e.close()


# (region, position, xor): region 0 = the two pointer records, 1..3 = slot headers; positions are
# drawn mostly from the bytes that carry fields (record bytes 0..63 and its CRC at 4092..4095,
# header bytes 0..(96 + 4n + 4)), sometimes from anywhere (mostly zero padding)
OUTCOMES = {}
mutation = st.tuples(st.integers(0, 3), st.one_of(st.integers(0, 63), st.integers(4092, 4095),
                                                   st.integers(4096, 4096 + 63), st.integers(8188, 8191),
                                                   st.integers(0, 8191)), st.integers(1, 255))


@settings(max_examples=400, deadline=None, suppress_health_check=[HealthCheck.function_scoped_fixture])
@given(muts=st.lists(mutation, min_size=1, max_size=4), truncate=st.sampled_from([None, None, None, 0.3, 0.7]),
       fallback=st.booleans())
def test_metadata_mutations_same_decision(pristine, tmp_path, muts, truncate, fallback):
    src, c, lcrc, regions = pristine
    path = str(tmp_path / "m.pcc")
    shutil.copyfile(src, path)
    with open(path, "r+b") as f:
        for region, where, x in muts:
            lo, size = regions[region]
            pos = lo + (where if region == 0 else where % (96 + 4 * c + 4 if where < 8000 else size))
            f.seek(pos)
            b = f.read(1)[0]
            f.seek(pos)
            f.write(bytes([b ^ x]))  # always a different byte (x != 0)
        if truncate is not None:
            f.truncate(int(os.path.getsize(path) * truncate))
    # pointer query: the same record wins (or none is valid) in both parsers
    lo, ll = pcc.latest(path) or (None, None), oracle.latest(path)
    if ll is None:
        assert lo == (None, None)
    else:
        assert lo == (ll[0], ll[1])
    rc_o, it_o, bad_o, _ = oracle.restore([path], N + 1, SIZES, [0] * len(SIZES), 256, CB, fallback=fallback)
    rc_l, it_l = _library_restore(path, c, lcrc, fallback)
    assert (rc_o == 0) == (rc_l == 0), (rc_o, rc_l)
    OUTCOMES[(rc_o, it_o if rc_o == 0 else None)] = OUTCOMES.get((rc_o, it_o if rc_o == 0 else None), 0) + 1
    if rc_o == 0:
        assert it_o == it_l and it_o in ITERS
        if not fallback:  # with PCC_FALLBACK, bad lists the first rejected candidate's chunks
            assert not bad_o


def test_fuzz_reached_every_outcome():
    """The mutations above must have produced the newest iter, a fallback and a rejection."""
    if not OUTCOMES:
        pytest.skip("run with the fuzz test")
    assert any(k[0] == 0 and k[1] == ITERS[-1] for k in OUTCOMES), OUTCOMES
    assert any(k[0] == 0 and k[1] < ITERS[-1] for k in OUTCOMES), OUTCOMES
    assert any(k[0] != 0 for k in OUTCOMES), OUTCOMES
