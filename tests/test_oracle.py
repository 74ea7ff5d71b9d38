"""Pins for the CPU oracle.  CPU only.

Every test here checks oracle/ against something other than itself: the RFC 3720
CRC32C vectors, the x86 SSE4.2 crc32 instruction, hand-computed layouts, the
definition-level properties of the packed image (round trip, zero pads, minimal
aligned offsets), an independent struct-based parse of the on-file records, and
fault injection that must never restore wrong bytes.
"""
import itertools
import os
import struct

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import oracle
from conftest import load_golden_crc, ROOT


# ---------------------------------------------------------------- P1 RFC vectors
@pytest.mark.parametrize("name,data,crc", load_golden_crc())
def test_rfc3720_vectors(name, data, crc):
    assert oracle.crc32c(data) == crc


# ------------------------------------------------------ P2 independent hardware CRC
def test_crc_matches_sse42_instruction(hwcrc):
    rng = np.random.default_rng(1)
    lengths = list(range(0, 70)) + [255, 256, 257, 4095, 4096, 4097, 65536 + 3, 1 << 20]
    for n in lengths:
        b = rng.integers(0, 256, n, dtype=np.uint8)
        assert oracle.crc32c(b) == hwcrc(b), n


# -------------------------------------------------------------- P3 layout by hand
def test_layout_hand_example():
    # off0=0 end=3; off1=256 end=556; off2=768 (0 bytes) end=768; off3=768 end=785; C=ceil(785/256)=4
    off, end, c = oracle.layout([3, 300, 0, 17], align=256, chunk_bytes=256)
    assert list(off) == [0, 256, 768, 768] and end == 785 and c == 4
    off, end, c = oracle.layout([], align=256, chunk_bytes=4096)
    assert end == 0 and c == 0
    off, end, c = oracle.layout([4096], align=256, chunk_bytes=4096)
    assert end == 4096 and c == 1


@settings(max_examples=200, deadline=None)
@given(st.lists(st.integers(0, 5000), min_size=1, max_size=12), st.sampled_from([16, 256, 4096]),
       st.sampled_from([16, 48, 4096]))
def test_layout_properties(nbytes, align, cb):
    off, end, c = oracle.layout(nbytes, align=align, chunk_bytes=cb)
    prev_end = 0
    for i, (o, n) in enumerate(zip(off, nbytes)):
        o = int(o)
        assert o % align == 0
        if i == 0:
            assert o == 0
        else:
            assert prev_end <= o < prev_end + align  # the smallest aligned offset at or past the previous end
        prev_end = o + n
    assert end == prev_end
    assert c == -(-end // cb)


def test_c1_layout_matches_survey():
    # SURVEY §8 size table [verified there]: C1 -> 17 chunks, layout end 67,124,208
    from synth import config_tensors
    specs = config_tensors("c1")
    nbytes = [s.nbytes for s in specs]
    assert len(specs) == 97 and sum(nbytes) == 64 << 20
    off, end, c = oracle.layout(nbytes, 256, 4 << 20)
    assert c == 17 and end == 67_124_208


# ------------------------------------------------------------ P4 pack definition
def _check_image(srcs, align, cb, img):
    nbytes = [len(s) for s in srcs]
    off, end, c = oracle.layout(nbytes, align, cb)
    assert img.nbytes == c * cb
    covered = np.zeros(img.nbytes, dtype=bool)
    for s, o in zip(srcs, off):
        o = int(o)
        assert img[o:o + len(s)].tobytes() == bytes(s)  # round trip: unpack(pack(S)) == S
        covered[o:o + len(s)] = True
    assert not img[~covered].any()  # every other byte is zero


def test_pack_bruteforce_tiny(hwcrc):
    """All registrations of <= 3 tensors with sizes from a tiny set, several CB/ALIGN."""
    sizes = [0, 1, 15, 16, 17, 40]
    rng = np.random.default_rng(7)
    n_cases = 0
    for k in range(1, 4):
        for combo in itertools.product(sizes, repeat=k):
            srcs = [rng.integers(1, 256, n, dtype=np.uint8).tobytes() for n in combo]
            for cb in (16, 32, 48, 64):
                for align in (16, 256):
                    img = oracle.pack(srcs, align=align, chunk_bytes=cb)
                    _check_image(srcs, align, cb, img)
                    crcs = oracle.chunk_crcs(img, cb)
                    assert [int(x) for x in crcs] == [hwcrc(img[i * cb:(i + 1) * cb]) for i in range(len(crcs))]
                    n_cases += 1
    assert n_cases > 1000


def test_pack_partial_range_equals_full_slice():
    rng = np.random.default_rng(3)
    srcs = [rng.integers(0, 256, n, dtype=np.uint8).tobytes() for n in (1000, 33, 5000, 7, 4096)]
    full = oracle.pack(srcs, align=256, chunk_bytes=512)
    c = full.nbytes // 512
    for first in range(c):
        for cnt in range(0, c - first + 1):
            part = oracle.pack(srcs, align=256, chunk_bytes=512, first_chunk=first, count=cnt)
            assert part.tobytes() == full[first * 512:(first + cnt) * 512].tobytes()


def test_pack_preserves_float_bit_patterns():
    # NaN payloads, signalling NaNs, -0.0 and denormals must survive as raw bytes (R1: no dtype conversion)
    pats = np.array([0x7FC00001, 0x7F800001, 0xFFBFFFFF, 0x80000000, 0x00000001, 0x807FFFFF], dtype=np.uint32)
    img = oracle.pack([pats.tobytes()], align=256, chunk_bytes=64)
    assert img[:pats.nbytes].view(np.uint32).tolist() == pats.tolist()


def test_rfc_pack_pin():
    """P4: pack + per-chunk CRC of the four RFC patterns predicts the whole table (golden file)."""
    srcs = [bytes(32), b"\xff" * 32, bytes(range(32)), bytes(range(31, -1, -1))]
    img = oracle.pack(srcs, align=256, chunk_bytes=32)
    got = [int(x) for x in oracle.chunk_crcs(img, 32)]
    exp = []
    with open(os.path.join(ROOT, "tests", "golden", "rfc_pack_pin.txt")) as f:
        for line in f:
            if line.startswith("#") or not line.strip():
                continue
            i, crc = line.split()
            exp.append(int(crc, 16))
    assert got == exp


@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
def test_slices_partition_chunks(world):
    for c in [0, 1, 5, 17, 264, 1475]:
        seen = []
        for r in range(world):
            a, n = oracle.rank_slice(c, r, world)
            seen.extend(range(a, a + n))
            assert c // world <= n <= -(-c // world)
        assert seen == list(range(c))


# -------------------------------------------------- P5 on-file records, parsed independently
def test_slot_header_independent_parse(hwcrc):
    crcs = [0x11111111, 0xDEADBEEF, 0x0]
    h = oracle.slot_header(2, 40, 7, 4096, 1, 4, 12, 3, 3, 97, 256, 0xABCDEF01, 0x12345678, 2, crcs)
    assert len(h) == 4096
    magic, state, ver, it, ctr, cb, rank, world, tot, first, n, nt, al, lcrc, dig, slot = struct.unpack_from(
        "<8sIIQQQIIIIIIIIII", h, 0)
    assert (magic, state, ver, it, ctr, cb, rank, world, tot, first, n, nt, al, lcrc, dig, slot) == (
        b"PCCSLOT1", 2, 1, 40, 7, 4096, 1, 4, 12, 3, 3, 97, 256, 0xABCDEF01, 0x12345678, 2)
    assert h[80:96] == bytes(16)
    assert list(struct.unpack_from("<3I", h, 96)) == crcs
    (hc,) = struct.unpack_from("<I", h, 96 + 12)
    assert hc == hwcrc(h[:96 + 12])
    assert h[96 + 16:] == bytes(4096 - 96 - 16)
    assert oracle.header_bytes(999) == 4096 and oracle.header_bytes(1000) == 8192


def test_ptr_record_independent_parse(hwcrc):
    r = oracle.ptr_record(8, 5, 50, 6, 2, 3, 40, 3)
    magic, ver, world, seq, li, lc, ls, rank, gi, ns = struct.unpack_from("<8sIIQQQIIQI", r, 0)
    assert (magic, ver, world, seq, li, lc, ls, rank, gi, ns) == (b"PCCPTR01", 1, 8, 5, 50, 6, 2, 3, 40, 3)
    assert r[60:4092] == bytes(4032)
    assert struct.unpack_from("<I", r, 4092)[0] == hwcrc(r[:4092])


def test_layout_crc_independent(hwcrc):
    nb, dt = [4, 1 << 33, 0], [1, 2, 3]
    ser = b"".join(struct.pack("<QI", n, d) for n, d in zip(nb, dt)) + struct.pack("<IQ", 256, 1 << 22)
    assert oracle.layout_crc(nb, dt, 256, 1 << 22) == hwcrc(ser)


# ---------------------------------------------------- P6 restore round trip + faults
def _state(seed, sizes):
    rng = np.random.default_rng(seed)
    return [rng.integers(0, 256, n, dtype=np.uint8) for n in sizes]


SIZES = [4000, 1, 12345, 0, 70000, 33, 8192]
CB = 4096
N_SLOTS = 3


def _write(path, state, slot, it, seq, rank=0, world=1, g=None):
    oracle.write_checkpoint(path, state, [1] * len(state), 256, CB, rank, world, N_SLOTS, slot, it, it // 10, seq,
                            global_iter=g)


@pytest.mark.parametrize("world", [1, 3])
def test_restore_roundtrip(tmp_path, world):
    st_ = _state(0, SIZES)
    paths = [str(tmp_path / f"r{r}.pcc") for r in range(world)]
    for r in range(world):
        _write(paths[r], st_, 0, 10, 1, r, world)
    rc, it, bad, outs = oracle.restore(paths, N_SLOTS, SIZES, [1] * len(SIZES), 256, CB)
    assert rc == 0 and it == 10 and bad == []
    assert all(o.tobytes() == s.tobytes() for o, s in zip(outs, st_))


def test_restore_empty_file_is_enoent(tmp_path):
    p = str(tmp_path / "e.pcc")
    with open(p, "wb") as f:
        f.write(bytes(8192))
    rc, *_ = oracle.restore([p], N_SLOTS, SIZES, [1] * len(SIZES), 256, CB)
    assert rc == oracle.ENOENT


def _two_ckpts(tmp_path):
    p = str(tmp_path / "f.pcc")
    old, new = _state(1, SIZES), _state(2, SIZES)
    _write(p, old, 0, 10, 1)
    _write(p, new, 1, 20, 2)
    return p, old, new


def _n_data_chunks():
    off, end, c = oracle.layout(SIZES, 256, CB)
    return c


def _chunk_file_off(slot, chunk):
    c = _n_data_chunks()
    return oracle.slot_offset(slot, c, CB) + oracle.header_bytes(c) + chunk * CB


def _inject(path, off, new_bytes):
    with open(path, "r+b") as f:
        f.seek(off)
        old = f.read(len(new_bytes))
        assert old != new_bytes, "injector must change bytes"
        f.seek(off)
        f.write(new_bytes)


FAULTS = ["bitflip", "burst32", "half_stale", "zero_tail", "header_crc_entry"]


@pytest.mark.parametrize("fault", FAULTS)
def test_restore_rejects_faults_and_falls_back(tmp_path, fault):
    p, old, new = _two_ckpts(tmp_path)
    chunk = 5
    o = _chunk_file_off(1, chunk)
    with open(p, "rb") as f:
        f.seek(o)
        cur = f.read(CB)
        f.seek(_chunk_file_off(0, chunk))
        stale = f.read(CB)
    if fault == "bitflip":
        _inject(p, o + 100, bytes([cur[100] ^ 0x10]))
    elif fault == "burst32":
        _inject(p, o + 64, bytes(b ^ 0xFF for b in cur[64:68]))
    elif fault == "half_stale":
        _inject(p, o + CB // 2, stale[CB // 2:])
    elif fault == "zero_tail":
        if cur[-256:] == bytes(256):
            pytest.skip("tail already zero")
        _inject(p, o + CB - 256, bytes(256))
    elif fault == "header_crc_entry":
        # rewrite one CRC table entry AND re-seal the header CRC, so only the chunk check can catch it
        c = _n_data_chunks()
        ho = oracle.slot_offset(1, c, CB)
        with open(p, "rb") as f:
            f.seek(ho)
            h = bytearray(f.read(oracle.header_bytes(c)))
        h[96 + 4 * chunk] ^= 0x01
        h[96 + 4 * c:96 + 4 * c + 4] = struct.pack("<I", oracle.crc32c(bytes(h[:96 + 4 * c])))
        _inject(p, ho, bytes(h))
    rc, it, bad, outs = oracle.restore([p], N_SLOTS, SIZES, [1] * len(SIZES), 256, CB)
    assert rc == oracle.ECORRUPT and bad == [chunk]
    rc, it, bad, outs = oracle.restore([p], N_SLOTS, SIZES, [1] * len(SIZES), 256, CB, fallback=True)
    assert rc == 0 and it == 10
    assert all(o.tobytes() == s.tobytes() for o, s in zip(outs, old))


def test_restore_torn_pointer_uses_other_record(tmp_path):
    p, old, new = _two_ckpts(tmp_path)
    # seq 2 lives at offset 0 (seq % 2 == 0); tear it
    _inject(p, 20, b"\x00\x00\x00\x09")
    assert oracle.latest(p)[2] == 1
    rc, it, bad, outs = oracle.restore([p], N_SLOTS, SIZES, [1] * len(SIZES), 256, CB)
    assert rc == 0 and it == 10
    assert all(o.tobytes() == s.tobytes() for o, s in zip(outs, old))


def test_restore_truncated_file(tmp_path):
    p, old, new = _two_ckpts(tmp_path)
    with open(p, "r+b") as f:
        f.truncate(_chunk_file_off(1, 3) + 17)
    rc, it, bad, outs = oracle.restore([p], N_SLOTS, SIZES, [1] * len(SIZES), 256, CB)
    assert rc == oracle.ECORRUPT and bad[0] == 3
    rc, it, bad, outs = oracle.restore([p], N_SLOTS, SIZES, [1] * len(SIZES), 256, CB, fallback=True)
    assert rc == 0 and it == 10


def test_restore_filling_header_not_accepted(tmp_path):
    p, old, new = _two_ckpts(tmp_path)
    c = _n_data_chunks()
    h = oracle.slot_header(1, 20, 2, CB, 0, 1, c, 0, c, len(SIZES), 256,
                           oracle.layout_crc(SIZES, [1] * len(SIZES), 256, CB), 0, 1, [0] * c)
    _inject(p, oracle.slot_offset(1, c, CB), h)
    rc, it, bad, outs = oracle.restore([p], N_SLOTS, SIZES, [1] * len(SIZES), 256, CB, fallback=True)
    assert rc == 0 and it == 10


def test_restore_layout_mismatch(tmp_path):
    p, old, new = _two_ckpts(tmp_path)
    rc, *_ = oracle.restore([p], N_SLOTS, SIZES, [2] * len(SIZES), 256, CB)
    assert rc == oracle.ELAYOUT


def test_restore_dp_global_iter_and_presence(tmp_path):
    """W=2: rank 1 never got iter 20 durable -> restore must pick the iter both hold (§8(e))."""
    world = 2
    paths = [str(tmp_path / f"r{r}.pcc") for r in range(world)]
    s10, s20 = _state(1, SIZES), _state(2, SIZES)
    for r in range(world):
        _write(paths[r], s10, 0, 10, 1, r, world, g=10)
    _write(paths[0], s20, 1, 20, 2, 0, world, g=20)  # only rank 0 holds 20 (its record even claims g=20)
    rc, it, bad, outs = oracle.restore(paths, N_SLOTS, SIZES, [1] * len(SIZES), 256, CB)
    assert rc == oracle.ENOENT
    rc, it, bad, outs = oracle.restore(paths, N_SLOTS, SIZES, [1] * len(SIZES), 256, CB, fallback=True)
    assert rc == 0 and it == 10
    assert all(o.tobytes() == s.tobytes() for o, s in zip(outs, s10))


def test_pack_chunks_sparse_equals_full_pack():
    """The sampled-chunk helper used at full sizes is the same O2 image, chunk for chunk."""
    rng = np.random.default_rng(11)
    sizes = [int(x) for x in rng.integers(0, 9000, 40)]
    srcs = [rng.integers(0, 256, n, dtype=np.uint8) for n in sizes]
    cb = 4096
    full = oracle.pack(srcs, 256, cb)
    off, end, c = oracle.layout(sizes, 256, cb)
    for j in range(c):
        need = {i: srcs[i] for i in range(len(sizes))
                if sizes[i] and int(off[i]) < (j + 1) * cb and int(off[i]) + sizes[i] > j * cb}
        part = oracle.pack_chunks_sparse(sizes, need, 256, cb, j, 1)
        assert part.tobytes() == full[j * cb:(j + 1) * cb].tobytes()
