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


def test_slices_hand_values():
    """orc_slice against hand-computed floor(r*C/W) bounds (FORMAT.md "Image"); a
    remainder-first split (the first C % W ranks take one extra chunk) would give (0,9)/(9,8)
    for C=17, W=2 and (0,3)/(3,3)/(6,2)/(8,2) for C=10, W=4, so it fails here."""
    assert [oracle.rank_slice(17, r, 2) for r in range(2)] == [(0, 8), (8, 9)]
    assert [oracle.rank_slice(10, r, 4) for r in range(4)] == [(0, 2), (2, 3), (5, 2), (7, 3)]
    # C4 (BLOOM-7b1, 1475 chunks of 64 MiB) at W = 8: floor(1475 r / 8) = 0, 184, 368, 553, 737, 921, 1106, 1290
    assert [oracle.rank_slice(1475, r, 8) for r in range(8)] == [
        (0, 184), (184, 184), (368, 185), (553, 184), (737, 184), (921, 185), (1106, 184), (1290, 185)]
    assert oracle.rank_slice(3, 2, 4) == (1, 1) and oracle.rank_slice(3, 0, 4) == (0, 0)


def test_slot_geometry_hand_values():
    """orc_header_bytes / orc_slot_stride / orc_slot_offset against FORMAT.md "File", by hand:
    H = align_up(96 + 4n + 4, 4096), stride = align_up(H + n*CB, 4096), slot s at 8192 + s*stride."""
    MiB = 1 << 20
    # n = 17, CB = 4 MiB: H = 4096 (168 B of fields); stride = 4096 + 71,303,168 = 71,307,264
    assert oracle.header_bytes(17) == 4096
    assert oracle.slot_stride(17, 4 * MiB) == 71_307_264
    assert oracle.slot_offset(0, 17, 4 * MiB) == 8192
    assert oracle.slot_offset(2, 17, 4 * MiB) == 8192 + 2 * 71_307_264 == 142_622_720
    # n = 999 still fits one page (96 + 3996 + 4 = 4096); n = 1000 needs two (4100 -> 8192)
    assert oracle.header_bytes(999) == 4096 and oracle.header_bytes(1000) == 8192
    # n = 1000, CB = 48 (not page-aligned data): stride = align_up(8192 + 48,000, 4096) = 57,344
    assert oracle.slot_stride(1000, 48) == 57_344
    assert oracle.slot_offset(3, 1000, 48) == 8192 + 3 * 57_344 == 180_224
    # n = 0: a bare header page per slot
    assert oracle.slot_stride(0, 64 * MiB) == 4096 and oracle.slot_offset(5, 0, 64 * MiB) == 8192 + 5 * 4096
    # C3 (OPT-1.3B, 236 chunks of 64 MiB): H = align_up(96 + 944 + 4, 4096) = 4096
    assert oracle.slot_offset(4, 236, 64 * MiB) == 8192 + 4 * (4096 + 236 * 64 * MiB)


def test_crc32c_extend_is_crc_of_concatenation(hwcrc):
    rng = np.random.default_rng(11)
    for na, nb in [(0, 0), (0, 7), (1, 1), (5, 4096), (4096, 3), (1 << 16, 1 << 16)]:
        a = rng.integers(0, 256, na, dtype=np.uint8)
        b = rng.integers(0, 256, nb, dtype=np.uint8)
        ab = np.concatenate([a, b])
        assert oracle.crc32c_extend(oracle.crc32c(a), b) == hwcrc(ab) == oracle.crc32c(ab)
    assert oracle.crc32c_extend(0, b"123456789") == 0xE3069283  # RFC 3720 check value from an empty prefix


def test_pack_range_equals_byte_loop():
    """pack_range (numpy slices) == pack (the C byte loop) on every chunk range of tiny
    registrations and on chunk ranges of C1 (97 tensors, 10 under 16 B, one spanning 8 chunks)."""
    rng = np.random.default_rng(12)
    sizes = [0, 1, 15, 16, 17, 40]
    for combo in itertools.product(sizes, repeat=3):
        srcs = [rng.integers(1, 256, n, dtype=np.uint8) for n in combo]
        for cb, align in ((16, 16), (48, 256), (64, 16)):
            full = oracle.pack(srcs, align=align, chunk_bytes=cb)
            c = full.nbytes // cb
            for first in range(c):
                for cnt in range(1, c - first + 1):
                    got = oracle.pack_range(list(combo), lambda i, a, b: srcs[i][a:b], align, cb, first, cnt)
                    assert got.tobytes() == full[first * cb:(first + cnt) * cb].tobytes()
    from synth import config_tensors
    specs = config_tensors("c1")
    nb = [s.nbytes for s in specs]
    srcs = [rng.integers(0, 256, n, dtype=np.uint8) for n in nb]
    cb = 4 << 20
    full = oracle.pack(srcs, 256, cb)
    for first, cnt in [(0, 1), (3, 5), (16, 1), (0, 17)]:
        got = oracle.pack_range(nb, lambda i, a, b: srcs[i][a:b], 256, cb, first, cnt)
        assert np.array_equal(got, full[first * cb:(first + cnt) * cb])


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


def test_fullsize_checker_accepts_oracle_file_and_rejects_faults(tmp_path):
    """The full-size GPU parity helper (tests/test_fullsize_gpu.oracle_check_slot) on a file the
    oracle wrote: it must accept it, and name a changed data byte, a changed CRC-table entry and a
    changed digest."""
    from synth import config_tensors, make_state, host_bytes
    from test_fullsize_gpu import oracle_check_slot
    specs = config_tensors("c1")
    ts = make_state(specs, "cpu", seed=3, it=1)
    cb = 4 << 20
    p = str(tmp_path / "c1.pcc")
    oracle.write_checkpoint(p, [host_bytes(t) for t in ts], [s.code for s in specs], 256, cb, 0, 1, 2, 1, 5, 1, 1)
    n = oracle.layout([s.nbytes for s in specs], 256, cb)[2]
    assert oracle_check_slot(p, specs, ts, 1, n, 0, cb)[0] == n
    base = oracle.slot_offset(1, n, cb)
    H = oracle.header_bytes(n)
    for at, what in [(base + H + 3 * cb + 12345, "chunks differ"), (base + 96 + 4 * 5, "header CRC32C"),
                     (base + 72, "digest")]:
        with open(p, "r+b") as f:
            f.seek(at)
            b = f.read(1)
            f.seek(at)
            f.write(bytes([b[0] ^ 0x10]))
        with pytest.raises(AssertionError, match=what):
            oracle_check_slot(p, specs, ts, 1, n, 0, cb)
        with open(p, "r+b") as f:
            f.seek(at)
            f.write(b)
