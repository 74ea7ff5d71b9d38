"""CPU model of the v7 CRC warps' index math (kernels.cu crc_tile_rot, crc32c.cuh T2 / S4), pinned
to the oracle's CRC32C.  Test infrastructure: it retypes the kernel's address arithmetic — word
rotation by l/4, funnel shift by 8(l mod 4), PRMT(byte c next to 4l) + 4(4i+c) into 256-B rows of
T2, the 4-byte shift through S4 — and checks, with tables built from the oracle's CRC only:

  * the lane register equals raw CRC32C of the lane's 8 spans with their 992-byte gaps (the
    definition the finalize kernel folds);
  * every lookup instruction (fixed i, c or fixed shift byte) hits 32 distinct banks across the
    warp (the claim that the tables need no per-lane copies);
  * the data loads (word (i + l/4) mod 8 of lane l's span) are conflict-free too.
A wrong rotation, a transposed table index or a wrap error in the doubled row fails here.
"""
import numpy as np

import oracle

ZERO_CACHE = {}


def raw(msg: bytes) -> int:
    """raw(M): register after feeding M into a zero register = std(M) ^ std(0^|M|) (linearity)."""
    n = len(msg)
    if n not in ZERO_CACHE:
        ZERO_CACHE[n] = oracle.crc32c(bytes(n))
    return oracle.crc32c(msg) ^ ZERO_CACHE[n]


def tables():
    # T_k[v] = raw(32-byte span with byte v at position k); S_b[v] = shift(v << 8b, 1024 bytes)
    T = np.zeros((32, 256), dtype=np.uint64)
    for k in range(32):
        for v in range(256):
            m = bytearray(32)
            m[k] = v
            T[k, v] = raw(bytes(m))
    S = np.zeros((4, 256), dtype=np.uint64)
    for b in range(4):
        for v in range(256):
            x = (v << (8 * b)).to_bytes(4, "little")
            S[b, v] = raw(x + bytes(1020))  # the register x shifted over 1024 bytes
    # the kernel's shared-memory images (32-bit words)
    T2 = np.zeros(256 * 64, dtype=np.uint64)
    for v in range(256):
        for P in range(64):
            T2[v * 64 + P] = T[P % 32, v]
    S4 = np.zeros(256 * 32, dtype=np.uint64)
    for v in range(256):
        for q in range(8):
            for b in range(4):
                S4[v * 32 + 4 * q + b] = S[b, v]
    return T2, S4


def prmt_byte_next_to(w, L4, c):  # prmt.b32 d, w, L4, 0x7604 | c << 4
    return (((w >> (8 * c)) & 0xFF) << 8) | (L4 & 0xFF)


def funnel_r(lo, hi, n):  # shf.r.clamp.b32: low 32 bits of (hi:lo) >> n
    return (((hi << 32) | lo) >> n) & 0xFFFFFFFF


def lane_register(tile_words, lane, T2, S4, banks):
    q, r = lane >> 2, lane & 3
    L4, r8 = 4 * lane, 8 * r
    O = [32 * lane + 4 * ((i + q) & 7) for i in range(8)]
    SB = [4 * (4 * q + ((c + r) & 3)) for c in range(4)]
    s = 0
    for rho in range(8):
        u = [int(tile_words[(rho * 1024 + O[i]) // 4]) for i in range(8)]
        for i in range(8):
            banks.setdefault(("data", rho, i), []).append(((rho * 1024 + O[i]) // 4) % 32)
        acc = 0
        if rho > 0:
            x = ((s >> r8) | (s << (32 - r8))) & 0xFFFFFFFF if r8 else s
            for c, sh in enumerate((-7, 1, 9, 17)):
                y = (x << 7) if sh < 0 else (x >> sh)
                off = (y & 0x7F80) | SB[c]
                banks.setdefault(("S", rho, c), []).append((off // 4) % 32)
                acc ^= int(S4[off // 4])
        for i in range(8):
            w = funnel_r(u[i], u[(i + 1) & 7], r8)
            for c in range(4):
                off = 4 * (4 * i + c) + prmt_byte_next_to(w, L4, c)
                banks.setdefault(("T", rho, i, c), []).append((off // 4) % 32)
                acc ^= int(T2[off // 4])
        s = acc
    return s


def test_rotated_tables_give_the_lane_registers_and_are_conflict_free():
    T2, S4 = tables()
    rng = np.random.default_rng(17)
    for trial in range(2):
        tile = rng.integers(0, 256, 8192, dtype=np.uint8)
        if trial == 1:
            tile[::7] = 0xFF  # structured bytes too
        words = tile.view("<u4")
        banks = {}
        for lane in range(32):
            got = lane_register(words, lane, T2, S4, banks)
            # definition: raw CRC of span_0 || 0^992 || span_1 || ... || span_7 of this lane
            msg = bytearray()
            for rho in range(8):
                if rho:
                    msg += bytes(992)
                msg += tile[rho * 1024 + 32 * lane: rho * 1024 + 32 * lane + 32].tobytes()
            assert got == raw(bytes(msg)), f"lane {lane}"
        for key, bl in banks.items():
            assert len(bl) == 32 and len(set(bl)) == 32, f"bank conflict in {key}: {sorted(bl)}"


def test_sum_of_lane_registers_is_the_tile_crc():
    """The finalize step the kernels share: shift lane l's register over 32(31-l) bytes and XOR
    the 32 lanes -> raw CRC of the whole 8 KiB tile."""
    T2, S4 = tables()
    rng = np.random.default_rng(3)
    tile = rng.integers(0, 256, 8192, dtype=np.uint8)
    words = tile.view("<u4")
    acc = 0
    for lane in range(32):
        s = lane_register(words, lane, T2, S4, {})
        acc ^= raw(s.to_bytes(4, "little") + bytes(32 * (31 - lane) - 4)) if lane < 31 else s
    assert acc == raw(tile.tobytes())
