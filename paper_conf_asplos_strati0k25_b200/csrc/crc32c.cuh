// crc32c.cuh — CRC32C arithmetic for the snapshot kernels (K3 of SURVEY §2.3).
//
// CRC32C (Castagnoli, reflected polynomial 0x82F63B78, init/xorout 0xFFFFFFFF) is the
// per-chunk checksum BASELINE.json's north_star fixes (reading R4; the paper
// itself has no checksum).  Everything here is GF(2)-linear algebra on the 32-bit register,
// written for the GPU's shared-memory / ALU pipes:
//
//   raw(M)            register after feeding M into a zero register (no init / xorout)
//   std(M)            = raw(M) ^ shift(0xFFFFFFFF, |M|) ^ 0xFFFFFFFF
//   raw(A || B)       = shift(raw(A), |B|) ^ raw(B)        (zero-init CRC is linear)
//   shift(v, n)       = v * x^(8n) mod P  (multmodp with x8n(n), or 4 byte-sliced tables)
//
// Independence: this file shares no code, table or generator with oracle/ (the oracle is
// a byte-at-a-time Sarwate loop in plain C).  Tables here are generated on the device.
#pragma once
#include <cstdint>

namespace pcc {

constexpr uint32_t kPoly = 0x82F63B78u;

// a * b mod P for reflected polynomials (bit 31 = x^0).  a == 0 -> 0.
__host__ __device__ __forceinline__ uint32_t multmodp(uint32_t a, uint32_t b) {
    uint32_t p = 0;
    uint32_t m = 1u << 31;
    while (a) {
        if (a & m) {
            p ^= b;
            a &= ~m;
        }
        m >>= 1;
        b = (b & 1u) ? (b >> 1) ^ kPoly : (b >> 1);
    }
    return p;
}

// x^(2^k) mod P for k = 0..63 (reflected).  No period-32 shortcut: unlike the IEEE CRC-32
// polynomial, the multiplicative order of x modulo the Castagnoli polynomial does not divide
// 2^32 - 1, so x^(2^(k+32)) != x^(2^k) in general (a 1.1 GB digest caught this).
constexpr int kX2n = 64;
__host__ __device__ inline void make_x2n(uint32_t *x2n) {
    uint32_t p = 1u << 30;  // x^1
    x2n[0] = p;
    for (int k = 1; k < kX2n; ++k) x2n[k] = p = multmodp(p, p);
}

// x^(8n) mod P using x2n[] (n bytes of zeros), n < 2^61.
__host__ __device__ inline uint32_t x8n(const uint32_t *x2n, uint64_t n) {
    uint32_t p = 1u << 31;  // x^0
    int k = 3;
    while (n) {
        if (n & 1) p = multmodp(x2n[k], p);
        n >>= 1;
        ++k;
    }
    return p;
}

// ---------------------------------------------------------------- kernel geometry
// One CTA per SM (all warps share one copy of the tables); the work item is an 8 KiB tile of
// one chunk, owned by one warp = 8 rounds of 1 KiB.  In round r lane l owns the 32 bytes at
// warp_base + r*1024 + 32*l: one 256-bit load and one 256-bit store per lane, so every warp
// access is 1 KiB contiguous.  Loads run kAheadOf<> rounds ahead in registers, and the round
// after those is prefetched into L2 (kPf2Of<>).  Per round:
//     x = shift(s, 992);  s = raw16(w0 ^ x);  s = raw16(w1 ^ s)
// (feeding a 16-byte word into register r equals raw16 of the word with its first 4 bytes
// XOR r).  After the last round every lane writes its register (relative to the end of its
// last span) to global memory; the finalize kernel shifts each lane to its warp-region end
// (NL tables, shift by 32*(31-l)), XORs a warp's 32 lanes into the 8 KiB sub-tile's raw CRC and
// folds sub-tiles, chunks and the slice digest.
//
// Lookups are tables replicated once per lane: entry (table t, value v) of lane l sits at
// word (t*V + v)*32 + l, i.e. always in bank l, so every shared load of the CRC is
// conflict-free (1 wavefront).  NT (the 16-byte word -> register map) is indexed by
// kNtBits-bit groups: 6 bits = 22 lookups per 16 B in 169 KiB; NF (the 992-byte gap shift of
// the register) by 5-bit groups, 7 lookups in 24.5 KiB.  A last group narrower than the others
// gets a table of only its own 2^bits values.  (Byte-indexed slicing-by-16 tables cost 20
// lookups per 16 B, but random indices collide in banks ~2.9-way on average; ncu showed the
// L1/shared pipe at 81% with that design, K1 at 0.45 of HBM.)
// Warps per CTA and rounds of loads held in registers ahead of the CRC, per direction (K1 packs,
// K2 unpacks; measured in DESIGN.md §6: K1 prefers 32 warps x 1 round, K2 28 warps x 2 rounds).
// A/B builds override them with -DPCC_KWARPS_PACK=... etc.
#ifndef PCC_KWARPS_PACK
#define PCC_KWARPS_PACK 32
#endif
#ifndef PCC_KAHEAD_PACK
#define PCC_KAHEAD_PACK 1
#endif
#ifndef PCC_KWARPS_UNPACK
#define PCC_KWARPS_UNPACK 28
#endif
#ifndef PCC_KAHEAD_UNPACK
#define PCC_KAHEAD_UNPACK 2
#endif
// Per-lane L2 prefetch of the round after the ones in registers (no registers): K1 +2-3.5%;
// K2 at 28 warps x 2 rounds loses 4% with it (ncu 400 -> 416 us), so only K1 uses it
#ifndef PCC_PF2_PACK
#define PCC_PF2_PACK 1
#endif
#ifndef PCC_PF2_UNPACK
#define PCC_PF2_UNPACK 0
#endif
// K1 also prefetches the first rounds of a warp's next item during its last rounds (+1.5-2%)
#ifndef PCC_XPF
#define PCC_XPF 1
#endif
constexpr bool kXpf = PCC_XPF != 0;
template <bool kPack> constexpr int kWarpsOf = kPack ? PCC_KWARPS_PACK : PCC_KWARPS_UNPACK;
template <bool kPack> constexpr int kThreadsOf = kWarpsOf<kPack> * 32;
template <bool kPack> constexpr int kAheadOf = kPack ? PCC_KAHEAD_PACK : PCC_KAHEAD_UNPACK;
template <bool kPack> constexpr bool kPf2Of = kPack ? PCC_PF2_PACK != 0 : PCC_PF2_UNPACK != 0;
constexpr int kWpl = 2;                              // 16-byte words per lane per round
constexpr uint32_t kLaneSpan = 16 * kWpl;            // 32 B
constexpr uint32_t kRound = 32 * kLaneSpan;          // 1 KiB per warp per round
constexpr uint32_t kWarpBytes = 8192;                // 8 KiB per warp per tile
constexpr int kRounds = kWarpBytes / kRound;         // 8
#ifndef PCC_KRUN
#define PCC_KRUN 1
#endif
// A lane's spans are contiguous for kRun rounds (a "run" of kRun*32 B); round r of lane l sits
// at (r / kRun) * kRun*kRound + l * kRun*kLaneSpan + (r % kRun) * kLaneSpan of the warp tile.
// kRun = 1: every warp access is 1 KiB contiguous and the register crosses a gap every round;
// larger kRun trades coalescing for fewer gap shifts (none at kRun = kRounds).
constexpr int kRun = PCC_KRUN;                       // (A/B builds: -DPCC_KRUN)
constexpr uint32_t kLaneRun = kRun * kLaneSpan;      // contiguous bytes of one lane
constexpr uint32_t kGap = kRun * kRound - kLaneRun;  // zero bytes between a lane's runs
constexpr uint32_t kTile = kWarpBytes;               // a work item: one warp's 8 KiB of one chunk
constexpr int kLaneOut = 32;                         // raw CRCs K1/K2 write per warp sub-tile (one per lane)

#ifndef PCC_NTBITS
#define PCC_NTBITS 6
#endif
constexpr int kNtBits = PCC_NTBITS;                  // NT group width (A/B builds: -DPCC_NTBITS=5)
constexpr int kNtVals = 1 << kNtBits;
constexpr int kG16 = (128 + kNtBits - 1) / kNtBits;  // groups in a 16-byte word: 22 (6-bit) / 26 (5-bit)
constexpr int kNtLastBits = 128 - (kG16 - 1) * kNtBits;
constexpr int kG32 = 7;                              // 5-bit groups in the 32-bit register (6 x 5 + 2)
constexpr uint32_t kNtTab = kNtVals * 128;           // bytes per full NT table (V values x 32 lanes x 4 B)
constexpr uint32_t kNtBytes = (kG16 - 1) * kNtTab + (1u << kNtLastBits) * 128;
constexpr uint32_t kRegTab = 32 * 128;               // bytes per full NF / NL table
constexpr uint32_t kRegBytes = (kG32 - 1) * kRegTab + (1u << 2) * 128;

// ------------------------------------------------ bank-rotated byte tables (the TMA kernels)
// The TMA-staged K1/K2 (v7, kernels.cu k_snap_tma) compute the SAME lane registers as the
// register-path kernel above, with byte-sliced tables that are conflict-free WITHOUT per-lane
// replication.  Per round a lane's register becomes
//     s' = raw32(span) ^ shift(s, 1024)          (the gap 992 + the span's own 32 bytes)
// raw32(span) = XOR over the 32 byte positions k of T_k[byte k]; shift(s, 1024) = XOR over
// the register's 4 bytes b of S_b[byte b].  Conflict-freedom comes from rotating the DATA, not
// from replicating the tables: lane l holds its span rotated by l bytes (register i byte c =
// span byte (4i + c + l) mod 32), so in the instruction for (i, c) lane l reads table
// T_{(4i+c+l) mod 32}, and T_k lives in bank k: 32 lanes, 32 different banks.
//   T2[v][P] (P = 0..63, 256-B rows) = T_{P mod 32}[v]: a lane's address is (v << 8) + 4l (one
//            PRMT: byte c of the register next to 4l) + 4(4i + c) (the LDS immediate); the
//            doubled row absorbs the wrap of 4i + c + l past 31.
//   S4[v][4q + b'] (128-B rows) = S_{b'}[v] for each q = l >> 2: the register rotated by
//            r = l & 3 bytes puts table S_{(c+r) & 3} at bank 4q + ((c + r) & 3).
// 36 lookups per 32 B (51 above) in 96 KiB of tables (193 KiB above), which leaves shared
// memory for a 128 KiB TMA staging ring.
constexpr uint32_t kT2Bytes = 256 * 64 * 4;  // 64 KiB
constexpr uint32_t kS4Bytes = 256 * 32 * 4;  // 32 KiB
constexpr uint32_t kTmaTableBytes = kT2Bytes + kS4Bytes;

// Table block.  K1/K2 load NT + NF (the first kK1TableBytes) into shared memory; NL is read by
// the finalize kernel only.  Word index of entry (t, v, l): t*V*32 + v*32 + l inside each part.
// The TMA kernels load T2 + S4 (kTmaTableBytes, contiguous).
struct CrcTables {
    uint32_t NT[kNtBytes / 4];   // NT[t][v][l] = raw16(16-byte word whose bits [kNtBits*t, +kNtBits) are v)
    uint32_t NF[kRegBytes / 4];  // NF[g][v][l] = shift(v << 5g, kGap): the zeros before a lane's next span
    uint32_t NL[kRegBytes / 4];  // NL[g][v][l] = shift(v << 5g, kLaneRun*(31-l)): lane -> warp-region end
    uint32_t T2[kT2Bytes / 4];   // T2[v*64 + P] = raw32(byte v at position P mod 32 of a 32-byte span)
    uint32_t S4[kS4Bytes / 4];   // S4[v*32 + 4q + b] = shift(v << 8b, 1024)
};
constexpr uint32_t kK1TableBytes = kNtBytes + kRegBytes;
static_assert(kK1TableBytes % 16 == 0, "TMA bulk copy size");
static_assert(kK1TableBytes + 1024 <= 227 * 1024, "K1 shared memory");
static_assert(kTmaTableBytes % 16 == 0 && (kNtBytes + 2 * kRegBytes) % 16 == 0, "TMA bulk copy size / alignment");

// Constants that do not need a table.
struct CrcConsts {
    uint32_t x2n[kX2n];
    uint32_t x8n_stride;          // x8n(32*16): generic (ragged-tile) path, one warp stride
};

// x >> k as IMAD.HI on the FMA pipe (a plain >> becomes SHF on the ALU pipe, which the
// LOP3s of the lookups already saturate); mul.hi by a power of two is not strength-reduced.
__device__ __forceinline__ uint32_t shr_fma(uint32_t x, uint32_t pow2) {
    uint32_t r;
    asm("mul.hi.u32 %0, %1, %2;" : "=r"(r) : "r"(x), "r"(pow2));
    return r;
}
// (hi:lo) >> n, low 32 bits (one SHF)
__device__ __forceinline__ uint32_t funnel_r(uint32_t lo, uint32_t hi, uint32_t n) {
    uint32_t r;
    asm("shf.r.clamp.b32 %0, %1, %2, %3;" : "=r"(r) : "r"(lo), "r"(hi), "r"(n));
    return r;
}
// (a & mask) | lane4 as ONE opaque LOP3: written in C the compiler re-associates it into an
// AND plus an IADD of a hoisted (table base + lane4) register — one extra instruction per
// lookup; kept opaque, the table base folds into the LDS's uniform-register + immediate.
template <uint32_t kMask>
__device__ __forceinline__ uint32_t grp_off(uint32_t a, uint32_t lane4) {
    uint32_t r;
    asm("lop3.b32 %0, %1, %2, %3, 0xEA;" : "=r"(r) : "r"(a), "r"(kMask), "r"(lane4));
    return r;
}

// word c of a 128-bit value (compile-time c)
template <int C>
__device__ __forceinline__ uint32_t comp(const uint4 &w) {
    return C == 0 ? w.x : C == 1 ? w.y : C == 2 ? w.z : C == 3 ? w.w : 0u;
}

// bits [B, B+W) of the little-endian bit string `w`, moved to bits 7.. (table stride 128 B);
// higher garbage bits are masked by grp_off
template <int B, int W>
__device__ __forceinline__ uint32_t grp_bits(const uint4 &w) {
    constexpr int wi = B / 32, bi = B % 32;
    const uint32_t lo = comp<wi>(w);
    if constexpr (bi <= 7) {
        return lo * (1u << (7 - bi));  // left shift (IMAD)
    } else if constexpr (bi + W <= 32) {
        return shr_fma(lo, 1u << (39 - bi));  // right shift by bi-7 (IMAD.HI)
    } else {
        return funnel_r(lo, comp<wi + 1>(w), bi - 7);  // the group crosses into the next word
    }
}

// entry of table G (groups of W bits, tables of kTab bytes) for the group's value in `w`
template <int G, int W, uint32_t kTab>
__device__ __forceinline__ uint32_t lk(const char *tab, uint32_t lane4, const uint4 &w) {
    constexpr uint32_t kMask = ((1u << W) - 1u) << 7;
    return *reinterpret_cast<const uint32_t *>(tab + G * kTab + grp_off<kMask>(grp_bits<W * G, W>(w), lane4));
}

template <int G>
__device__ __forceinline__ uint32_t nt(const char *t, uint32_t lane4, const uint4 &w) {
    if constexpr (G < kG16) return lk<G, kNtBits, kNtTab>(t, lane4, w);
    else return 0u;
}

// raw16(w): the CRC register of the 16 bytes w fed into a zero register (kG16 lookups);
// raw16(w with w.x ^= r) = the register r after absorbing w.  XOR tree in 3-input LOP3s.
__device__ __forceinline__ uint32_t raw16(const char *t, uint32_t lane4, const uint4 &w) {
    uint32_t a = nt<0>(t, lane4, w) ^ nt<1>(t, lane4, w) ^ nt<2>(t, lane4, w);
    uint32_t b = nt<3>(t, lane4, w) ^ nt<4>(t, lane4, w) ^ nt<5>(t, lane4, w);
    uint32_t c = nt<6>(t, lane4, w) ^ nt<7>(t, lane4, w) ^ nt<8>(t, lane4, w);
    uint32_t d = nt<9>(t, lane4, w) ^ nt<10>(t, lane4, w) ^ nt<11>(t, lane4, w);
    uint32_t e = nt<12>(t, lane4, w) ^ nt<13>(t, lane4, w) ^ nt<14>(t, lane4, w);
    uint32_t f = nt<15>(t, lane4, w) ^ nt<16>(t, lane4, w) ^ nt<17>(t, lane4, w);
    uint32_t g = nt<18>(t, lane4, w) ^ nt<19>(t, lane4, w) ^ nt<20>(t, lane4, w);
    uint32_t h = nt<21>(t, lane4, w) ^ nt<22>(t, lane4, w) ^ nt<23>(t, lane4, w);
    uint32_t i = nt<24>(t, lane4, w) ^ nt<25>(t, lane4, w);
    static_assert(kG16 <= 26, "raw16 unrolls at most 26 groups");
    return a ^ b ^ c ^ d ^ e ^ f ^ g ^ h ^ i;
}

// a 32-bit register through one of the 7-table (5-bit) sets NF / NL: 7 lookups
__device__ __forceinline__ uint32_t shift32(const char *tab, uint32_t lane4, uint32_t x) {
    const uint4 w = make_uint4(x, 0, 0, 0);
    return lk<0, 5, kRegTab>(tab, lane4, w) ^ lk<1, 5, kRegTab>(tab, lane4, w) ^ lk<2, 5, kRegTab>(tab, lane4, w) ^
           lk<3, 5, kRegTab>(tab, lane4, w) ^ lk<4, 5, kRegTab>(tab, lane4, w) ^ lk<5, 5, kRegTab>(tab, lane4, w) ^
           lk<6, 5, kRegTab>(tab, lane4, w);
}

}  // namespace pcc
