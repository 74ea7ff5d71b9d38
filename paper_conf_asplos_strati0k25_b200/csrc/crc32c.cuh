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
// One CTA of 32 warps per SM (all warps share one 96 KiB copy of the tables), tile = 256 KiB
// of one chunk, warp region = 8 KiB = 8 rounds of 1 KiB.  In round r lane l owns the 32 bytes
// at warp_base + r*1024 + 32*l: one 256-bit load and one 256-bit store per lane, so every warp
// access is 1 KiB contiguous.  Loads run kAhead rounds ahead in registers.  Per round:
//     x = shift(s, 992);  s = raw16(w0 ^ x);  s = raw16(w1 ^ s)
// (feeding a 16-byte word into register r equals raw16 of the word with its first 4 bytes
// XOR r).  After the last round a lane's register is shifted to its warp-region end
// (shift by 32*(31-l)) and XOR-reduced over the warp: one raw CRC per 8 KiB sub-tile; the
// finalize kernel folds sub-tiles, chunks and the slice digest.
//
// Lookups are NIBBLE tables replicated once per lane: entry (table t, nibble v) of lane l
// sits at word (t*16 + v)*32 + l, i.e. always in bank l.  Every shared load of the CRC is
// therefore conflict-free (1 wavefront), at 36 lookups per 16 bytes.  (Byte-indexed
// slicing-by-16 tables cost 20 lookups per 16 B, but random indices collide in banks ~2.9-way
// on average; ncu showed the L1/shared pipe at 81% with that design, K1 at 0.45 of HBM.)
#ifndef PCC_KWARPS
#define PCC_KWARPS 32
#endif
constexpr int kWarps = PCC_KWARPS;                   // warps per CTA (A/B builds: -DPCC_KWARPS)
constexpr int kThreads = kWarps * 32;
constexpr int kWpl = 2;                              // 16-byte words per lane per round
constexpr uint32_t kLaneSpan = 16 * kWpl;            // 32 B
constexpr uint32_t kRound = 32 * kLaneSpan;          // 1 KiB per warp per round
constexpr uint32_t kWarpBytes = 8192;                // 8 KiB per warp per tile
constexpr int kRounds = kWarpBytes / kRound;         // 8
#ifndef PCC_KAHEAD
#define PCC_KAHEAD 1
#endif
constexpr int kAhead = PCC_KAHEAD;                   // rounds loaded ahead of the CRC (A/B builds: -DPCC_KAHEAD)
constexpr uint32_t kGap = kRound - kLaneSpan;        // zero bytes between a lane's spans
constexpr uint32_t kTile = kWarps * kWarpBytes;      // 256 KiB per CTA tile
constexpr int kMaxTileRows = 512;                    // segment rows staged per tile (more -> read from global)

// Shared-memory table block (160 KiB): 5-bit-indexed tables, replicated once per lane.
// Entry (table t, value v) of lane l is word (t*32 + v)*32 + l: always bank l.  A 16-byte word
// is 26 five-bit groups (25 x 5 bits + 3), the 32-bit register 7 groups (6 x 5 + 2).
constexpr int kG16 = 26;  // 5-bit groups in 128 bits
constexpr int kG32 = 7;   // 5-bit groups in 32 bits
struct CrcTables {
    uint32_t NT[kG16][32][32];  // NT[g][v][l] = raw16(16-byte word whose bits [5g, 5g+5) are v)
    uint32_t NF[kG32][32][32];  // NF[g][v][l] = shift(v << 5g, kGap): the zeros before a lane's next span
    uint32_t NL[kG32][32][32];  // NL[g][v][l] = shift(v << 5g, kLaneSpan*(31-l)): lane -> warp-region end
};
static_assert(sizeof(CrcTables) == 160 * 1024, "table block size");

// Constants that do not need a table.
struct CrcConsts {
    uint32_t x2n[kX2n];
    uint32_t warp_shift[kWarps];  // x8n((kWarps-1-w) * kWarpBytes)
    uint32_t x8n_stride;          // x8n(kThreads*16): generic (ragged-tile) path, one thread stride
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
// (a & 0xF80) | lane4 as ONE opaque LOP3: written in C the compiler re-associates it into an
// AND plus an IADD of a hoisted (table base + lane4) register — one extra instruction per
// lookup; kept opaque, the table base folds into the LDS's uniform-register + immediate.
__device__ __forceinline__ uint32_t grp_off(uint32_t a, uint32_t lane4) {
    uint32_t r;
    asm("lop3.b32 %0, %1, %2, %3, 0xEA;" : "=r"(r) : "r"(a), "r"(0xF80u), "r"(lane4));
    return r;
}

// word c of a 128-bit value (compile-time c)
template <int C>
__device__ __forceinline__ uint32_t comp(const uint4 &w) {
    return C == 0 ? w.x : C == 1 ? w.y : C == 2 ? w.z : C == 3 ? w.w : 0u;
}

// bits [B, B+5) of the little-endian bit string `w`, moved to bits 7..11 (table stride 128 B)
template <int B>
__device__ __forceinline__ uint32_t grp_bits(const uint4 &w) {
    constexpr int wi = B / 32, bi = B % 32;
    const uint32_t lo = comp<wi>(w);
    if constexpr (bi <= 7) {
        return lo * (1u << (7 - bi));  // left shift (IMAD)
    } else if constexpr (bi <= 27) {
        return shr_fma(lo, 1u << (39 - bi));  // right shift by bi-7 (IMAD.HI)
    } else {
        return funnel_r(lo, comp<wi + 1>(w), bi - 7);  // the group crosses into the next word
    }
}

template <int G>
__device__ __forceinline__ uint32_t lk(const char *tab, uint32_t lane4, const uint4 &w) {
    return *reinterpret_cast<const uint32_t *>(tab + G * 4096 + grp_off(grp_bits<5 * G>(w), lane4));
}

// raw16(w): the CRC register of the 16 bytes w fed into a zero register (26 lookups);
// raw16(w with w.x ^= r) = the register r after absorbing w.
__device__ __forceinline__ uint32_t raw16(const CrcTables &tb, uint32_t lane4, const uint4 &w) {
    const char *t = reinterpret_cast<const char *>(&tb.NT[0][0][0]);
    uint32_t a = lk<0>(t, lane4, w) ^ lk<1>(t, lane4, w) ^ lk<2>(t, lane4, w);
    uint32_t b = lk<3>(t, lane4, w) ^ lk<4>(t, lane4, w) ^ lk<5>(t, lane4, w);
    uint32_t c = lk<6>(t, lane4, w) ^ lk<7>(t, lane4, w) ^ lk<8>(t, lane4, w);
    uint32_t d = lk<9>(t, lane4, w) ^ lk<10>(t, lane4, w) ^ lk<11>(t, lane4, w);
    uint32_t e = lk<12>(t, lane4, w) ^ lk<13>(t, lane4, w) ^ lk<14>(t, lane4, w);
    uint32_t f = lk<15>(t, lane4, w) ^ lk<16>(t, lane4, w) ^ lk<17>(t, lane4, w);
    uint32_t g = lk<18>(t, lane4, w) ^ lk<19>(t, lane4, w) ^ lk<20>(t, lane4, w);
    uint32_t h = lk<21>(t, lane4, w) ^ lk<22>(t, lane4, w) ^ lk<23>(t, lane4, w);
    uint32_t i = lk<24>(t, lane4, w) ^ lk<25>(t, lane4, w);
    return a ^ b ^ c ^ d ^ e ^ f ^ g ^ h ^ i;
}

// a 32-bit register through one of the 7-table sets (NF / NL): 7 lookups
__device__ __forceinline__ uint32_t shift32(const char *tab, uint32_t lane4, uint32_t x) {
    const uint4 w = make_uint4(x, 0, 0, 0);
    return lk<0>(tab, lane4, w) ^ lk<1>(tab, lane4, w) ^ lk<2>(tab, lane4, w) ^ lk<3>(tab, lane4, w) ^
           lk<4>(tab, lane4, w) ^ lk<5>(tab, lane4, w) ^ lk<6>(tab, lane4, w);
}

}  // namespace pcc
