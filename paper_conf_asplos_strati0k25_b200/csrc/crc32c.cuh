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
constexpr int kWarps = 32;
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

// Shared-memory table block (96 KiB), per-lane replicated nibble tables.
struct CrcTables {
    uint32_t NT[32][16][32];  // NT[q][v][l] = raw16(16-byte word whose nibble q is v, others 0)
    uint32_t NF[8][16][32];   // NF[q][v][l] = shift(v << 4q, kGap): the zeros before a lane's next span
    uint32_t NL[8][16][32];   // NL[q][v][l] = shift(v << 4q, kLaneSpan*(31-l)): lane -> warp-region end
};
static_assert(sizeof(CrcTables) == 96 * 1024, "table block size");

// Constants that do not need a table.
struct CrcConsts {
    uint32_t x2n[kX2n];
    uint32_t warp_shift[kWarps];  // x8n((kWarps-1-w) * kWarpBytes)
    uint32_t x8n_stride;          // x8n(kThreads*16): generic (ragged-tile) path, one thread stride
};

// XOR of the 8 nibble-table entries selected by the nibbles of x.  `tab` = byte address of
// table t0 (a shared-memory constant), lane4 = lane*4; entry (t0+k, v) of this lane lives at
// tab + k*2048 + v*128 + lane4.  ((x >> 4k) & 15) << 7 == (x >> (4k-7)) & 0x780.
// x >> k as IMAD.HI on the FMA pipe (a plain >> becomes SHF on the ALU pipe, which the
// LOP3s of the lookups already saturate); mul.hi by a power of two is not strength-reduced.
__device__ __forceinline__ uint32_t shr_fma(uint32_t x, uint32_t pow2) {
    uint32_t r;
    asm("mul.hi.u32 %0, %1, %2;" : "=r"(r) : "r"(x), "r"(pow2));
    return r;
}

// (a & 0x780) | lane4 as ONE opaque LOP3: written in C the compiler re-associates it into an
// AND plus an IADD of a hoisted (table base + lane4) register — one extra instruction per
// lookup; kept opaque, the table base folds into the LDS's uniform-register + immediate.
__device__ __forceinline__ uint32_t nib_off(uint32_t a, uint32_t lane4) {
    uint32_t r;
    asm("lop3.b32 %0, %1, %2, %3, 0xEA;" : "=r"(r) : "r"(a), "r"(0x780u), "r"(lane4));
    return r;
}

__device__ __forceinline__ uint32_t nib8(const char *tab, uint32_t lane4, uint32_t x) {
    const uint32_t o0 = nib_off(x * 128u, lane4);                 // nibble 0: << 7
    const uint32_t o1 = nib_off(x * 8u, lane4);                   // nibble 1: << 3
    const uint32_t o2 = nib_off(shr_fma(x, 1u << 31), lane4);     // nibble k: >> (4k-7)
    const uint32_t o3 = nib_off(shr_fma(x, 1u << 27), lane4);
    const uint32_t o4 = nib_off(shr_fma(x, 1u << 23), lane4);
    const uint32_t o5 = nib_off(shr_fma(x, 1u << 19), lane4);
    const uint32_t o6 = nib_off(shr_fma(x, 1u << 15), lane4);
    const uint32_t o7 = nib_off(shr_fma(x, 1u << 11), lane4);
    const uint32_t a = *reinterpret_cast<const uint32_t *>(tab + 0 * 2048 + o0) ^
                       *reinterpret_cast<const uint32_t *>(tab + 1 * 2048 + o1) ^
                       *reinterpret_cast<const uint32_t *>(tab + 2 * 2048 + o2);
    const uint32_t b = *reinterpret_cast<const uint32_t *>(tab + 3 * 2048 + o3) ^
                       *reinterpret_cast<const uint32_t *>(tab + 4 * 2048 + o4) ^
                       *reinterpret_cast<const uint32_t *>(tab + 5 * 2048 + o5);
    const uint32_t c = *reinterpret_cast<const uint32_t *>(tab + 6 * 2048 + o6) ^
                       *reinterpret_cast<const uint32_t *>(tab + 7 * 2048 + o7);
    return a ^ b ^ c;
}

// raw16(w): CRC register of the 16 bytes w fed into a zero register (32 nibble lookups).
// raw16(w with w.x ^= r) = the register r after absorbing w.
__device__ __forceinline__ uint32_t raw16(const CrcTables &tb, uint32_t lane4, uint4 w) {
    const char *t = reinterpret_cast<const char *>(&tb.NT[0][0][0]);
    return nib8(t, lane4, w.x) ^ nib8(t + 8 * 2048, lane4, w.y) ^ nib8(t + 16 * 2048, lane4, w.z) ^
           nib8(t + 24 * 2048, lane4, w.w);
}

}  // namespace pcc
