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
// One CTA = 8 warps.  Lane-strided layout: in round r, lane l owns the 16-byte word at
// warp_base + r*512 + 16*l, so every warp load / store is a contiguous 512 B.  A lane's
// register is advanced by the 496 zero bytes between its words (gap table G) and then
// absorbs its word with slicing-by-16 (tables T).  Lanes combine with a 5-level shuffle
// tree (tables L[k] shift by 16*2^k bytes), warps with x8n constants, tiles and chunks in
// the finalize kernel.
constexpr int kWarps = 8;
constexpr int kThreads = kWarps * 32;
constexpr int kRounds = 8;                       // rounds per warp per tile
constexpr uint32_t kRound = 512;                 // bytes per warp per round
constexpr uint32_t kWarpBytes = kRounds * kRound;  // 4 KiB per warp
constexpr uint32_t kTile = kWarps * kWarpBytes;    // 32 KiB per CTA tile
constexpr uint32_t kGap = kRound - 16;             // zero bytes between a lane's words

// Shared-memory table block (40 KiB): slicing-by-16, gap shift, 5 tree-level shifts.
struct CrcTables {
    uint32_t T[16][256];     // T[k][b] = raw(b followed by k zero bytes)
    uint32_t G[4][256];      // G[i][b] = shift(b << 8i, kGap): the zero bytes before a lane's next word
    uint32_t L[5][4][256];   // L[k][i][b] = shift(b << 8i, 16 << k)
};
static_assert(sizeof(CrcTables) == 40 * 1024, "table block size");

// Constants that do not need a table.
struct CrcConsts {
    uint32_t x2n[kX2n];
    uint32_t warp_shift[kWarps];  // x8n((kWarps-1-w) * kWarpBytes)
    uint32_t x8n_stride_gap;      // x8n(kThreads*16 - 16): generic (ragged-tile) path, zeros between a thread's words
};

__device__ __forceinline__ uint32_t shift4(const uint32_t (*S)[256], uint32_t v) {
    return S[0][v & 0xFF] ^ S[1][(v >> 8) & 0xFF] ^ S[2][(v >> 16) & 0xFF] ^ S[3][v >> 24];
}

// register s absorbs the 16 bytes w (little-endian words): slicing-by-16.
__device__ __forceinline__ uint32_t update16(const uint32_t (*T)[256], uint32_t s, uint4 w) {
    uint32_t x = w.x ^ s;
    return T[15][x & 0xFF] ^ T[14][(x >> 8) & 0xFF] ^ T[13][(x >> 16) & 0xFF] ^ T[12][x >> 24] ^
           T[11][w.y & 0xFF] ^ T[10][(w.y >> 8) & 0xFF] ^ T[9][(w.y >> 16) & 0xFF] ^ T[8][w.y >> 24] ^
           T[7][w.z & 0xFF] ^ T[6][(w.z >> 8) & 0xFF] ^ T[5][(w.z >> 16) & 0xFF] ^ T[4][w.z >> 24] ^
           T[3][w.w & 0xFF] ^ T[2][(w.w >> 8) & 0xFF] ^ T[1][(w.w >> 16) & 0xFF] ^ T[0][w.w >> 24];
}

}  // namespace pcc
