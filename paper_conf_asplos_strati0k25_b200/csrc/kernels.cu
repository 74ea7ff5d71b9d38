// kernels.cu — K1 (gather-pack + CRC32C), K2 (unpack-verify-scatter), the CRC finalize
// kernel and the table builders, for sm_100a.
//
// K1 is the snapshot copy C_x of PAPER.md Fig 3/Fig 6 (L75, L131, L139 §3.1): it reads
// every registered tensor out of HBM exactly once and lays the bytes into fixed-size
// chunks (reading R1: registration order, 256-B aligned, zero pads), computing the
// per-chunk CRC32C of BASELINE.json's north_star (R4) on the way.  K2 is the recovery
// load of L287 §4.2 with verification (R13).  No floating point is involved: bytes are
// moved verbatim, so NaN payloads / denormals survive (R1).
//
// Execution model:
//   * one CTA = 8 warps processes 32 KiB tiles of one chunk, grid-stride over
//     (chunk, tile) items; grid = SMs x resident CTAs (or the pack_ctas cap);
//   * in each of 8 rounds a warp moves 512 contiguous bytes: every lane one 16-B
//     vector (ld.global.nc.v4 / st.global.cs.v4) — all 8 rounds are loaded before any
//     CRC work so 8 x 16 B per lane are in flight;
//   * the segment-table row under each word is tracked by a per-lane cursor; a 16-B word
//     holds bytes of at most one row because rows start 16-B aligned in the chunk;
//   * CRC: per-lane register, advanced by the gap table and slicing-by-16 (20 shared
//     memory lookups per 16 B), 5-level shuffle tree, warp combine with x8n constants;
//     tile CRCs go to global memory and k_finalize folds tiles -> chunk -> slice digest.
#include <cuda_runtime.h>
#include <cstdint>
#include <mutex>

#include "kernels.hpp"

namespace pcc {

// ------------------------------------------------------------------ table builders
__global__ void k_build_tables(CrcTables *tb, CrcConsts *cs) {
    __shared__ uint32_t x2n[kX2n];
    const int b = threadIdx.x;  // 256 threads
    if (b == 0) make_x2n(x2n);
    // T[0]: the byte-wise table, T[k]: byte followed by k zero bytes
    uint32_t r = b;
    for (int k = 0; k < 8; ++k) r = (r & 1u) ? (r >> 1) ^ kPoly : (r >> 1);
    tb->T[0][b] = r;
    __syncthreads();
    __threadfence_block();
    for (int k = 1; k < 16; ++k) {
        uint32_t v = tb->T[k - 1][b];
        v = (v >> 8) ^ tb->T[0][v & 0xFF];
        tb->T[k][b] = v;
        __syncthreads();
    }
    const uint32_t g = x8n(x2n, kGap);
    for (int i = 0; i < 4; ++i) tb->G[i][b] = multmodp(g, (uint32_t)b << (8 * i));
    for (int k = 0; k < 5; ++k) {
        const uint32_t m = x8n(x2n, 16u << k);
        for (int i = 0; i < 4; ++i) tb->L[k][i][b] = multmodp(m, (uint32_t)b << (8 * i));
    }
    if (b < kX2n) cs->x2n[b] = x2n[b];
    if (b < kWarps) cs->warp_shift[b] = x8n(x2n, (uint64_t)(kWarps - 1 - b) * kWarpBytes);
    if (b == 0) cs->x8n_stride_gap = x8n(x2n, (uint64_t)kThreads * 16 - 16);
}

__global__ void k_setup_geometry(uint32_t *tile_shift, uint32_t *chunk_shift, uint32_t *ff, const CrcConsts *cs,
                                 uint64_t cb, uint32_t n, uint32_t tpc) {
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < tpc) {
        uint64_t end = (uint64_t)(i + 1) * kTile;
        if (end > cb) end = cb;
        tile_shift[i] = x8n(cs->x2n, cb - end);
    }
    if (i < n) chunk_shift[i] = x8n(cs->x2n, (uint64_t)(n - 1 - i) * cb);
    if (i == 0) {
        ff[0] = multmodp(x8n(cs->x2n, cb), 0xFFFFFFFFu);
        ff[1] = multmodp(x8n(cs->x2n, (uint64_t)n * cb), 0xFFFFFFFFu);
    }
}

// ------------------------------------------------------------------ memory helpers
__device__ __forceinline__ uint4 ld_stream(const void *p) {
    uint4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
                 : "l"(p));
    return v;
}
__device__ __forceinline__ void st_stream(void *p, uint4 v) {
    asm volatile("st.global.cs.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
                 : "memory");
}

// first row in [lo, hi) whose end (dst_off + len) is > pos
__device__ __forceinline__ int lower_row(const SegRow *rows, int lo, int hi, uint32_t pos) {
    while (lo < hi) {
        int mid = (lo + hi) >> 1;
        SegRow r = rows[mid];
        if (r.dst_off + r.len <= pos) lo = mid + 1; else hi = mid;
    }
    return lo;
}

// Per-lane cursor over the rows of one chunk.  Positions fed to it only increase.
struct RowCursor {
    const SegRow *rows;
    int cur, end;
    uint64_t ptr;
    uint32_t off, stop;  // [off, stop) = the current row's chunk range
    __device__ __forceinline__ void init(const SegRow *r, int lo, int hi, uint32_t pos) {
        rows = r;
        end = hi;
        cur = lower_row(r, lo, hi, pos);
        load();
    }
    __device__ __forceinline__ void load() {
        if (cur < end) {
            SegRow r = rows[cur];
            ptr = r.ptr;
            off = r.dst_off;
            stop = r.dst_off + r.len;
        } else {
            off = stop = 0xFFFFFFFFu;
        }
    }
    // Returns bytes of the row under [p, p+16) (0 = pad) and the row address of byte p.
    __device__ __forceinline__ uint32_t at(uint32_t p, uint64_t &addr) {
        while (cur < end && stop <= p) {
            ++cur;
            load();
        }
        if (cur >= end || p < off) return 0;
        addr = ptr + (p - off);
        const uint32_t k = stop - p;
        return k < 16 ? k : 16;
    }
};

__device__ __forceinline__ uint4 load_bytes(uint64_t addr, uint32_t k) {
    uint32_t w[4] = {0, 0, 0, 0};
    const uint8_t *s = reinterpret_cast<const uint8_t *>(addr);
    if (k == 16 && (addr & 3) == 0) {
        const uint32_t *s4 = reinterpret_cast<const uint32_t *>(addr);
#pragma unroll
        for (int i = 0; i < 4; ++i) w[i] = __ldg(s4 + i);
    } else {
        for (uint32_t i = 0; i < k; ++i) w[i >> 2] |= (uint32_t)__ldg(s + i) << (8 * (i & 3));
    }
    return make_uint4(w[0], w[1], w[2], w[3]);
}

__device__ __forceinline__ void store_bytes(uint64_t addr, uint32_t k, uint4 v) {
    const uint32_t w[4] = {v.x, v.y, v.z, v.w};
    if (k == 16 && (addr & 15) == 0) {
        *reinterpret_cast<uint4 *>(addr) = v;
    } else if (k == 16 && (addr & 3) == 0) {
        uint32_t *d = reinterpret_cast<uint32_t *>(addr);
#pragma unroll
        for (int i = 0; i < 4; ++i) d[i] = w[i];
    } else {
        uint8_t *d = reinterpret_cast<uint8_t *>(addr);
        for (uint32_t i = 0; i < k; ++i) d[i] = (uint8_t)(w[i >> 2] >> (8 * (i & 3)));
    }
}

// gather the 16-byte image word at chunk position p
__device__ __forceinline__ uint4 gather_word(RowCursor &rc, uint32_t p) {
    uint64_t addr = 0;
    const uint32_t k = rc.at(p, addr);
    if (k == 16 && (addr & 15) == 0) return ld_stream(reinterpret_cast<const void *>(addr));
    if (k == 0) return make_uint4(0, 0, 0, 0);
    return load_bytes(addr, k);
}

__device__ __forceinline__ void scatter_word(RowCursor &rc, uint32_t p, uint4 v) {
    uint64_t addr = 0;
    const uint32_t k = rc.at(p, addr);
    if (k) store_bytes(addr, k, v);
}

// ------------------------------------------------------------------------- K1 / K2
template <bool kPack>
__device__ __forceinline__ uint32_t tile_fast(const SnapParams &P, const CrcTables &tb, char *chunk,
                                              const uint32_t *warp_shift, uint32_t *warp_crc, int rb, int re,
                                              uint32_t tile0) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t wbase = tile0 + warp * kWarpBytes;
    RowCursor rc;
    rc.init(P.rows, rb, re, wbase + lane * 16);
    uint4 w[kRounds];
    if (kPack) {
#pragma unroll
        for (int r = 0; r < kRounds; ++r) w[r] = gather_word(rc, wbase + r * kRound + lane * 16);
#pragma unroll
        for (int r = 0; r < kRounds; ++r) st_stream(chunk + wbase + r * kRound + lane * 16, w[r]);
    } else {
#pragma unroll
        for (int r = 0; r < kRounds; ++r) w[r] = ld_stream(chunk + wbase + r * kRound + lane * 16);
    }
    uint32_t s = 0;
#pragma unroll
    for (int r = 0; r < kRounds; ++r) {
        s = shift4(tb.G, s);
        s = update16(tb.T, s, w[r]);
    }
    if (!kPack) {
#pragma unroll
        for (int r = 0; r < kRounds; ++r) scatter_word(rc, wbase + r * kRound + lane * 16, w[r]);
    }
    // lanes -> warp: level k joins groups of 2^k lanes; the right group spans 16*2^k bytes
#pragma unroll
    for (int k = 0; k < 5; ++k) {
        const uint32_t o = __shfl_up_sync(0xFFFFFFFFu, s, 1 << k);
        if ((lane & ((2 << k) - 1)) == (2 << k) - 1) s = shift4(tb.L[k], o) ^ s;
    }
    if (lane == 31) warp_crc[warp] = multmodp(warp_shift[warp], s);
    __syncthreads();
    uint32_t t = 0;
    if (threadIdx.x == 0) {
#pragma unroll
        for (int i = 0; i < kWarps; ++i) t ^= warp_crc[i];
    }
    return t;  // valid in thread 0
}

// Ragged tile (tile_len < kTile, a multiple of 16): block-strided words, generic shifts.
template <bool kPack>
__device__ __noinline__ uint32_t tile_generic(const SnapParams &P, const CrcTables &tb, char *chunk,
                                              uint32_t *warp_crc, int rb, int re, uint32_t tile0,
                                              uint32_t tile_len) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t tile_end = tile0 + tile_len;
    RowCursor rc;
    rc.init(P.rows, rb, re, tile0 + threadIdx.x * 16);
    uint32_t s = 0, e = 0;
    bool any = false;
    for (uint32_t p = tile0 + threadIdx.x * 16; p < tile_end; p += kThreads * 16) {
        uint4 w;
        if (kPack) {
            w = gather_word(rc, p);
            st_stream(chunk + p, w);
        } else {
            w = ld_stream(chunk + p);
            scatter_word(rc, p, w);
        }
        if (any) s = multmodp(P.consts->x8n_stride_gap, s);
        s = update16(tb.T, s, w);
        e = p + 16;
        any = true;
    }
    uint32_t c = any ? multmodp(x8n(P.consts->x2n, tile_end - e), s) : 0u;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) c ^= __shfl_xor_sync(0xFFFFFFFFu, c, o);
    if (lane == 0) warp_crc[warp] = c;
    __syncthreads();
    uint32_t t = 0;
    if (threadIdx.x == 0) {
        for (int i = 0; i < kWarps; ++i) t ^= warp_crc[i];
    }
    return t;
}

template <bool kPack>
__global__ void __launch_bounds__(kThreads) k_snapshot(const SnapParams P) {
    extern __shared__ __align__(16) uint8_t smem[];
    CrcTables &tb = *reinterpret_cast<CrcTables *>(smem);
    __shared__ uint32_t warp_crc[kWarps];
    __shared__ uint32_t warp_shift[kWarps];
    {
        const uint4 *g = reinterpret_cast<const uint4 *>(P.tables);
        uint4 *d = reinterpret_cast<uint4 *>(smem);
        for (int i = threadIdx.x; i < (int)(sizeof(CrcTables) / 16); i += kThreads) d[i] = g[i];
        if (threadIdx.x < kWarps) warp_shift[threadIdx.x] = P.consts->warp_shift[threadIdx.x];
    }
    __syncthreads();
    const uint32_t n_items = P.count * P.tpc;
    for (uint32_t item = blockIdx.x; item < n_items; item += gridDim.x) {
        const uint32_t jl = item / P.tpc, t = item - jl * P.tpc;
        const uint32_t j = P.first + jl;
        char *chunk = P.ring_base + ((P.ring_head + j) % P.ring_slots) * P.chunk_bytes;
        const uint32_t tile0 = t * kTile;
        const uint64_t rem = P.chunk_bytes - tile0;
        const uint32_t tile_len = rem < kTile ? (uint32_t)rem : kTile;
        const int rb = P.row_begin[j], re = P.row_begin[j + 1];
        uint32_t crc;
        if (tile_len == kTile)
            crc = tile_fast<kPack>(P, tb, chunk, warp_shift, warp_crc, rb, re, tile0);
        else
            crc = tile_generic<kPack>(P, tb, chunk, warp_crc, rb, re, tile0, tile_len);
        if (threadIdx.x == 0) P.tile_crc[(uint64_t)j * P.tpc + t] = crc;
        __syncthreads();  // warp_crc reuse
    }
}

// tiles -> chunk CRC (+ verify) -> slice digest.  One CTA per chunk.
__global__ void __launch_bounds__(256) k_finalize(const FinalizeParams F) {
    __shared__ uint32_t red[8];
    const uint32_t j = blockIdx.x;
    uint32_t v = 0;
    for (uint32_t t = threadIdx.x; t < F.tpc; t += blockDim.x)
        v ^= multmodp(F.tile_shift[t], F.tile_crc[(uint64_t)j * F.tpc + t]);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v ^= __shfl_xor_sync(0xFFFFFFFFu, v, o);
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = v;
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t raw = 0;
        for (int i = 0; i < (int)(blockDim.x >> 5); ++i) raw ^= red[i];
        const uint32_t crc = raw ^ F.ff[0] ^ 0xFFFFFFFFu;
        F.crc_out[j] = crc;
        if (F.expect) {
            const uint32_t badj = crc != F.expect[j];
            F.bad[j] = badj;
            if (badj) atomicAdd(&F.scratch[2], 1u);
        }
        atomicXor(&F.scratch[0], multmodp(F.chunk_shift[j], raw));
        __threadfence();
        if (atomicAdd(&F.scratch[1], 1u) == F.n - 1) {
            __threadfence();
            const uint32_t acc = atomicXor(&F.scratch[0], 0u);
            F.scratch[3] = acc ^ F.ff[1] ^ 0xFFFFFFFFu;
        }
    }
}

// ------------------------------------------------------------------------ host side
namespace {
struct TableCache {
    std::mutex mu;
    CrcTables *tables[64] = {};
    CrcConsts *consts[64] = {};
};
TableCache &cache() {
    static TableCache c;
    return c;
}
}  // namespace

cudaError_t device_tables(int device, const CrcTables **tables, const CrcConsts **consts) {
    TableCache &c = cache();
    std::lock_guard<std::mutex> lk(c.mu);
    if (device < 0 || device >= 64) return cudaErrorInvalidDevice;
    if (!c.tables[device]) {
        CrcTables *t = nullptr;
        CrcConsts *k = nullptr;
        cudaError_t e = cudaMalloc(&t, sizeof(CrcTables));
        if (e != cudaSuccess) return e;
        e = cudaMalloc(&k, sizeof(CrcConsts));
        if (e != cudaSuccess) return e;
        k_build_tables<<<1, 256>>>(t, k);
        e = cudaDeviceSynchronize();
        if (e != cudaSuccess) return e;
        c.tables[device] = t;
        c.consts[device] = k;
    }
    *tables = c.tables[device];
    *consts = c.consts[device];
    return cudaSuccess;
}

cudaError_t setup_geometry(DevGeometry *g, uint64_t chunk_bytes, uint32_t n, cudaStream_t s) {
    int dev = 0;
    cudaGetDevice(&dev);
    const CrcTables *tb;
    const CrcConsts *cs;
    cudaError_t e = device_tables(dev, &tb, &cs);
    if (e != cudaSuccess) return e;
    free_geometry(g);
    g->chunk_bytes = chunk_bytes;
    g->n = n;
    g->tpc = (uint32_t)((chunk_bytes + kTile - 1) / kTile);
    if ((e = cudaMalloc(&g->tile_shift, sizeof(uint32_t) * g->tpc)) != cudaSuccess) return e;
    if ((e = cudaMalloc(&g->chunk_shift, sizeof(uint32_t) * (n ? n : 1))) != cudaSuccess) return e;
    if ((e = cudaMalloc(&g->ff, sizeof(uint32_t) * 2)) != cudaSuccess) return e;
    const uint32_t m = g->tpc > n ? g->tpc : (n ? n : 1);
    k_setup_geometry<<<(m + 255) / 256, 256, 0, s>>>(g->tile_shift, g->chunk_shift, g->ff, cs, chunk_bytes, n, g->tpc);
    return cudaGetLastError();
}

void free_geometry(DevGeometry *g) {
    if (g->tile_shift) cudaFree(g->tile_shift);
    if (g->chunk_shift) cudaFree(g->chunk_shift);
    if (g->ff) cudaFree(g->ff);
    g->tile_shift = g->chunk_shift = g->ff = nullptr;
}

static int resident_ctas(int device) {
    static int cached[64] = {};
    if (device < 0 || device >= 64) return 1;
    if (!cached[device]) {
        int per_sm = 0, sms = 0;
        cudaFuncSetAttribute(k_snapshot<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, sizeof(CrcTables));
        cudaFuncSetAttribute(k_snapshot<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, sizeof(CrcTables));
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_snapshot<true>, kThreads, sizeof(CrcTables));
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
        cached[device] = (per_sm > 0 ? per_sm : 1) * (sms > 0 ? sms : 1);
    }
    return cached[device];
}

int snapshot_grid(int device, uint32_t n_items, uint32_t cap) {
    int g = resident_ctas(device);
    if (cap && (int)cap < g) g = (int)cap;
    if ((uint32_t)g > n_items) g = (int)n_items;
    return g < 1 ? 1 : g;
}

cudaError_t launch_pack(const SnapParams &p, int grid, cudaStream_t s) {
    if (p.count == 0) return cudaSuccess;
    k_snapshot<true><<<grid, kThreads, sizeof(CrcTables), s>>>(p);
    return cudaGetLastError();
}

cudaError_t launch_unpack(const SnapParams &p, int grid, cudaStream_t s) {
    if (p.count == 0) return cudaSuccess;
    k_snapshot<false><<<grid, kThreads, sizeof(CrcTables), s>>>(p);
    return cudaGetLastError();
}

cudaError_t launch_finalize(const FinalizeParams &p, cudaStream_t s) {
    if (p.n == 0) return cudaSuccess;
    k_finalize<<<p.n, 256, 0, s>>>(p);
    return cudaGetLastError();
}

}  // namespace pcc
