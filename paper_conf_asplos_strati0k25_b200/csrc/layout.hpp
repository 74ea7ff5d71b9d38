// layout.hpp — registration -> image layout -> segment table.
//
// Reading R1 (PAPER.md L127/L281 only say the checkpoint is "contiguous"
// on storage): tensors are laid out in registration order, tensor i at
// off_i = align_up(off_{i-1} + nbytes_{i-1}, align), C = ceil(end / chunk_bytes) chunks,
// every byte not covered by a tensor is zero.  Rank r of W owns chunks
// [floor(rC/W), floor((r+1)C/W)).  The segment table lists, for every chunk
// of the slice, the pieces of tensors that land in it; K1 gathers them, K2 scatters them.
#pragma once
#include <cstdint>
#include <algorithm>
#include <vector>

#include "../../include/pccheck.h"
#include "kernels.hpp"

namespace pcc {

struct HostLayout {
    std::vector<uint64_t> off;      // image offset of each tensor
    uint64_t end = 0, C = 0;        // image end (bytes), total chunks
    uint64_t first = 0, n = 0;      // chunk range the rows describe
    std::vector<SegRow> rows;       // sorted by (chunk, dst_off)
    std::vector<uint32_t> row_begin;  // [n+1]
    std::vector<uint32_t> tile_rows;  // [2*n*tpc] (first row, count) of the rows overlapping each K1 tile
};

// Rows overlapping each tile [t*tile, (t+1)*tile) of each chunk (K1 stages them in shared memory).
inline void build_tile_rows(HostLayout *L, uint64_t cb, uint32_t tile) {
    const uint64_t tpc = (cb + tile - 1) / tile;
    L->tile_rows.assign(2 * L->n * tpc, 0);
    for (uint64_t j = 0; j < L->n; ++j) {
        uint32_t r = L->row_begin[j];
        const uint32_t re = L->row_begin[j + 1];
        for (uint64_t t = 0; t < tpc; ++t) {
            const uint64_t t0 = t * tile, t1 = std::min<uint64_t>(t0 + tile, cb);
            while (r < re && (uint64_t)L->rows[r].dst_off + L->rows[r].len <= t0) ++r;
            uint32_t e = r;
            while (e < re && L->rows[e].dst_off < t1) ++e;
            L->tile_rows[2 * (j * tpc + t)] = r;
            L->tile_rows[2 * (j * tpc + t) + 1] = e - r;
        }
    }
}

inline uint64_t align_up(uint64_t x, uint64_t a) { return (x + a - 1) / a * a; }

inline void slice_of(uint64_t C, uint32_t rank, uint32_t world, uint64_t *first, uint64_t *n) {
    const uint64_t a = C * rank / world, b = C * (rank + 1) / world;
    *first = a;
    *n = b - a;
}

// Rows for chunks [first, first + n) of the image.  Returns -PCC_EINVAL on bad geometry.
inline int build_layout(const pcc_tensor *t, uint32_t nt, uint32_t align, uint64_t cb, uint64_t first, int64_t n_or_all,
                        HostLayout *L) {
    if (align == 0 || cb == 0 || cb % 16 || align % 16 || cb >= (1ull << 32)) return -PCC_EINVAL;
    L->off.assign(nt, 0);
    uint64_t end = 0;
    for (uint32_t i = 0; i < nt; ++i) {
        const uint64_t o = i == 0 ? 0 : align_up(end, align);
        L->off[i] = o;
        end = o + t[i].nbytes;
    }
    L->end = end;
    L->C = (end + cb - 1) / cb;
    L->first = first;
    L->n = n_or_all < 0 ? (L->C > first ? L->C - first : 0) : (uint64_t)n_or_all;
    if (first + L->n > L->C && L->n) return -PCC_EINVAL;
    L->rows.clear();
    L->row_begin.assign(L->n + 1, 0);
    const uint64_t lo = first * cb, hi = (first + L->n) * cb;
    std::vector<uint32_t> count(L->n, 0);
    for (uint32_t i = 0; i < nt; ++i) {
        const uint64_t a = L->off[i], b = a + t[i].nbytes;
        if (t[i].nbytes == 0 || b <= lo || a >= hi) continue;
        for (uint64_t p = a > lo ? a : lo; p < b && p < hi;) {
            const uint64_t c = p / cb;
            const uint64_t ce = (c + 1) * cb;
            const uint64_t q = b < ce ? b : ce;
            SegRow r;
            r.ptr = reinterpret_cast<uint64_t>(t[i].dev_ptr) + (p - a);
            r.dst_off = (uint32_t)(p - c * cb);
            r.len = (uint32_t)(q - p);
            L->rows.push_back(r);
            ++count[c - first];
            p = q;
        }
    }
    // tensors are in image order, so rows already come sorted by chunk then dst_off
    for (uint64_t j = 0; j < L->n; ++j) L->row_begin[j + 1] = L->row_begin[j] + count[j];
    return PCC_OK;
}

}  // namespace pcc
