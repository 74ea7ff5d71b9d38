// kernels.hpp — host-side interface of the snapshot kernels (internal to the library).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "crc32c.cuh"

namespace pcc {

// One row of the segment table: the piece of one tensor that falls into one chunk
// (SURVEY §8(a) row a0).  ptr = address of the piece's first byte (source when packing,
// destination when restoring); dst_off = its offset inside the chunk; len = bytes.
struct SegRow {
    uint64_t ptr;
    uint32_t dst_off;
    uint32_t len;
};
static_assert(sizeof(SegRow) == 16, "SegRow");

// Device-resident per-registration constants (built by setup_geometry).
struct DevGeometry {
    uint64_t chunk_bytes = 0;
    uint32_t n = 0;              // chunks in this rank's slice
    uint32_t tpc = 0;            // tiles per chunk = ceil(chunk_bytes / kTile), a tile = one warp's 8 KiB
    uint32_t *tile_shift = nullptr;   // [tpc] x8n(CB - end of tile t)
    uint32_t *chunk_shift = nullptr;  // [n]    x8n((n-1-j) * CB)
    uint32_t *ff = nullptr;           // [2]    shift(~0, CB), shift(~0, n*CB)
};

// One launch of K1 / K2 over slice chunks [first, first+count).  Chunk j's packed bytes
// live at ring_base + ((ring_head + j) % ring_slots) * chunk_bytes (HBM ring, pinned
// host-mapped staging or the registered file mapping — any address the SMs can store to).
struct SnapParams {
    const SegRow *rows;
    const uint32_t *row_begin;   // [n+1] rows of slice chunk j: [row_begin[j], row_begin[j+1])
    const uint2 *tile_rows;      // [n*tpc] rows overlapping tile (j, t): x = first row index, y = count
    uint64_t chunk_bytes;
    uint32_t first, count, tpc;
    char *ring_base;
    uint64_t ring_head, ring_slots;
    uint32_t *tile_crc;          // [n * tpc * kLaneOut] raw lane CRCs (relative to each lane's last span end)
    const CrcTables *tables;
    const CrcConsts *consts;
};

struct FinalizeParams {
    uint32_t *tile_crc;          // K1/K2's lane CRCs, tile_crc_words(tpc) per chunk (overwritten)
    const CrcTables *tables;     // NL (lane -> sub-tile end shifts)
    uint32_t n, tpc;             // tiles per chunk
    const uint32_t *tile_shift, *chunk_shift, *ff;
    uint32_t *crc_out;           // [n] standard CRC32C per chunk
    const uint32_t *expect;      // restore: [n] expected CRCs (nullptr when packing)
    uint32_t *bad;               // restore: [n] 1 = mismatch
    uint32_t *scratch;           // [4] zeroed: unused, unused, n_bad, digest out
};

// words of K1/K2 lane-CRC output per chunk
inline uint64_t tile_crc_words(uint32_t tpc) { return (uint64_t)tpc * kLaneOut; }

// Builds the CRC tables once per device (device memory owned by a process-wide cache).
cudaError_t device_tables(int device, const CrcTables **tables, const CrcConsts **consts);
cudaError_t setup_geometry(DevGeometry *g, uint64_t chunk_bytes, uint32_t n, cudaStream_t s);
void free_geometry(DevGeometry *g);

int snapshot_grid(int device, uint32_t n_items, uint32_t cap, bool pack);  // CTAs for K1 (pack) / K2
cudaError_t launch_pack(const SnapParams &p, int grid, cudaStream_t s);
cudaError_t launch_unpack(const SnapParams &p, int grid, cudaStream_t s);
cudaError_t launch_finalize(const FinalizeParams &p, cudaStream_t s);  // kFinalizeLaunches kernels
constexpr int kFinalizeLaunches = 2;
// One no-work launch of each pipeline kernel (+ its launch attributes) so that lazy module
// loading happens at open time, not inside a checkpoint.  Synchronous.
cudaError_t warm_kernels(int device, const CrcTables *tables);

}  // namespace pcc
