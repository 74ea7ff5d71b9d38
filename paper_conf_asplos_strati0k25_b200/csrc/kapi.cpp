// kapi.cpp — pccheck_kernels.h: K1 / K2 on caller buffers (no manager, no file).
#include <cuda_runtime.h>

#include <cstring>
#include <vector>

#include "../../include/pccheck_kernels.h"
#include "errors.hpp"
#include "kernels.hpp"
#include "layout.hpp"
#include "nccl_shim.hpp"

namespace pcc {
int cuda_error(cudaError_t e, const char *what);  // runtime.cpp
}

using namespace pcc;

namespace {

struct Scratch {
    SegRow *rows = nullptr;
    uint32_t *row_begin = nullptr, *tile_crc = nullptr, *scratch = nullptr, *crc_tmp = nullptr;
    uint2 *tile_rows = nullptr;
    DevGeometry geom;
    ~Scratch() {
        cudaFree(rows);
        cudaFree(row_begin);
        cudaFree(tile_crc);
        cudaFree(scratch);
        cudaFree(crc_tmp);
        cudaFree(tile_rows);
        free_geometry(&geom);
    }
};

int prepare(const pcc_tensor *t, uint32_t n, uint32_t align, uint64_t cb, uint64_t first, uint64_t count,
            cudaStream_t s, HostLayout *L, Scratch *S, SnapParams *P) {
    if ((n && !t) || count == 0) return count == 0 ? PCC_OK : set_error(PCC_EINVAL, "null tensor table");
    int rc = build_layout(t, n, align ? align : 256, cb, first, (int64_t)count, L);
    if (rc) return set_error(PCC_EINVAL, "bad geometry");
    if (first + count > L->C) return set_error(PCC_EINVAL, "chunk range beyond the image");
    build_tile_rows(L, cb, kTile);
    cudaError_t e;
    int dev = 0;
    cudaGetDevice(&dev);
    const CrcTables *tb;
    const CrcConsts *cs;
    if ((e = device_tables(dev, &tb, &cs)) != cudaSuccess) return cuda_error(e, "tables");
    if ((e = setup_geometry(&S->geom, cb, (uint32_t)count, s)) != cudaSuccess) return cuda_error(e, "geometry");
    const size_t nrows = L->rows.size() ? L->rows.size() : 1;
    if ((e = cudaMalloc(&S->rows, nrows * sizeof(SegRow))) != cudaSuccess) return cuda_error(e, "rows");
    if ((e = cudaMalloc(&S->row_begin, (count + 1) * sizeof(uint32_t))) != cudaSuccess) return cuda_error(e, "rb");
    if ((e = cudaMalloc(&S->tile_crc, count * tile_crc_words(S->geom.tpc) * sizeof(uint32_t))) != cudaSuccess)
        return cuda_error(e, "tile crc");
    if ((e = cudaMalloc(&S->tile_rows, L->tile_rows.size() * sizeof(uint32_t))) != cudaSuccess)
        return cuda_error(e, "tile rows");
    cudaMemcpyAsync(S->tile_rows, L->tile_rows.data(), L->tile_rows.size() * sizeof(uint32_t), cudaMemcpyHostToDevice,
                    s);
    if ((e = cudaMalloc(&S->scratch, 4 * sizeof(uint32_t))) != cudaSuccess) return cuda_error(e, "scratch");
    if (!L->rows.empty())
        cudaMemcpyAsync(S->rows, L->rows.data(), L->rows.size() * sizeof(SegRow), cudaMemcpyHostToDevice, s);
    cudaMemcpyAsync(S->row_begin, L->row_begin.data(), (count + 1) * sizeof(uint32_t), cudaMemcpyHostToDevice, s);
    cudaMemsetAsync(S->scratch, 0, 4 * sizeof(uint32_t), s);
    // host staging vectors must outlive the async copies
    if ((e = cudaStreamSynchronize(s)) != cudaSuccess) return cuda_error(e, "upload");
    P->rows = S->rows;
    P->row_begin = S->row_begin;
    P->tile_rows = S->tile_rows;
    P->chunk_bytes = cb;
    P->first = 0;
    P->count = (uint32_t)count;
    P->tpc = S->geom.tpc;
    P->ring_head = 0;
    P->ring_slots = count;
    P->tile_crc = S->tile_crc;
    P->tables = tb;
    P->consts = cs;
    return PCC_OK;
}

}  // namespace

extern "C" int pcc_k_layout(const pcc_tensor *t, uint32_t n, uint32_t align, uint64_t chunk_bytes, uint64_t *off,
                            uint64_t *end_bytes, uint64_t *n_chunks) {
    HostLayout L;
    int rc = build_layout(t, n, align ? align : 256, chunk_bytes, 0, 0, &L);
    if (rc) return rc;
    if (off) std::memcpy(off, L.off.data(), n * sizeof(uint64_t));
    if (end_bytes) *end_bytes = L.end;
    if (n_chunks) *n_chunks = L.C;
    return PCC_OK;
}

extern "C" int pcc_k_pack(const pcc_tensor *t, uint32_t n, uint32_t align, uint64_t chunk_bytes,
                          uint64_t first_chunk, uint64_t count, void *dst, uint32_t *crc, uint32_t *digest,
                          void *stream) {
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    HostLayout L;
    Scratch S;
    SnapParams P{};
    int rc = prepare(t, n, align, chunk_bytes, first_chunk, count, s, &L, &S, &P);
    if (rc || count == 0) return rc;
    P.ring_base = static_cast<char *>(dst);
    int dev = 0;
    cudaGetDevice(&dev);
    cudaError_t e = launch_pack(P, snapshot_grid(dev, (uint32_t)(count * P.tpc), 0, true), s);
    if (e != cudaSuccess) return cuda_error(e, "K1 launch");
    FinalizeParams F{};
    F.tile_crc = S.tile_crc;
    F.tables = P.tables;
    F.n = (uint32_t)count;
    F.tpc = P.tpc;
    F.tile_shift = S.geom.tile_shift;
    F.chunk_shift = S.geom.chunk_shift;
    F.ff = S.geom.ff;
    F.crc_out = crc;
    F.scratch = S.scratch;
    if ((e = launch_finalize(F, s)) != cudaSuccess) return cuda_error(e, "finalize launch");
    cudaMemcpyAsync(digest, S.scratch + 3, 4, cudaMemcpyDeviceToDevice, s);
    if ((e = cudaStreamSynchronize(s)) != cudaSuccess) return cuda_error(e, "K1");
    return PCC_OK;
}

extern "C" int pcc_k_unpack(const pcc_tensor *t, uint32_t n, uint32_t align, uint64_t chunk_bytes,
                            uint64_t first_chunk, uint64_t count, const void *src, const uint32_t *expect,
                            uint32_t *bad, uint32_t *n_bad, uint32_t *digest, void *stream) {
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    HostLayout L;
    Scratch S;
    SnapParams P{};
    int rc = prepare(t, n, align, chunk_bytes, first_chunk, count, s, &L, &S, &P);
    if (rc || count == 0) return rc;
    P.ring_base = const_cast<char *>(static_cast<const char *>(src));
    cudaError_t e;
    if ((e = cudaMalloc(&S.crc_tmp, count * sizeof(uint32_t))) != cudaSuccess) return cuda_error(e, "crc tmp");
    int dev = 0;
    cudaGetDevice(&dev);
    e = launch_unpack(P, snapshot_grid(dev, (uint32_t)(count * P.tpc), 0, false), s);
    if (e != cudaSuccess) return cuda_error(e, "K2 launch");
    FinalizeParams F{};
    F.tile_crc = S.tile_crc;
    F.tables = P.tables;
    F.n = (uint32_t)count;
    F.tpc = P.tpc;
    F.tile_shift = S.geom.tile_shift;
    F.chunk_shift = S.geom.chunk_shift;
    F.ff = S.geom.ff;
    F.crc_out = S.crc_tmp;
    F.expect = expect;
    F.bad = bad;
    F.scratch = S.scratch;
    if ((e = launch_finalize(F, s)) != cudaSuccess) return cuda_error(e, "finalize launch");
    cudaMemcpyAsync(n_bad, S.scratch + 2, 4, cudaMemcpyDeviceToDevice, s);
    cudaMemcpyAsync(digest, S.scratch + 3, 4, cudaMemcpyDeviceToDevice, s);
    if ((e = cudaStreamSynchronize(s)) != cudaSuccess) return cuda_error(e, "K2");
    return PCC_OK;
}

extern "C" int pcc_k_nccl_selftest(int device, const int64_t *vals, uint32_t n, int64_t *out_min, int64_t *out_max,
                                   uint32_t *gather_ok) {
    if (!vals || !out_min || !out_max || !gather_ok || n == 0 || n > 64) return set_error(PCC_EINVAL, "args");
    cudaError_t e = cudaSetDevice(device);
    if (e != cudaSuccess) return cuda_error(e, "set device");
    uint8_t uid[128];
    int rc = pcc_nccl_unique_id_impl(uid);
    if (rc) return rc;
    NcclComm comm;
    if ((rc = comm.init(uid, 1, 0))) return rc;
    int64_t *dev = nullptr, *pinned = nullptr;
    uint8_t *send = nullptr, *recv = nullptr;
    cudaStream_t s = nullptr;
    const size_t gb = 4096;
    std::vector<uint8_t> pat(gb), back(gb);
    for (size_t i = 0; i < gb; ++i) pat[i] = (uint8_t)(i * 131 + 7);
    if ((e = cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking)) || (e = cudaMalloc(&dev, 64 * sizeof(int64_t))) ||
        (e = cudaMallocHost(&pinned, 64 * sizeof(int64_t))) || (e = cudaMalloc(&send, gb)) || (e = cudaMalloc(&recv, gb)))
        rc = cuda_error(e, "selftest alloc");
    if (!rc) {
        std::memcpy(out_min, vals, n * sizeof(int64_t));
        rc = comm.allreduce_i64(out_min, n, NcclComm::kMin, dev, pinned, s);
    }
    if (!rc) {
        std::memcpy(out_max, vals, n * sizeof(int64_t));
        rc = comm.allreduce_i64(out_max, n, NcclComm::kMax, dev, pinned, s);
    }
    if (!rc) {
        cudaMemcpyAsync(send, pat.data(), gb, cudaMemcpyHostToDevice, s);
        cudaMemsetAsync(recv, 0, gb, s);
        rc = comm.allgather(send, recv, gb, s);
        if (!rc) {
            cudaMemcpyAsync(back.data(), recv, gb, cudaMemcpyDeviceToHost, s);
            if ((e = cudaStreamSynchronize(s))) rc = cuda_error(e, "selftest sync");
            *gather_ok = !rc && std::memcmp(back.data(), pat.data(), gb) == 0;
        }
    }
    comm.destroy();
    if (send) cudaFree(send);
    if (recv) cudaFree(recv);
    if (dev) cudaFree(dev);
    if (pinned) cudaFreeHost(pinned);
    if (s) cudaStreamDestroy(s);
    return rc;
}
