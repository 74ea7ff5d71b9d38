/*
 * pccheck_kernels.h — kernel-level entry points of the snapshot path (K1, K2) without the
 * checkpoint manager, for parity tests and microbenchmarks.  Same conventions as
 * pccheck.h (0 / -PCC_E* returns, void* streams, plain device pointers).
 *
 * The image is the one of reading R1: tensors t[0..n) in order, tensor i at
 * align_up(end of i-1, align), zero-filled, cut into chunk_bytes chunks (PAPER.md L127,
 * L281 "contiguous"; L176 chunks of size b).  CRC32C per chunk: BASELINE.json north_star.
 */
#ifndef PCCHECK_KERNELS_H
#define PCCHECK_KERNELS_H

#include <stdint.h>
#include "pccheck.h"

#ifdef __cplusplus
extern "C" {
#endif

/* K1: packs image chunks [first_chunk, first_chunk + count) into dst (count*chunk_bytes
 * bytes at any address the GPU can store to: device memory or host-mapped pinned memory;
 * 16-B aligned), writes the standard CRC32C of each chunk to crc[count] and the CRC32C of
 * the whole packed range to *digest (both DEVICE pointers).  Source tensors may have any
 * alignment.  Stream-ordered on `stream`; the call synchronizes the stream before returning
 * (it frees its scratch).  chunk_bytes % 16 == 0, < 4 GiB; align % 16 == 0. */
PCC_API int pcc_k_pack(const pcc_tensor *t, uint32_t n, uint32_t align, uint64_t chunk_bytes, uint64_t first_chunk,
               uint64_t count, void *dst, uint32_t *crc, uint32_t *digest, void *stream);

/* K2: verifies and scatters.  src holds image chunks [first_chunk, first_chunk+count)
 * (device or host-mapped); every chunk's CRC32C is recomputed and compared with
 * expect[count] (DEVICE pointer); bad[count] (DEVICE) receives 1 for a mismatching chunk,
 * *n_bad (DEVICE) the number of mismatches, *digest (DEVICE) the recomputed range digest.
 * The bytes of every tensor piece inside the range are written to t[i].dev_ptr (the
 * tensors are the destinations), regardless of the verdict (single pass). */
PCC_API int pcc_k_unpack(const pcc_tensor *t, uint32_t n, uint32_t align, uint64_t chunk_bytes, uint64_t first_chunk,
                 uint64_t count, const void *src, const uint32_t *expect, uint32_t *bad, uint32_t *n_bad,
                 uint32_t *digest, void *stream);

/* Transport self-test of the commit collective (C1 of SURVEY §2.3; §4.1, reading
 * R9): a one-rank NCCL communicator on `device` runs the calls the commit and restore paths
 * issue over the library's own communicator — ncclAllReduce of int64 with MIN and with MAX on
 * vals[n] (HOST arrays; out_min / out_max receive the reduced vectors, equal to vals with one
 * rank) and ncclAllGather of bytes (*gather_ok = 1 when the gathered bytes equal the sent
 * ones).  For tests: one GPU cannot host two NCCL ranks.  -PCC_ENCCL when libnccl.so.2 cannot
 * be loaded or a call fails, -PCC_ECUDA on a CUDA error. */
PCC_API int pcc_k_nccl_selftest(int device, const int64_t *vals, uint32_t n, int64_t *out_min, int64_t *out_max,
                                uint32_t *gather_ok);

/* Layout queries (host only, no GPU needed): image offsets of the n tensors and the chunk
 * count C for this registration. */
PCC_API int pcc_k_layout(const pcc_tensor *t, uint32_t n, uint32_t align, uint64_t chunk_bytes, uint64_t *off,
                 uint64_t *end_bytes, uint64_t *n_chunks);

#ifdef __cplusplus
}
#endif
#endif
