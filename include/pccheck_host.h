/*
 * pccheck_host.h — the commit engine alone (no GPU): Listing 1's counter / free-slot
 * queue / CAS on CHECK_ADDR and the data-parallel commit rule, over the same rank file the
 * full library writes (FORMAT.md).  This is the metadata subsystem the runtime drives from
 * its persist threads; it is exposed so that host logic can
 * be tested on CPU (tests under gloo drive one engine per rank and do the MIN themselves).
 * It moves no checkpoint data: the caller writes chunk bytes into the slot's data region
 * (pcc_host_data_offset) before calling pcc_host_complete.
 */
#ifndef PCCHECK_HOST_H
#define PCCHECK_HOST_H

#include <stdint.h>
#include "pccheck.h"

#ifdef __cplusplus
extern "C" {
#endif

typedef struct pcc_host pcc_host;

typedef struct {
    const char *path;          /* rank file; NULL = no file (in-memory commit)               */
    uint64_t chunk_bytes;
    uint32_t max_inflight;     /* N (N+1 slots)                                               */
    uint32_t rank, world;
    uint32_t total_chunks;     /* C of the whole image; this rank owns its slice (R1, §8(e))   */
    uint32_t n_tensors, align, layout_crc;
    uint32_t fsync;            /* 1: fdatasync / fsync as in FORMAT.md's commit order          */
} pcc_host_config;

PCC_API int pcc_host_open(const pcc_host_config *cfg, pcc_host **out);
/* Listing 1 lines 3-11.  -PCC_EAGAIN when no slot is free (the caller must wait / commit). */
PCC_API int pcc_host_begin(pcc_host *h, uint64_t iter, uint64_t *counter, uint32_t *slot);
/* R18: header FILLING (+fdatasync) before the slot's data is overwritten. */
PCC_API int pcc_host_filling(pcc_host *h, uint64_t counter);
/* Lines 16-34 once the caller wrote the slot's chunks: header COMPLETE with crc[n] / digest,
 * CAS (W = 1) or in-order local commit (W > 1).  *state = PCC_ST_* of THIS checkpoint. */
PCC_API int pcc_host_complete(pcc_host *h, uint64_t counter, const uint32_t *crc, uint32_t digest, int *state);
PCC_API int pcc_host_fail(pcc_host *h, uint64_t counter);
/* State of any checkpoint begun on this engine (W > 1: LOCAL_COMMIT arrives in order). */
PCC_API int pcc_host_state(pcc_host *h, uint64_t counter, int *state);
PCC_API uint64_t pcc_host_local_latest(pcc_host *h);   /* L_r, PCC_NONE if none             */
PCC_API uint64_t pcc_host_global(pcc_host *h);         /* g as last applied                  */
PCC_API int pcc_host_apply_global(pcc_host *h, uint64_t g);  /* W > 1: free slots below g    */
PCC_API uint32_t pcc_host_free_slots(pcc_host *h);
/* slice geometry: first chunk, chunk count n, byte offset of slot s's data region */
PCC_API int pcc_host_geometry(pcc_host *h, uint32_t *first, uint32_t *n, uint32_t *n_slots);
PCC_API uint64_t pcc_host_data_offset(pcc_host *h, uint32_t slot);
/* held (committed, not freed) iters: writes up to cap (iter, slot) pairs, returns count */
PCC_API uint32_t pcc_host_held(pcc_host *h, uint64_t *iters, uint32_t *slots, uint32_t cap);

/* The restore agreement of pcc_restore (R8, R10) over this engine's rank file,
 * with the collectives and the slice verification supplied by the caller: `reduce` performs an
 * in-place allreduce of one int64 across ranks (is_max: MAX else MIN; identity for W = 1),
 * `verify` checks this rank's slice of `iter` in `slot` (0 = intact).  COLLECTIVE: every rank
 * calls it with the same want_iter / flags.  Returns 0 and *restored_iter, or -PCC_E*. */
typedef int (*pcc_reduce_fn)(void *ctx, int64_t *value, int is_max);
typedef int (*pcc_verify_fn)(void *ctx, uint64_t iter, uint32_t slot);
PCC_API int pcc_host_restore_plan(pcc_host *h, uint64_t want_iter, uint32_t flags, pcc_reduce_fn reduce,
                                  pcc_verify_fn verify, void *ctx, uint64_t *restored_iter);
PCC_API int pcc_host_close(pcc_host *h);

#ifdef __cplusplus
}
#endif
#endif
