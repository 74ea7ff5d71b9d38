/*
 * pccheck.h — C ABI of the B200-native PCcheck snapshot path.
 *
 * PCcheck (Strati, Friedman, Klimovic, ASPLOS '25) checkpoints model and optimizer state
 * concurrently with training: up to N checkpoints in flight, each copied GPU -> DRAM in
 * chunks and persisted by several threads, with a crash-consistent pointer to the newest
 * complete checkpoint (§3.1, §4.1 Listing 1, §4.2).
 * This library is the GPU-side hot path of that method for one process per GPU:
 *
 *   pcc_register    the state tensors (model params, optimizer moments, step tensors)
 *   pcc_checkpoint  Listing 1 lines 3-13: counter, free slot, then the fused gather-pack +
 *                   CRC32C kernel (K1) packs the state into fixed-size chunks in HBM; copy
 *                   engines stream them to host DRAM; persist threads write them to the slot
 *   pcc_guard       the U-gate (L139): training's next update waits until K1 read the state
 *   pcc_poll/wait   per-checkpoint state machine
 *   pcc_commit      Listing 1 lines 16-34 + the distributed step of L283 (allreduce MIN)
 *   pcc_restore     L287: verify every chunk's CRC32C and scatter back (kernel K2)
 *
 * Every call returns int: PCC_OK (0) or a negative PCC_E* code; outputs go through
 * pointer arguments.  One pcc_ctx per process/GPU.  pcc_* calls on one ctx must come from
 * one host thread at a time; the library owns its internal threads.  No call takes or
 * returns torch types: device memory is a plain pointer, a stream is a cudaStream_t passed
 * as void* (NULL = the legacy default stream).
 *
 * Readings R1..R20 cited below are listed in DESIGN.md §3; the on-file format is FORMAT.md.
 */
#ifndef PCCHECK_H
#define PCCHECK_H

#include <stdint.h>

#if defined(__GNUC__)
#define PCC_API __attribute__((visibility("default")))
#else
#define PCC_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

#define PCC_ABI_VERSION 2u
#define PCC_LATEST UINT64_MAX   /* pcc_restore want_iter: newest globally committed */
#define PCC_NONE UINT64_MAX     /* "no checkpoint" iter sentinel */

/* ---- error codes (negated in return values) ---------------------------------------- */
enum {
    PCC_OK = 0,
    PCC_EINVAL = 1,    /* bad argument or config                                          */
    PCC_ENOMEM = 2,    /* host / device / pinned allocation failed                        */
    PCC_EBUSY = 3,     /* re-register while checkpoints are in flight                     */
    PCC_EAGAIN = 4,    /* non-blocking call could not proceed                             */
    PCC_EIO = 5,       /* file I/O error (errno kept, see pcc_last_errno)                 */
    PCC_ECUDA = 6,     /* CUDA runtime error (message via pcc_last_error)                 */
    PCC_ENCCL = 7,     /* NCCL error                                                      */
    PCC_EORDER = 8,    /* checkpoint iter not strictly increasing (R5)                    */
    PCC_ECORRUPT = 9,  /* restore: a chunk / header CRC mismatch (R13)                    */
    PCC_ELAYOUT = 10,  /* restore: registration differs from the checkpoint's layout      */
    PCC_ENOENT = 11,   /* no valid checkpoint                                             */
    PCC_ETIMEDOUT = 12,
    PCC_ESTATE = 13,   /* call not valid in the current state (e.g. not registered)       */
};

/* ---- config flags -------------------------------------------------------------------- */
enum {
    PCC_ODIRECT = 1u << 0,  /* open the file O_DIRECT (falls back to buffered on EINVAL)     */
    PCC_FSYNC = 1u << 1,    /* fdatasync data before the COMPLETE header, fsync header/pointer */
    PCC_ZEROCOPY = 1u << 2, /* Variant A: K1 stores straight into host-mapped memory (no CE)  */
    PCC_NULLSINK = 1u << 3, /* benchmark: no file; chunks land in pinned staging and are dropped */
    PCC_MAPFILE = 1u << 4,  /* the file's slots are mmap'd + cudaHostRegister'ed: the copy
                               engine (or K1 with ZEROCOPY) writes straight into the file's
                               pages (DRAM-backed file, e.g. tmpfs); persist = fdatasync only */
    PCC_NOCOMM = 1u << 5,   /* world > 1 without NCCL: this process alone plays rank `rank` of
                               `world` (packs, persists and commits only its 1/world slice; the
                               global commit reduces over itself).  For measuring one rank's
                               share on one GPU; a restore then covers only this slice. */
    PCC_SHARDED = 1u << 6,  /* FSDP / ZeRO state (L152 §3.1: "each worker has its own model
                               shard"): every rank registers its OWN tensors and checkpoints all
                               of them — no 1/world slicing, no restore fan-out; the global commit
                               and the restore agreement still run across ranks. */
    PCC_D2H_UPFRONT = 1u << 7, /* the copy-engine D2H of each K1 window is enqueued by the thread
                               that launches the window, at once (no pacing, no queue drains), so the
                               transfer needs no later CUDA call from the library's threads.  For
                               training loops run as CUDA graphs: a host thread blocked in
                               cudaGraphLaunch (GPU queue full) stalls every other thread's CUDA calls
                               for up to one replay.  Eager loops that read values to
                               the host every step want the default (drained, optionally paced). */
};

/* ---- per-checkpoint states (pcc_poll) — SURVEY §8(b) state machine ------------------- */
enum {
    PCC_ST_QUEUED = 0,        /* counter taken, slot dequeued (Listing 1 lines 5-11)          */
    PCC_ST_PACKING = 1,       /* K1 issued; the U-gate is closed until it finished             */
    PCC_ST_PACKED = 2,        /* all chunks out of the registered tensors                      */
    PCC_ST_PERSISTED = 3,     /* every chunk written to its slot                               */
    PCC_ST_LOCAL_COMMIT = 4,  /* header COMPLETE + pointer record name it (lines 16-25)        */
    PCC_ST_GLOBAL_COMMIT = 5, /* every rank holds it (peer_check, L283); W=1: == LOCAL_COMMIT  */
    PCC_ST_OBSOLETE = 6,      /* lost the CAS to a newer counter (lines 29-31), slot recycled  */
    PCC_ST_FAILED = 7,        /* I/O / CUDA / NCCL error; pointer untouched                    */
};

/* dtype codes hashed into the layout CRC (R1: bytes are copied verbatim, no conversion) */
enum { PCC_U8 = 0, PCC_F32 = 1, PCC_BF16 = 2, PCC_F16 = 3, PCC_F64 = 4, PCC_I64 = 5, PCC_I32 = 6 };

typedef struct pcc_ctx pcc_ctx;
typedef uint64_t pcc_handle;

/* Caller-supplied collectives (optional, world > 1): when set they replace the library's NCCL
 * communicator — e.g. a framework that owns its transport, or gloo on CPU.  Both are COLLECTIVE
 * and called from the thread that called the pcc_* function, in the same order on every rank.
 *   allreduce: values[count] in place, MAX if is_max else MIN, across all ranks
 *   allgather: recv[rank * bytes + i] = send_of_rank[i], HOST buffers
 * Return 0 on success. */
typedef int (*pcc_allreduce_i64_fn)(void *ctx, int64_t *values, uint32_t count, int is_max);
typedef int (*pcc_allgather_fn)(void *ctx, const void *send, void *recv, uint64_t bytes_per_rank);

/* Table 2 (L205-L213) configuration parameters, plus placement. */
typedef struct {
    uint32_t abi_version;      /* PCC_ABI_VERSION                                                  */
    const char *path;          /* this rank's checkpoint file (created; (N+1) slots, FORMAT.md)    */
    uint64_t chunk_bytes;      /* b, the chunk = DRAM buffer = CRC unit (R2). Multiple of 16;
                                  of 4096 with PCC_ODIRECT or PCC_MAPFILE                          */
    uint32_t max_inflight;     /* N >= 1; the file holds N+1 slots (L158, L229)                   */
    uint64_t staging_bytes;    /* M: pinned DRAM pool, c = M / chunk_bytes slots (L176); ignored
                                  with PCC_MAPFILE (the file pages are the staging)               */
    uint64_t ring_bytes;       /* HBM chunk ring for Variant B; 0 = one whole slice (the "extra
                                  copy of the weights" of L139, affordable in 180 GB)             */
    uint32_t writer_threads;   /* p persist threads (L176: 2-4); 0 = 4                              */
    uint32_t flags;            /* PCC_* flags above                                               */
    int32_t device;            /* CUDA device ordinal                                              */
    int32_t rank, world;       /* data-parallel rank / world size (R8, R9)                        */
    const void *nccl_unique_id;/* 128-byte ncclUniqueId from pcc_nccl_unique_id on rank 0,
                                  broadcast by the caller; required when world > 1                 */
    uint32_t align;            /* image alignment of each tensor (R1); 0 = 256                    */
    uint32_t pack_ctas;        /* grid cap for K1 (0 = all SMs); small caps leave SMs to training */
    pcc_allreduce_i64_fn allreduce; /* optional caller collectives (see above); both or neither */
    pcc_allgather_fn allgather;
    void *coll_ctx;
    /* D2H pacing of the copy-engine transfer (Variant B).  A saturating D2H burst slows an
       eager training loop by ~10% while it lasts (measured: 1.9 ms per 1.1 GB on VGG-16): the
       link's posted writes delay the GPU front-end's command fetches.  Copies of at most
       d2h_quantum bytes issued no faster than d2h_mbps once the chunks are in the HBM ring cut
       that to ~0.2 ms.  0 / 0 = one copy per chunk group at full link rate. */
    uint32_t d2h_mbps;         /* pace in MB/s (10^6 B/s); 0 = unpaced                           */
    uint32_t d2h_quantum;      /* bytes per copy-engine copy; 0 = whole chunk groups (<= 64 MiB) */
} pcc_config;

typedef struct {
    const void *dev_ptr;       /* device address of the tensor's first byte (any alignment)       */
    uint64_t nbytes;           /* bytes, contiguous from dev_ptr                                   */
    uint32_t dtype;            /* PCC_F32 ... (only hashed into the layout CRC)                    */
    const char *name;          /* optional, may be NULL                                            */
} pcc_tensor;

typedef struct {
    uint64_t iter, counter;
    uint32_t slot, state;
    uint32_t digest;           /* CRC32C of this rank's slice (R4)                                 */
    uint32_t n_chunks;         /* chunks in this rank's slice                                      */
    double t_call_us;          /* host steady-clock stamps relative to pcc_open, microseconds:     */
    double t_packed_us;        /*   K1 + finalize done (event observed)                             */
    double t_landed_us;        /*   last chunk landed in host memory                                */
    double t_persisted_us;     /*   last chunk persisted                                            */
    double t_committed_us;     /*   local commit                                                    */
    float pack_ms;             /* CUDA-event span of K1: first launch start -> last launch end      */
                               /*   (the U-gate span; includes waits for ring space between launches) */
    float finalize_ms;         /* CUDA-event time of the CRC finalize kernels                      */
    float k1_busy_ms;          /* sum of the K1 launches' own CUDA-event durations                 */
    float snapshot_ms;         /* CUDA-event time from K1's start to the last chunk's D2H end      */
} pcc_ckpt_info;

/* Opens (creates) the checkpoint file, allocates staging / HBM ring, starts the persist
 * threads and (world > 1) the NCCL communicator.  On error *out is NULL. */
PCC_API int pcc_open(const pcc_config *cfg, pcc_ctx **out);

/* Registers the state tensors in checkpoint order (R11).  Builds the layout (R1: tensor i
 * at align_up(end of i-1, align)), the segment table and this rank's slice
 * [floor(rC/W), floor((r+1)C/W)) and uploads them to the device.  The table t[] is copied;
 * the device memory stays owned by the caller and must stay alive and unmoved until close
 * or the next register.  -PCC_EBUSY while checkpoints are in flight.  n may be 0. */
PCC_API int pcc_register(pcc_ctx *ctx, const pcc_tensor *t, uint32_t n);

/* Starts checkpoint `iter` of the registered state as it is on `train_stream` now.
 * Listing 1 lines 3-11 (sample the pointer, take the counter, dequeue a free slot — this
 * BLOCKS while N checkpoints hold all N+1 slots, the paper's stall, L139 Fig 6), records an
 * event on train_stream, and enqueues K1 on the library's pack stream behind that event when
 * the HBM ring has room for the slice; otherwise hands the checkpoint to the library's packer
 * thread, which launches K1 in windows as ring space frees.  It never waits for ring space or
 * for an earlier checkpoint's transfer.  iter must strictly increase (-PCC_EORDER).  *out
 * receives the handle.  World > 1: COLLECTIVE when a rank has no free slot (backpressure). */
PCC_API int pcc_checkpoint(pcc_ctx *ctx, uint64_t iter, void *train_stream, pcc_handle *out);

/* U-gate (L139): makes train_stream wait (cudaStreamWaitEvent) until the newest checkpoint's
 * K1 finished reading the registered tensors.  Call before the optimizer step that overwrites
 * them.  Returns at once when that checkpoint's K1 windows are enqueued; when the packer thread
 * still holds some (ring space), it first waits on the host until they are — the training
 * stream is only ever made to wait for work already on the GPU (a stream-side wait for work
 * another thread enqueues later deadlocks under lazy module loading and pageable copies,
 * profiles/r02_gate_probe_*.txt).  No-op before any checkpoint. */
PCC_API int pcc_guard(pcc_ctx *ctx, void *train_stream);

/* Handles stay valid until pcc_close: pcc_poll / pcc_wait answer for every handle ever returned
 * (the outcome of an old terminal checkpoint is kept in 16 bytes); pcc_info keeps the full record
 * of the newest 64 terminal checkpoints and returns -PCC_EINVAL ("record pruned") for older ones. */
PCC_API int pcc_poll(pcc_ctx *ctx, pcc_handle h, int *state);

/* Blocks until the checkpoint reached LOCAL_COMMIT (or OBSOLETE / FAILED); timeout_us < 0 =
 * forever.  Returns PCC_OK, -PCC_ETIMEDOUT, or the checkpoint's error. */
PCC_API int pcc_wait(pcc_ctx *ctx, pcc_handle h, int64_t timeout_us);

/* Blocks until every issued checkpoint is terminal. */
PCC_API int pcc_drain(pcc_ctx *ctx, int64_t timeout_us);

/* Distributed commit (L283; R8, R9, R20).  world == 1: returns the newest local commit.
 * world > 1: COLLECTIVE — every rank calls it at the same program point; g =
 * allreduce_MIN(latest locally committed iter) over NCCL, written to the pointer record as
 * global_iter, and slots holding iters < g are freed.  *committed_iter = g (PCC_NONE if none). */
PCC_API int pcc_commit(pcc_ctx *ctx, uint64_t *committed_iter);

/* Read-only query of a rank file's pointer records (valid record with the largest seq). */
PCC_API int pcc_latest(const char *path, uint64_t *global_iter, uint64_t *local_iter);

/* Restores the registered tensors from the file (L287).  want_iter = PCC_LATEST: the newest
 * globally consistent iter (world > 1: agreed with allreduce MAX/MIN); else
 * exactly want_iter.  Every chunk is verified against the slot header's CRC32C table by K2
 * while it scatters; world > 1 ranks exchange their verified slices with ncclAllGather.
 * flags & PCC_FALLBACK: on a rejected candidate retry the newest older iter every rank holds
 * (R10).  On -PCC_ECORRUPT the tensors are unspecified; bad_chunks receives up to bad_cap
 * global chunk indices that failed, *n_bad their count.  COLLECTIVE when world > 1. */
#define PCC_FALLBACK 1u
PCC_API int pcc_restore(pcc_ctx *ctx, uint64_t want_iter, uint32_t flags, uint64_t *restored_iter,
                uint32_t *bad_chunks, uint32_t bad_cap, uint32_t *n_bad);

/* Where the last pcc_restore's time went (storage read, H2D, K2, allgather), this
 * rank.  Times are summed over every candidate checkpoint the restore tried (fallback). */
typedef struct {
    uint64_t bytes;            /* slice bytes read + verified from this rank's file             */
    uint32_t attempts;         /* candidate checkpoints verified (1 + fallbacks)                 */
    float total_ms;            /* pcc_restore call -> return (host clock)                        */
    float read_ms;             /* storage read: pread into pinned staging (host clock); 0 with
                                  PCC_MAPFILE, where the copy engine reads the mapped file pages */
    float h2d_ms;              /* first H2D start -> last H2D end (CUDA events, copy stream)     */
    float k2_ms;               /* the K2 launches over this rank's slice, summed (CUDA events)   */
    float finalize_ms;         /* chunk CRCs + digest compare (CUDA events)                       */
    float fanout_ms;           /* world > 1: allgather of the other ranks' chunks + their K2
                                  (host clock); 0 at world 1                                      */
} pcc_restore_info;
PCC_API int pcc_restore_stats(pcc_ctx *ctx, pcc_restore_info *out);

/* Diagnostics of one checkpoint (timings, digest) and its chunk CRC table (crc_cap entries). */
PCC_API int pcc_info(pcc_ctx *ctx, pcc_handle h, pcc_ckpt_info *info, uint32_t *crc, uint32_t crc_cap);

/* Geometry of the current registration: chunks total, slice first/count, image end bytes. */
PCC_API int pcc_geometry(pcc_ctx *ctx, uint64_t *n_chunks, uint64_t *first, uint64_t *count, uint64_t *end_bytes);

/* Number of kernels this ctx has launched so far (bench: gpu_launches). */
PCC_API uint64_t pcc_kernel_launches(pcc_ctx *ctx);

/* Drains in-flight checkpoints, joins threads, frees everything. */
PCC_API int pcc_close(pcc_ctx *ctx);

/* 128-byte NCCL unique id for world > 1 (rank 0 creates; the caller broadcasts it). */
PCC_API int pcc_nccl_unique_id(void *out128);

/* sizeof(pcc_config) (which = 0), sizeof(pcc_tensor) (1), sizeof(pcc_ckpt_info) (2), else 0:
 * lets a binding check its struct mirrors against this build. */
PCC_API uint64_t pcc_struct_size(int which);
PCC_API const char *pcc_strerror(int err);
PCC_API const char *pcc_last_error(void);   /* thread-local detail of the last failure */
PCC_API int pcc_last_errno(void);

#ifdef __cplusplus
}
#endif
#endif
