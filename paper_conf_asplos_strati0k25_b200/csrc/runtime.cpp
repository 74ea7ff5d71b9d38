// runtime.cpp — the PCcheck manager on one B200 (pccheck.h).
//
// PAPER.md Fig 5 (L117) / §3.1 L125-L141 on B200, one process per GPU:
//   training thread   pcc_checkpoint: Listing 1 lines 3-11 (CommitEngine::begin), then K1
//                     on the pack stream: the registered tensors -> the HBM chunk ring with
//                     CRC32C (the "extra copy of the weights" of L139, affordable in 180 GB,
//                     so the U-gate only waits for an HBM->HBM pack, not for PCIe)
//   orchestrator      one thread: FILLING header, then per chunk a copy-engine D2H from the
//                     ring into host DRAM (L164: copy engines, pinned memory) — straight into
//                     the registered file mapping (PCC_MAPFILE) or a pinned staging slot
//   persist pool      p threads (L168, L176): wait for the chunk's copy, pwrite it to the
//                     slot (PWRITE mode), recycle ring / staging; the last chunk runs
//                     Listing 1 lines 16-34 (CommitEngine::complete)
// Chunks of a checkpoint land contiguously in their slot (L127, L281: "contiguous on
// storage"), N checkpoints may be in flight (L139, Fig 6), copy and persist overlap per
// chunk (L141, Fig 7).
#include <cuda_runtime.h>
#include <fcntl.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <unistd.h>

#include <algorithm>
#include <atomic>
#include <cerrno>
#include <chrono>
#include <condition_variable>
#include <cstdlib>
#include <cstring>
#include <deque>
#include <map>
#include <unordered_map>
#include <memory>
#include <mutex>
#include <set>
#include <string>
#include <thread>
#include <vector>

#include "../../include/pccheck.h"
#include "commit.hpp"
#include "errors.hpp"
#include "fault.hpp"
#include "kernels.hpp"
#include "layout.hpp"
#include "nccl_shim.hpp"
#include "nvtx3/nvToolsExt.h"

namespace pcc {

int cuda_error(cudaError_t e, const char *what) {
    char b[512];
    std::snprintf(b, sizeof b, "%s: %s", what, cudaGetErrorString(e));
    err_state().msg = b;
    return -PCC_ECUDA;
}

using Clock = std::chrono::steady_clock;

// NVTX ranges around the pipeline stages (pack, D2H, persist, commit): free when no tool is
// attached; nsys / ncu --nvtx show them on the timeline (SURVEY §8(d) "Evidence").
struct NvtxRange {
    explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
    NvtxRange(const NvtxRange &) = delete;
    NvtxRange &operator=(const NvtxRange &) = delete;
};

// PCC_TRACE=1: one stderr line per pipeline event (debugging hangs on the GPU box)
static bool trace_on() {
    static int on = -1;
    if (on < 0) on = std::getenv("PCC_TRACE") ? 1 : 0;
    return on;
}
static double trace_ms() {
    static const auto t0 = std::chrono::steady_clock::now();
    return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
}
#define PCC_TRACE(...)                                             \
    do {                                                           \
        if (trace_on()) {                                          \
            std::fprintf(stderr, "[pcc %10.3f] ", trace_ms());     \
            std::fprintf(stderr, __VA_ARGS__);                     \
            std::fputc('\n', stderr);                              \
        }                                                          \
    } while (0)

struct Launch {
    uint32_t first, count;
    cudaEvent_t ev;
};

struct Ckpt {
    Ticket t;
    uint32_t seq = 0;  // 1, 2, ... in pcc_checkpoint order (U-gate bookkeeping)
    std::atomic<int> state{PCC_ST_QUEUED};
    std::atomic<int> err{0};
    std::atomic<bool> packed_recorded{false};  // ev_packed recorded by the packer thread
    uint64_t ring_start = 0;
    std::mutex mu;
    std::condition_variable cv;
    std::vector<Launch> launches;
    uint32_t launched = 0;  // chunks launched (guarded by mu)
    bool launch_failed = false;
    bool final_recorded = false;  // ev_final recorded (guarded by mu): finish must not sync it before
    std::atomic<uint32_t> remaining{0};
    cudaEvent_t ev_train = nullptr, ev_begin = nullptr, ev_packed = nullptr, ev_fin_k = nullptr, ev_final = nullptr;
    cudaEvent_t ev_landed = nullptr;  // copy stream, after the last chunk's D2H (timing)
    std::atomic<bool> landed_recorded{false};  // (a failed checkpoint never records it)
    double t_call = 0, t_packed = 0, t_landed = 0, t_persisted = 0, t_committed = 0;
    float pack_ms = 0, fin_ms = 0, k1_busy_ms = 0, snap_ms = 0;
    // timing events around every K1 launch: the kernel's busy time, without the gaps in which
    // the host waits for ring space between launches (those count in pack_ms, the U-gate span)
    std::vector<std::pair<cudaEvent_t, cudaEvent_t>> k1_ev;
    uint32_t digest = 0;
    std::vector<uint32_t> crc;
};

struct PersistTask {
    std::shared_ptr<Ckpt> ck;
    uint32_t j;
    char *dest;  // host address of the chunk (staging slot or file mapping)
    cudaEvent_t ev;
    bool pooled_ev;
    uint32_t nchunks = 1;  // MAPFILE: chunks [j, j+nchunks) landed by one coalesced copy
};

template <class T>
class BlockingQueue {
   public:
    void push(T v) {
        {
            std::lock_guard<std::mutex> lk(mu_);
            q_.push_back(std::move(v));
        }
        cv_.notify_one();
    }
    bool pop(T *out) {  // false on close
        std::unique_lock<std::mutex> lk(mu_);
        cv_.wait(lk, [&] { return closed_ || !q_.empty(); });
        if (q_.empty()) return false;
        *out = std::move(q_.front());
        q_.pop_front();
        return true;
    }
    void close() {
        {
            std::lock_guard<std::mutex> lk(mu_);
            closed_ = true;
        }
        cv_.notify_all();
    }

   private:
    std::mutex mu_;
    std::condition_variable cv_;
    std::deque<T> q_;
    bool closed_ = false;
};

}  // namespace pcc

using namespace pcc;

struct pcc_ctx {
    pcc_config cfg{};
    std::string path;
    int device = 0;
    Clock::time_point t0;
    cudaStream_t pack_stream = nullptr, copy_stream = nullptr, aux_stream = nullptr;
    cudaEvent_t ev_guard = nullptr;
    bool guard_armed = false;
    const CrcTables *tables = nullptr;
    const CrcConsts *consts = nullptr;
    std::atomic<uint64_t> launches{0};

    // registration
    bool registered = false;
    std::vector<pcc_tensor> tensors;
    std::vector<std::string> names;
    HostLayout layout;
    uint64_t first = 0, n = 0;
    SegRow *rows_dev = nullptr;
    uint32_t *row_begin_dev = nullptr;
    uint2 *tile_rows_dev = nullptr;
    DevGeometry geom;
    SlotGeom sgeom{};
    uint32_t lcrc = 0;
    uint32_t n_slots = 0;
    // per storage slot scratch (a slot belongs to at most one checkpoint in flight)
    std::vector<uint32_t *> tile_crc_dev, crc_dev, scratch_dev;
    std::vector<uint32_t *> crc_host;  // pinned [n + 1] (+ digest)
    uint32_t *rexpect_dev = nullptr, *rbad_dev = nullptr;  // restore: expected CRCs, bad flags [n]

    // HBM ring (Variant B).  Positions are absolute (checkpoint k's chunk j sits at position
    // ring_start(k) + j, in ring slot position % ring_slots); [ring_tail, ring_head) are
    // reserved, a position is released once its D2H landed (or it was never issued), and the
    // tail only advances over released positions — keyed by absolute position, so a release
    // can never alias a slot another in-flight chunk still owns.
    char *ring = nullptr;
    uint64_t ring_slots = 0, ring_head = 0, ring_tail = 0;
    std::set<uint64_t> ring_released;  // released positions >= ring_tail
    std::mutex ring_mu;
    std::condition_variable ring_cv;

    // U-gate bookkeeping.  The training stream may only ever wait for GPU work that is ALREADY
    // enqueued (an event): a stream-side wait for work another host thread enqueues later
    // deadlocks under PyTorch's lazy module loading and while any thread sits in a pageable
    // memcpy, which holds a process-wide driver lock (profiles/r02_gate_probe_*.txt).
    uint32_t issued_seq = 0;                 // caller thread: seq of the newest pcc_checkpoint
    std::atomic<uint32_t> packed_seq{0};     // seq whose K1 windows + ev_guard are enqueued
    uint32_t handed_seq = 0;                 // caller thread: newest seq handed to the packer thread
    std::mutex pk_mu;
    std::condition_variable pk_cv;

    // pinned staging pool (PWRITE / NULLSINK)
    char *staging = nullptr;
    uint64_t staging_slots = 0;
    std::vector<char *> staging_free;
    std::mutex st_mu;
    std::condition_variable st_cv;

    // file
    int fd = -1;
    bool odirect = false;
    char *map = nullptr;
    uint64_t map_bytes = 0;
    char *map_dev = nullptr;

    std::unique_ptr<CommitEngine> engine;
    std::mutex ck_mu;
    std::condition_variable ck_cv;
    std::map<uint64_t, std::shared_ptr<Ckpt>> ckpts;  // handle (= counter) -> record
    // terminal records pruned by gc_ckpts: handle -> outcome, so pcc_poll / pcc_wait still answer
    // for every handle until close (16 B per checkpoint; pcc_info needs the full record)
    struct Outcome {
        int state, err;
        uint64_t iter;
    };
    std::unordered_map<uint64_t, Outcome> pruned;
    pcc_restore_info rstats{};  // the last pcc_restore's breakdown

    // threads: packer (K1 windows, in checkpoint order), orchestrator (D2H), persist pool
    BlockingQueue<std::shared_ptr<Ckpt>> packs;
    std::thread packer;
    BlockingQueue<std::shared_ptr<Ckpt>> jobs;
    BlockingQueue<PersistTask> tasks;
    std::thread orchestrator;
    std::vector<std::thread> persisters;
    std::mutex evpool_mu;
    std::vector<cudaEvent_t> evpool;

    // NCCL (world > 1)
    NcclComm nccl;
    int64_t *red_dev = nullptr;
    int64_t *red_host = nullptr;

    double now_us() const { return std::chrono::duration<double, std::micro>(Clock::now() - t0).count(); }
    bool mapfile() const { return cfg.flags & PCC_MAPFILE; }
    bool nullsink() const { return cfg.flags & PCC_NULLSINK; }
    bool zerocopy() const { return cfg.flags & PCC_ZEROCOPY; }
    bool upfront() const { return (cfg.flags & PCC_D2H_UPFRONT) && !zerocopy(); }
    uint64_t cb() const { return cfg.chunk_bytes; }
    uint64_t slot_data_off(uint32_t s) const { return slot_offset(s, n, cb()) + header_bytes(n); }
};

namespace {

// a timing event pair for one K1 launch of ck (destroyed with the checkpoint's events)
std::pair<cudaEvent_t, cudaEvent_t> k1_events(Ckpt *ck) {
    std::pair<cudaEvent_t, cudaEvent_t> p{nullptr, nullptr};
    cudaEventCreate(&p.first);
    cudaEventCreate(&p.second);
    ck->k1_ev.push_back(p);
    return p;
}

cudaEvent_t get_event(pcc_ctx *c) {
    {
        std::lock_guard<std::mutex> lk(c->evpool_mu);
        if (!c->evpool.empty()) {
            cudaEvent_t e = c->evpool.back();
            c->evpool.pop_back();
            return e;
        }
    }
    cudaEvent_t e = nullptr;
    cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
    return e;
}

void put_event(pcc_ctx *c, cudaEvent_t e) {
    std::lock_guard<std::mutex> lk(c->evpool_mu);
    c->evpool.push_back(e);
}

void set_state(pcc_ctx *c, Ckpt *ck, int st) {
    {
        std::lock_guard<std::mutex> lk(c->ck_mu);
        ck->state.store(st);
    }
    c->ck_cv.notify_all();
}

void ring_release(pcc_ctx *c, uint64_t pos) {
    {
        std::lock_guard<std::mutex> lk(c->ring_mu);
        if (pos >= c->ring_tail) c->ring_released.insert(pos);
        auto it = c->ring_released.begin();
        while (it != c->ring_released.end() && *it == c->ring_tail) {
            it = c->ring_released.erase(it);
            ++c->ring_tail;
        }
    }
    c->ring_cv.notify_all();
}

char *staging_acquire(pcc_ctx *c) {
    std::unique_lock<std::mutex> lk(c->st_mu);
    c->st_cv.wait(lk, [&] { return !c->staging_free.empty(); });
    char *p = c->staging_free.back();
    c->staging_free.pop_back();
    return p;
}

void staging_release(pcc_ctx *c, char *p) {
    {
        std::lock_guard<std::mutex> lk(c->st_mu);
        c->staging_free.push_back(p);
    }
    c->st_cv.notify_one();
}

int pwrite_full(int fd, const char *p, uint64_t n, uint64_t off) {
    while (n) {
        ssize_t w = ::pwrite(fd, p, n, (off_t)off);
        if (w < 0) {
            if (errno == EINTR) continue;
            return set_errno_error("pwrite chunk", errno);
        }
        p += w;
        n -= (uint64_t)w;
        off += (uint64_t)w;
    }
    return PCC_OK;
}

void fail_ckpt(pcc_ctx *c, const std::shared_ptr<Ckpt> &ck, int err) {
    int expected = 0;
    ck->err.compare_exchange_strong(expected, err);
}

// Listing 1 lines 16-34 for a checkpoint whose chunks are all durable.
void finish_ckpt(pcc_ctx *c, const std::shared_ptr<Ckpt> &ck) {
    PCC_TRACE("finish: ckpt %llu", (unsigned long long)ck->t.counter);
    {
        // the chunks may all have landed before the training thread recorded ev_final (the
        // finalize kernel + CRC table copy): syncing an unrecorded event returns at once
        std::unique_lock<std::mutex> lk(ck->mu);
        ck->cv.wait(lk, [&] { return ck->final_recorded; });
    }
    cudaError_t e = cudaEventSynchronize(ck->ev_final);
    if (e != cudaSuccess) fail_ckpt(c, ck, cuda_error(e, "finalize"));
    cudaEventElapsedTime(&ck->pack_ms, ck->ev_begin, ck->ev_packed);
    // K1 start -> last chunk in host memory, on the GPU's clock; Variant A's K1
    // stores into host memory itself
    if (c->zerocopy() || c->n == 0 || !ck->landed_recorded.load() ||
        cudaEventElapsedTime(&ck->snap_ms, ck->ev_begin, ck->ev_landed) != cudaSuccess)
        ck->snap_ms = ck->pack_ms;
    ck->k1_busy_ms = 0;
    for (auto &p : ck->k1_ev) {
        float ms = 0;
        if (cudaEventElapsedTime(&ms, p.first, p.second) == cudaSuccess) ck->k1_busy_ms += ms;
    }
    cudaEventElapsedTime(&ck->fin_ms, ck->ev_packed, ck->ev_fin_k);  // the finalize kernel alone
    const uint32_t *h = c->crc_host[ck->t.slot];
    ck->crc.assign(h, h + c->n);
    ck->digest = h[c->n];
    ck->t_persisted = c->now_us();
    if (ck->err.load()) {
        c->engine->fail(ck->t);
        set_state(c, ck.get(), PCC_ST_FAILED);
        return;
    }
    if (c->fd >= 0 && (c->cfg.flags & PCC_FSYNC) && ::fdatasync(c->fd) != 0) {
        fail_ckpt(c, ck, set_errno_error("fdatasync", errno));
        c->engine->fail(ck->t);
        set_state(c, ck.get(), PCC_ST_FAILED);
        return;
    }
    set_state(c, ck.get(), PCC_ST_PERSISTED);
    NvtxRange nv("pcc.commit");
    int st = PCC_ST_FAILED;
    int rc = c->engine->complete(ck->t, ck->crc.data(), ck->digest, &st);
    PCC_TRACE("finish: ckpt %llu committed state %d rc %d", (unsigned long long)ck->t.counter, st, rc);
    if (rc) fail_ckpt(c, ck, rc);
    if (c->cfg.world == 1 || st == PCC_ST_FAILED) {
        ck->t_committed = c->now_us();
        set_state(c, ck.get(), st);
    }
    // world > 1: the engine's on_state callback moves it to LOCAL_COMMIT in counter order
}

void persist_loop(pcc_ctx *c) {
    cudaSetDevice(c->device);
    PersistTask task;
    while (c->tasks.pop(&task)) {
        NvtxRange nv("pcc.persist");
        Ckpt *ck = task.ck.get();
        PCC_TRACE("persist: ckpt %llu chunk %u wait", (unsigned long long)ck->t.counter, task.j);
        cudaError_t e = cudaEventSynchronize(task.ev);
        PCC_TRACE("persist: ckpt %llu chunk %u landed (%s)", (unsigned long long)ck->t.counter, task.j, cudaGetErrorString(e));
        if (e != cudaSuccess) fail_ckpt(c, task.ck, cuda_error(e, "chunk copy"));
        if (task.pooled_ev) put_event(c, task.ev);
        if (!c->zerocopy())
            for (uint32_t q = 0; q < task.nchunks; ++q) ring_release(c, ck->ring_start + task.j + q);
        const double t = c->now_us();
        if (!c->mapfile()) {
            if (!c->nullsink() && !ck->err.load()) {
                int rc = pwrite_full(c->fd, task.dest, c->cb(), c->slot_data_off(ck->t.slot) + task.j * c->cb());
                if (rc) fail_ckpt(c, task.ck, rc);
            }
            staging_release(c, task.dest);
        }
        {
            std::lock_guard<std::mutex> lk(ck->mu);
            ck->t_landed = std::max(ck->t_landed, t);
        }
        PCC_TRACE("persist: ckpt %llu chunk %u done", (unsigned long long)ck->t.counter, task.j);
        if (fault_hit("chunk")) fault_die();
        if (ck->remaining.fetch_sub(task.nchunks) == task.nchunks) finish_ckpt(c, task.ck);
    }
}

void orchestrate_loop(pcc_ctx *c) {
    cudaSetDevice(c->device);
    // D2H pieces and queue depth (PCC_D2H_PIECE_MIB / PCC_D2H_DEPTH: A/B hooks)
    static const uint64_t d2h_piece = [] {
        const char *e = std::getenv("PCC_D2H_PIECE_MIB");
        const uint64_t m = e ? std::strtoull(e, nullptr, 10) : 0;
        return (m ? m : 64ull) << 20;
    }();
    static const size_t d2h_depth = [] {
        const char *e = std::getenv("PCC_D2H_DEPTH");
        const size_t d = e ? (size_t)std::strtoull(e, nullptr, 10) : 0;
        return d ? d : (size_t)4;
    }();
    // ... and every d2h_drain BYTES the queue runs empty once: a copy engine that always has
    // work queued from one stream never serves another stream's copy (measured: a 4-byte
    // .item() on the training stream waited 105 ms for the whole 8 GiB stream at depth 2-4,
    // 0.1 ms with a gap), and HF models read a flag to the host every forward pass.  128 MiB
    // bounds that wait to ~2.4 ms (profiles/r01_d2h_starvation.md: OPT-1.3B unpaced slowdown
    // 41-46% -> 12.7%, C2 snapshot 55.7 GB/s).  Counted in bytes, not copies: with the pacer's
    // 0.5 MiB quanta a per-copy count drained every 1 MiB and the host round trips capped the
    // paced transfer at ~9.5 GB/s against a 28.6 GB/s target.  A paced transfer
    // never drains: its own gaps already let other streams' copies through.
    // With small unpaced copies (d2h_quantum <= 2 MiB: the tuner's choice under an eager loop)
    // the queue drains every 16 MiB: eager OPT-1.3B 8.8% -> 7.6% (profiles/r02e2_eager_piece.jsonl).
    static const uint64_t d2h_drain_env = [] {
        const char *e = std::getenv("PCC_D2H_DRAIN_MIB");
        return e ? std::strtoull(e, nullptr, 10) << 20 : ~0ull;  // 0 = never
    }();

    uint64_t since_drain = 0;
    std::deque<cudaEvent_t> queued;  // completion events of the pieces on the copy engine
    // waited for by polling cudaEventQuery between yields: cudaEventSynchronize's spin delayed
    // the K1 launches of the training thread by ~20 us (K1 0.41 -> 0.43 ms in the C2 bench),
    // and blocking-sync events wake up too late to keep the link busy (47.6 GB/s)
    auto q_wait = [](cudaEvent_t e) {
        while (cudaEventQuery(e) == cudaErrorNotReady) std::this_thread::yield();
    };
    std::shared_ptr<Ckpt> ck;
    while (c->jobs.pop(&ck)) {
        PCC_TRACE("orch: ckpt %llu iter %llu slot %u", (unsigned long long)ck->t.counter,
                  (unsigned long long)ck->t.iter, ck->t.slot);
        NvtxRange nv("pcc.d2h");
        if (c->fd >= 0 && !c->zerocopy()) {
            int rc = c->engine->filling(ck->t);  // R18: before any data byte of this slot changes
            if (rc) fail_ckpt(c, ck, rc);
        }
        size_t li = 0;
        uint32_t issued = 0;
        // D2H pacing (pcc_config d2h_mbps / d2h_quantum): copies of at most `quantum` bytes,
        // issued no faster than `pace` bytes per microsecond once the chunks exist in HBM
        const uint64_t pace = c->cfg.d2h_mbps;  // MB/s == bytes per microsecond
        const uint64_t quantum = c->cfg.d2h_quantum;
        const uint64_t d2h_drain = d2h_drain_env != ~0ull                      ? d2h_drain_env
                                   : (quantum && quantum <= (2ull << 20)) ? (16ull << 20)
                                                                          : (128ull << 20);
        Clock::time_point t_pace{};
        bool pace_started = false;
        uint64_t paced_bytes = 0;
        for (uint32_t j = 0; j < c->n;) {
            Launch L;
            {
                std::unique_lock<std::mutex> lk(ck->mu);
                ck->cv.wait(lk, [&] { return ck->launched > j || ck->launch_failed; });
                if (ck->launch_failed && ck->launched <= j) break;
                while (!(j >= ck->launches[li].first && j < ck->launches[li].first + ck->launches[li].count)) ++li;
                L = ck->launches[li];
            }
            PersistTask task{ck, j, nullptr, nullptr, false};
            if (c->zerocopy()) {
                task.ev = L.ev;  // K1 stored the chunk straight into the file mapping
                task.dest = c->map + c->slot_data_off(ck->t.slot) + (uint64_t)j * c->cb();
            } else {
                if (j == L.first) cudaStreamWaitEvent(c->copy_stream, L.ev, 0);
                const uint64_t r0 = (ck->ring_start + j) % c->ring_slots;
                if (pace && j == L.first) {
                    cudaEventSynchronize(L.ev);  // pace from when the chunks exist
                    if (!pace_started) t_pace = Clock::now();
                    pace_started = true;
                }
                if (c->mapfile()) {
                    // coalesce chunks of this launch that are contiguous in the ring (and, always,
                    // in the slot) into one copy of up to kCoalesceBytes: fewer, larger D2H
                    static const uint64_t kCoalesceBytes = [] {  // PCC_COALESCE_MIB: A/B hook
                        const char *e = std::getenv("PCC_COALESCE_MIB");
                        const uint64_t mib = e ? std::strtoull(e, nullptr, 10) : 0;
                        return (mib ? mib : 64ull) << 20;
                    }();
                    uint64_t k = 1;
                    const uint64_t kmax = std::max<uint64_t>(1, kCoalesceBytes / c->cb());
                    while (k < kmax && j + k < L.first + L.count && r0 + k < c->ring_slots) ++k;
                    task.nchunks = (uint32_t)k;
                    task.dest = c->map + c->slot_data_off(ck->t.slot) + (uint64_t)j * c->cb();
                } else {
                    task.dest = staging_acquire(c);
                }
                PCC_TRACE("orch: ckpt %llu chunks %u+%u -> %p", (unsigned long long)ck->t.counter, j, task.nchunks,
                          (void *)task.dest);
                const char *src = c->ring + r0 * c->cb();
                const uint64_t total = task.nchunks * c->cb();
                const uint64_t q = quantum ? quantum : std::min<uint64_t>(total, d2h_piece);
                for (uint64_t o = 0; o < total; o += q) {
                    const uint64_t len = std::min(q, total - o);
                    if (pace) {
                        std::this_thread::sleep_until(t_pace + std::chrono::microseconds(paced_bytes / pace));
                        paced_bytes += len;
                    }
                    // bounded copy queue with periodic gaps: any D2H the training issues (even a
                    // 4-byte .item()) waits behind the copies on the copy engine; queued back to
                    // back, a whole checkpoint (OPT-1.3B: 16 GB) stalled the iteration after each
                    // checkpoint by ~230 ms
                    const bool drain = !pace && d2h_drain && since_drain >= d2h_drain;
                    if (drain) since_drain = 0;
                    since_drain += len;
                    while (!queued.empty() && (drain || queued.size() >= d2h_depth)) {
                        q_wait(queued.front());
                        put_event(c, queued.front());
                        queued.pop_front();
                    }
                    cudaError_t e = cudaMemcpyAsync(task.dest + o, src + o, len, cudaMemcpyDeviceToHost, c->copy_stream);
                    if (e != cudaSuccess) fail_ckpt(c, ck, cuda_error(e, "D2H"));
                    cudaEvent_t qe = get_event(c);
                    cudaEventRecord(qe, c->copy_stream);
                    queued.push_back(qe);
                }
                if (j + task.nchunks == c->n) {  // before the task
                    cudaEventRecord(ck->ev_landed, c->copy_stream);
                    ck->landed_recorded = true;
                }
                task.ev = get_event(c);
                task.pooled_ev = true;
                cudaEventRecord(task.ev, c->copy_stream);
            }
            const uint32_t adv = task.nchunks;
            c->tasks.push(task);
            issued += adv;
            j += adv;
        }
        // chunks never issued (K1 launch failed) count as done so the checkpoint still
        // terminates, and give their reserved ring chunks back
        const uint32_t unissued = (uint32_t)c->n - issued;
        if (!c->zerocopy())
            for (uint32_t j = issued; j < c->n; ++j) ring_release(c, ck->ring_start + j);
        if (c->n == 0 || (unissued && ck->remaining.fetch_sub(unissued) == unissued)) finish_ckpt(c, ck);
    }
    for (cudaEvent_t e : queued) {
        cudaEventSynchronize(e);
        put_event(c, e);
    }
}

int free_registration(pcc_ctx *c) {
    cudaFree(c->rows_dev);
    cudaFree(c->row_begin_dev);
    cudaFree(c->tile_rows_dev);
    c->rows_dev = nullptr;
    c->row_begin_dev = nullptr;
    c->tile_rows_dev = nullptr;
    free_geometry(&c->geom);
    for (auto p : c->tile_crc_dev) cudaFree(p);
    for (auto p : c->crc_dev) cudaFree(p);
    for (auto p : c->scratch_dev) cudaFree(p);
    for (auto p : c->crc_host) cudaFreeHost(p);
    cudaFree(c->rexpect_dev);
    cudaFree(c->rbad_dev);
    c->rexpect_dev = c->rbad_dev = nullptr;
    c->tile_crc_dev.clear();
    c->crc_dev.clear();
    c->scratch_dev.clear();
    c->crc_host.clear();
    if (c->ring) cudaFree(c->ring);
    c->ring = nullptr;
    if (c->staging) cudaFreeHost(c->staging);
    c->staging = nullptr;
    c->staging_free.clear();
    if (c->map) {
        cudaHostUnregister(c->map);
        munmap(c->map, c->map_bytes);
        c->map = nullptr;
        c->map_dev = nullptr;
    }
    c->engine.reset();
    c->registered = false;
    return PCC_OK;
}

void destroy_ckpt_events(pcc_ctx *c, Ckpt *ck) {
    cudaEventDestroy(ck->ev_train);
    cudaEventDestroy(ck->ev_begin);
    cudaEventDestroy(ck->ev_packed);
    cudaEventDestroy(ck->ev_landed);
    cudaEventDestroy(ck->ev_fin_k);
    cudaEventDestroy(ck->ev_final);
    for (auto &L : ck->launches) put_event(c, L.ev);
    ck->launches.clear();
    for (auto &p : ck->k1_ev) {
        cudaEventDestroy(p.first);
        cudaEventDestroy(p.second);
    }
    ck->k1_ev.clear();
}

// keeps the newest kKeep terminal records queryable (pcc_info), frees older ones
void gc_ckpts(pcc_ctx *c) {
    constexpr size_t kKeep = 64;
    std::vector<std::shared_ptr<Ckpt>> dead;
    {
        std::lock_guard<std::mutex> lk(c->ck_mu);
        if (c->ckpts.size() <= kKeep) return;
        size_t excess = c->ckpts.size() - kKeep;
        for (auto it = c->ckpts.begin(); it != c->ckpts.end() && excess;) {
            int s = it->second->state.load();
            bool term = s == PCC_ST_LOCAL_COMMIT || s == PCC_ST_GLOBAL_COMMIT || s == PCC_ST_OBSOLETE ||
                        s == PCC_ST_FAILED;
            if (term && it->second->remaining.load() == 0) {
                dead.push_back(it->second);
                c->pruned[it->first] = {s, it->second->err.load(), it->second->t.iter};
                it = c->ckpts.erase(it);
                --excess;
            } else {
                ++it;
            }
        }
    }
    for (auto &ck : dead) destroy_ckpt_events(c, ck.get());
}

bool any_inflight(pcc_ctx *c) {
    std::lock_guard<std::mutex> lk(c->ck_mu);
    for (auto &kv : c->ckpts) {
        int s = kv.second->state.load();
        if (s != PCC_ST_LOCAL_COMMIT && s != PCC_ST_GLOBAL_COMMIT && s != PCC_ST_OBSOLETE && s != PCC_ST_FAILED)
            return true;
    }
    return false;
}

// K1 for one checkpoint, after the caller's event on the training stream: run inline by
// pcc_checkpoint when the ring already has room, else by the packer thread, strictly in
// checkpoint order either way, so K1 windows, ev_guard and the finalize kernels of successive
// checkpoints are stream-ordered on the pack stream.  Waiting for HBM ring space (Variant B
// with a ring smaller than the slices in flight) happens in the packer thread, never in the
// caller's pcc_checkpoint.
void pack_one(pcc_ctx *c, const std::shared_ptr<Ckpt> &ck) {
    NvtxRange nv("pcc.pack");
    const uint32_t s = ck->t.slot;
    cudaStreamWaitEvent(c->pack_stream, ck->ev_train, 0);
    if (c->fd >= 0 && (c->zerocopy() || c->upfront())) {
        // R18: the reused slot's header becomes FILLING before any data byte of the slot changes.
        // In ZEROCOPY mode K1 itself stores into the slot's file pages, and with D2H_UPFRONT the
        // copies are enqueued with the K1 windows, so this happens before K1 is launched (ADVICE
        // r01); otherwise the orchestrator writes it before its first D2H.
        int rc = c->engine->filling(ck->t);
        if (rc) fail_ckpt(c, ck, rc);
    }
    set_state(c, ck.get(), PCC_ST_PACKING);
    SnapParams P{};
    P.rows = c->rows_dev;
    P.row_begin = c->row_begin_dev;
    P.tile_rows = c->tile_rows_dev;
    P.chunk_bytes = c->cb();
    P.tpc = c->geom.tpc;
    P.tile_crc = c->tile_crc_dev[s];
    P.tables = c->tables;
    P.consts = c->consts;
    cudaError_t e = cudaSuccess;
    // publishes a successful window to the orchestrator (a failed one never is); with
    // D2H_UPFRONT this thread enqueues the window's copy-engine D2H itself, right away
    uint32_t issued = 0;
    auto publish = [&](uint32_t first, uint32_t count) {
        cudaEvent_t ev = get_event(c);
        cudaEventRecord(ev, c->pack_stream);
        if (c->upfront()) {
            cudaStreamWaitEvent(c->copy_stream, ev, 0);
            for (uint32_t j = first; j < first + count;) {
                const uint64_t r0 = (ck->ring_start + j) % c->ring_slots;
                uint32_t k = 1;  // chunks contiguous in the ring, up to 64 MiB per copy
                const uint64_t kmax = std::max<uint64_t>(1, (64ull << 20) / c->cb());
                while (k < kmax && j + k < first + count && r0 + k < c->ring_slots) ++k;
                PersistTask task{ck, j, c->map + c->slot_data_off(ck->t.slot) + (uint64_t)j * c->cb(), nullptr, true, k};
                cudaError_t e2 = cudaMemcpyAsync(task.dest, c->ring + r0 * c->cb(), (uint64_t)k * c->cb(),
                                                 cudaMemcpyDeviceToHost, c->copy_stream);
                if (e2 != cudaSuccess) fail_ckpt(c, ck, cuda_error(e2, "D2H"));
                if (j + k == c->n) {
                    cudaEventRecord(ck->ev_landed, c->copy_stream);
                    ck->landed_recorded = true;
                }
                task.ev = get_event(c);
                cudaEventRecord(task.ev, c->copy_stream);
                c->tasks.push(task);
                j += k;
                issued = j;
            }
        }
        {
            std::lock_guard<std::mutex> lk(ck->mu);
            ck->launches.push_back({first, count, ev});
            ck->launched = first + count;
        }
        ck->cv.notify_all();  // the orchestrator may already be waiting for this launch
    };
    cudaEventRecord(ck->ev_begin, c->pack_stream);  // K1 time excludes the caller's wait
    if (c->zerocopy()) {  // Variant A: K1 stores into the registered file mapping over PCIe
        P.first = 0;
        P.count = (uint32_t)c->n;
        P.ring_base = c->map_dev + c->slot_data_off(s);
        P.ring_head = 0;
        P.ring_slots = c->n ? c->n : 1;
        const auto k1e = k1_events(ck.get());
        cudaEventRecord(k1e.first, c->pack_stream);
        e = launch_pack(P, snapshot_grid(c->device, P.count * P.tpc, c->cfg.pack_ctas, true), c->pack_stream);
        cudaEventRecord(k1e.second, c->pack_stream);
        c->launches += c->n ? 1 : 0;
        if (e == cudaSuccess) publish(0, (uint32_t)c->n);
    } else {  // Variant B: HBM ring, windowed by ring space
        {
            std::lock_guard<std::mutex> lk(c->ring_mu);
            ck->ring_start = c->ring_head;
            c->ring_head += c->n;
        }
        uint64_t done = 0;
        while (done < c->n && e == cudaSuccess) {
            uint64_t k;
            {
                // launch windows of at least half the ring (or the rest of the slice): when the
                // link is the bottleneck the ring frees a chunk or two at a time, and a K1 launch
                // per freed chunk pays the table load and launch latency each time (C3 with
                // N = 4 over a 2-slice ring: 114 launches per checkpoint, 11.7 ms of K1 instead
                // of 5.7).  The chunks already packed keep the copy engine busy meanwhile.  Half
                // (round 2; a quarter before): a 2-slice ring packs each back-to-back checkpoint
                // in one launch (1.9 before), a 1-slice ring in at most two.
#ifndef PCC_RING_WINDOW_DIV  // A/B hook: 4 = the earlier quarter-ring rule
#define PCC_RING_WINDOW_DIV 2
#endif
                const uint64_t want =
                    std::min<uint64_t>(c->n - done, std::max<uint64_t>(1, c->ring_slots / PCC_RING_WINDOW_DIV));
                std::unique_lock<std::mutex> lk(c->ring_mu);
                c->ring_cv.wait(lk, [&] { return c->ring_tail + c->ring_slots >= ck->ring_start + done + want; });
                k = std::min<uint64_t>(c->n - done, c->ring_tail + c->ring_slots - (ck->ring_start + done));
            }
            P.first = (uint32_t)done;
            P.count = (uint32_t)k;
            P.ring_base = c->ring;
            P.ring_head = ck->ring_start % c->ring_slots;
            P.ring_slots = c->ring_slots;
            const auto k1e = k1_events(ck.get());
            cudaEventRecord(k1e.first, c->pack_stream);
            // PCC_FAULT=k1_fail:<n>: the n-th K1 window of the process fails to launch (test hook)
            e = fault_hit("k1_fail") ? cudaErrorLaunchFailure
                                     : launch_pack(P, snapshot_grid(c->device, P.count * P.tpc, c->cfg.pack_ctas, true),
                                                   c->pack_stream);
            cudaEventRecord(k1e.second, c->pack_stream);
            c->launches += 1;
            if (e != cudaSuccess) break;
            PCC_TRACE("pack: ckpt %llu window %llu+%llu launched", (unsigned long long)ck->t.counter,
                      (unsigned long long)done, (unsigned long long)k);
            publish((uint32_t)done, (uint32_t)k);
            done += k;
        }
    }
    cudaEventRecord(ck->ev_packed, c->pack_stream);
    ck->packed_recorded = true;
    // the U-gate event: after the last K1 window (recorded even when a launch failed, so a
    // guarded training stream is never left waiting)
    cudaEventRecord(c->ev_guard, c->pack_stream);
    // chunk CRCs -> slice digest, then the table to pinned host memory for the header
    cudaMemsetAsync(c->scratch_dev[s], 0, 4 * sizeof(uint32_t), c->pack_stream);
    FinalizeParams F{};
    F.tile_crc = c->tile_crc_dev[s];
    F.tables = c->tables;
    F.n = (uint32_t)c->n;
    F.tpc = c->geom.tpc;
    F.tile_shift = c->geom.tile_shift;
    F.chunk_shift = c->geom.chunk_shift;
    F.ff = c->geom.ff;
    F.crc_out = c->crc_dev[s];
    F.scratch = c->scratch_dev[s];
    if (e == cudaSuccess) e = launch_finalize(F, c->pack_stream);
    cudaEventRecord(ck->ev_fin_k, c->pack_stream);
    if (c->n) c->launches += kFinalizeLaunches;
    cudaMemcpyAsync(c->crc_dev[s] + c->n, c->scratch_dev[s] + 3, 4, cudaMemcpyDeviceToDevice, c->pack_stream);
    cudaMemcpyAsync(c->crc_host[s], c->crc_dev[s], (c->n + 1) * sizeof(uint32_t), cudaMemcpyDeviceToHost,
                    c->pack_stream);
    cudaEventRecord(ck->ev_final, c->pack_stream);
    {
        std::lock_guard<std::mutex> lk(ck->mu);
        ck->final_recorded = true;
        if (e != cudaSuccess) {
            fail_ckpt(c, ck, cuda_error(e, "K1 launch"));
            ck->launch_failed = true;
        }
    }
    ck->cv.notify_all();
    {  // everything of this checkpoint is on the pack stream: pcc_guard may take ev_guard now
        std::lock_guard<std::mutex> lk(c->pk_mu);
        c->packed_seq.store(ck->seq);
    }
    c->pk_cv.notify_all();
    if (c->upfront()) {  // the orchestrator's end-of-checkpoint accounting, done here
        const uint32_t unissued = (uint32_t)c->n - issued;
        for (uint32_t j = issued; j < c->n; ++j) ring_release(c, ck->ring_start + j);  // never issued
        if (c->n == 0 || (unissued && ck->remaining.fetch_sub(unissued) == unissued)) finish_ckpt(c, ck);
    }
}

void pack_loop(pcc_ctx *c) {
    cudaSetDevice(c->device);
    std::shared_ptr<Ckpt> ck;
    while (c->packs.pop(&ck)) pack_one(c, ck);
}

}  // namespace

// ============================================================================ C ABI
extern "C" {

const char *pcc_strerror(int err) {
    switch (err < 0 ? -err : err) {
        case PCC_OK: return "ok";
        case PCC_EINVAL: return "invalid argument";
        case PCC_ENOMEM: return "out of memory";
        case PCC_EBUSY: return "checkpoints in flight";
        case PCC_EAGAIN: return "try again";
        case PCC_EIO: return "I/O error";
        case PCC_ECUDA: return "CUDA error";
        case PCC_ENCCL: return "NCCL error";
        case PCC_EORDER: return "iter not strictly increasing";
        case PCC_ECORRUPT: return "checksum mismatch";
        case PCC_ELAYOUT: return "layout mismatch";
        case PCC_ENOENT: return "no valid checkpoint";
        case PCC_ETIMEDOUT: return "timed out";
        case PCC_ESTATE: return "invalid state";
        default: return "unknown error";
    }
}
uint64_t pcc_struct_size(int which) {
    return which == 0   ? sizeof(pcc_config)
           : which == 1 ? sizeof(pcc_tensor)
           : which == 2 ? sizeof(pcc_ckpt_info)
           : which == 3 ? sizeof(pcc_restore_info)
                        : 0;
}
const char *pcc_last_error(void) { return err_state().msg.c_str(); }
int pcc_last_errno(void) { return err_state().err_no; }

int pcc_open(const pcc_config *cfg, pcc_ctx **out) {
    if (!out) return set_error(PCC_EINVAL, "out");
    *out = nullptr;
    if (!cfg || cfg->abi_version != PCC_ABI_VERSION) return set_error(PCC_EINVAL, "abi version");
    if (cfg->chunk_bytes == 0 || cfg->chunk_bytes % 16 || cfg->chunk_bytes >= (1ull << 32) || cfg->max_inflight == 0)
        return set_error(PCC_EINVAL, "chunk_bytes / max_inflight");
    if (cfg->world < 1 || cfg->rank < 0 || cfg->rank >= cfg->world) return set_error(PCC_EINVAL, "rank/world");
    const bool nullsink = cfg->flags & PCC_NULLSINK;
    if (!nullsink && !cfg->path) return set_error(PCC_EINVAL, "path");
    if ((cfg->flags & (PCC_MAPFILE | PCC_ODIRECT)) && cfg->chunk_bytes % kPage)
        return set_error(PCC_EINVAL, "chunk_bytes must be a multiple of 4096 with ODIRECT/MAPFILE");
    if ((cfg->flags & PCC_ZEROCOPY) && !(cfg->flags & PCC_MAPFILE))
        return set_error(PCC_EINVAL, "ZEROCOPY needs MAPFILE");
    if (nullsink && (cfg->flags & PCC_MAPFILE)) return set_error(PCC_EINVAL, "NULLSINK excludes MAPFILE");
    if ((cfg->flags & PCC_D2H_UPFRONT) && !(cfg->flags & PCC_MAPFILE))
        return set_error(PCC_EINVAL, "D2H_UPFRONT needs MAPFILE (copies straight into the file pages)");
    if ((cfg->allreduce == nullptr) != (cfg->allgather == nullptr))
        return set_error(PCC_EINVAL, "allreduce and allgather callbacks go together");
    if (cfg->world > 1 && !(cfg->flags & PCC_NOCOMM) && !cfg->allreduce && !cfg->nccl_unique_id)
        return set_error(PCC_EINVAL, "world > 1 needs nccl_unique_id, caller collectives or PCC_NOCOMM");
    std::unique_ptr<pcc_ctx> c(new pcc_ctx());
    c->cfg = *cfg;
    if (cfg->path) c->path = cfg->path;
    c->cfg.path = c->path.c_str();
    if (!c->cfg.align) c->cfg.align = 256;
    if (c->cfg.align % 16) return set_error(PCC_EINVAL, "align % 16");
    if (!c->cfg.writer_threads) c->cfg.writer_threads = 4;
    c->device = cfg->device;
    c->t0 = Clock::now();
    cudaError_t e = cudaSetDevice(c->device);
    if (e != cudaSuccess) return cuda_error(e, "cudaSetDevice");
    if ((e = device_tables(c->device, &c->tables, &c->consts)) != cudaSuccess) return cuda_error(e, "CRC tables");
    // load every kernel the pipeline launches now, on the caller's thread: under lazy module
    // loading (PyTorch's default) a first launch synchronises the context, which must not happen
    // inside a checkpoint
    if ((e = warm_kernels(c->device, c->tables)) != cudaSuccess) return cuda_error(e, "kernel warm-up");
    int lo = 0, hi = 0;
    cudaDeviceGetStreamPriorityRange(&lo, &hi);
    // PCC_PACK_PRIO=low|default (experiments): K1's stream priority relative to training
    const char *pp = std::getenv("PCC_PACK_PRIO");
    const int prio = pp && !std::strcmp(pp, "low") ? lo : pp && !std::strcmp(pp, "default") ? 0 : hi;
    if ((e = cudaStreamCreateWithPriority(&c->pack_stream, cudaStreamNonBlocking, prio)) != cudaSuccess)
        return cuda_error(e, "stream");
    cudaStreamCreateWithFlags(&c->copy_stream, cudaStreamNonBlocking);
    cudaStreamCreateWithFlags(&c->aux_stream, cudaStreamNonBlocking);
    cudaEventCreateWithFlags(&c->ev_guard, cudaEventDisableTiming);
    if (!nullsink) {
        int flags = O_RDWR | O_CREAT;
        if ((cfg->flags & PCC_ODIRECT) && !(cfg->flags & PCC_MAPFILE)) flags |= O_DIRECT;
        c->fd = ::open(c->path.c_str(), flags, 0644);
        if (c->fd < 0 && (flags & O_DIRECT) && errno == EINVAL) {
            flags &= ~O_DIRECT;  // filesystem without O_DIRECT: buffered
            c->fd = ::open(c->path.c_str(), flags, 0644);
        }
        if (c->fd < 0) return set_errno_error("open checkpoint file", errno);
        c->odirect = flags & O_DIRECT;
    }
    if (cfg->world > 1 && !(cfg->flags & PCC_NOCOMM) && !cfg->allreduce) {
        int rc = c->nccl.init(cfg->nccl_unique_id, cfg->world, cfg->rank);
        if (rc) return rc;
        cudaMalloc(&c->red_dev, 4 * sizeof(int64_t));
        cudaMallocHost(&c->red_host, 4 * sizeof(int64_t));
    }
    pcc_ctx *raw = c.get();
    raw->packer = std::thread(pack_loop, raw);
    raw->orchestrator = std::thread(orchestrate_loop, raw);
    for (uint32_t i = 0; i < raw->cfg.writer_threads; ++i) raw->persisters.emplace_back(persist_loop, raw);
    *out = c.release();
    return PCC_OK;
}

int pcc_register(pcc_ctx *c, const pcc_tensor *t, uint32_t nt) {
    if (!c || (nt && !t)) return set_error(PCC_EINVAL, "args");
    if (any_inflight(c)) return set_error(PCC_EBUSY, "checkpoints in flight");
    cudaSetDevice(c->device);
    free_registration(c);
    c->tensors.assign(t, t + nt);
    c->names.clear();
    for (uint32_t i = 0; i < nt; ++i) {
        c->names.emplace_back(t[i].name ? t[i].name : "");
        c->tensors[i].name = nullptr;
    }
    HostLayout full;
    int rc = build_layout(t, nt, c->cfg.align, c->cb(), 0, 0, &full);
    if (rc) return set_error(PCC_EINVAL, "layout");
    if (c->cfg.flags & PCC_SHARDED) {  // each rank's registration is its own shard: all of it
        c->first = 0;
        c->n = full.C;
    } else {
        slice_of(full.C, c->cfg.rank, c->cfg.world, &c->first, &c->n);
    }
    rc = build_layout(t, nt, c->cfg.align, c->cb(), c->first, (int64_t)c->n, &c->layout);
    if (rc) return set_error(PCC_EINVAL, "layout slice");
    build_tile_rows(&c->layout, c->cb(), kTile);
    std::vector<uint64_t> nb(nt);
    std::vector<uint32_t> dt(nt);
    for (uint32_t i = 0; i < nt; ++i) {
        nb[i] = t[i].nbytes;
        dt[i] = t[i].dtype;
    }
    c->lcrc = layout_crc(nt, nb.data(), dt.data(), c->cfg.align, c->cb());
    c->sgeom = SlotGeom{c->cb(), (uint32_t)c->cfg.rank, (uint32_t)c->cfg.world, (uint32_t)c->layout.C,
                        (uint32_t)c->first, (uint32_t)c->n, nt, c->cfg.align, c->lcrc};
    c->n_slots = c->cfg.max_inflight + 1;
    cudaError_t e;
    const size_t nrows = c->layout.rows.empty() ? 1 : c->layout.rows.size();
    if ((e = cudaMalloc(&c->rows_dev, nrows * sizeof(SegRow))) != cudaSuccess) return cuda_error(e, "rows");
    if ((e = cudaMalloc(&c->row_begin_dev, (c->n + 1) * sizeof(uint32_t))) != cudaSuccess) return cuda_error(e, "rb");
    if (!c->layout.rows.empty())
        cudaMemcpyAsync(c->rows_dev, c->layout.rows.data(), c->layout.rows.size() * sizeof(SegRow),
                        cudaMemcpyHostToDevice, c->pack_stream);
    // NB: uploads go on the pack stream, never the legacy stream: a pageable cudaMemcpy may return
    // before its DMA lands, and the library's streams do not synchronise with the legacy stream
    cudaMemcpyAsync(c->row_begin_dev, c->layout.row_begin.data(), (c->n + 1) * sizeof(uint32_t), cudaMemcpyHostToDevice,
                    c->pack_stream);
    {
        const size_t tb = std::max<size_t>(c->layout.tile_rows.size(), 2) * sizeof(uint32_t);
        if ((e = cudaMalloc(&c->tile_rows_dev, tb)) != cudaSuccess) return cuda_error(e, "tile rows");
        if (!c->layout.tile_rows.empty())
            cudaMemcpyAsync(c->tile_rows_dev, c->layout.tile_rows.data(), c->layout.tile_rows.size() * sizeof(uint32_t),
                            cudaMemcpyHostToDevice, c->pack_stream);
    }
    if ((e = setup_geometry(&c->geom, c->cb(), (uint32_t)c->n, c->pack_stream)) != cudaSuccess)
        return cuda_error(e, "geometry");
    const uint64_t nn = c->n ? c->n : 1;
    for (uint32_t s = 0; s < c->n_slots; ++s) {
        uint32_t *a = nullptr, *b = nullptr, *d = nullptr, *h = nullptr;
        if ((e = cudaMalloc(&a, nn * tile_crc_words(c->geom.tpc) * sizeof(uint32_t))) != cudaSuccess)
            return cuda_error(e, "tile crc");
        if ((e = cudaMalloc(&b, (nn + 1) * sizeof(uint32_t))) != cudaSuccess) return cuda_error(e, "crc");
        if ((e = cudaMalloc(&d, 4 * sizeof(uint32_t))) != cudaSuccess) return cuda_error(e, "scratch");
        if ((e = cudaMallocHost(&h, (nn + 1) * sizeof(uint32_t))) != cudaSuccess) return cuda_error(e, "crc host");
        c->tile_crc_dev.push_back(a);
        c->crc_dev.push_back(b);
        c->scratch_dev.push_back(d);
        c->crc_host.push_back(h);
    }
    if ((e = cudaMalloc(&c->rexpect_dev, nn * 4)) != cudaSuccess) return cuda_error(e, "restore buffers");
    if ((e = cudaMalloc(&c->rbad_dev, nn * 4)) != cudaSuccess) return cuda_error(e, "restore buffers");
    // HBM ring: default one whole slice (L139's extra copy)
    if (!c->zerocopy()) {
        uint64_t r = c->cfg.ring_bytes ? c->cfg.ring_bytes / c->cb() : c->n;
        if (r == 0) r = 1;
        if (r > 8 * nn) r = 8 * nn;  // more than 8 slices of ring cannot be used (N in flight)
        c->ring_slots = r;
        if ((e = cudaMalloc(&c->ring, r * c->cb())) != cudaSuccess) return cuda_error(e, "HBM ring");
        c->ring_released.clear();
        c->ring_head = c->ring_tail = 0;
    }
    // staging pool (c = M / b, L176)
    if (!c->mapfile()) {
        uint64_t k = c->cfg.staging_bytes / c->cb();
        if (k == 0) k = std::max<uint64_t>(2 * c->cfg.writer_threads, 4);
        if (k > nn) k = nn;
        c->staging_slots = k;
        if ((e = cudaHostAlloc(&c->staging, k * c->cb(), cudaHostAllocPortable)) != cudaSuccess)
            return cuda_error(e, "pinned staging");
        for (uint64_t i = 0; i < k; ++i) c->staging_free.push_back(c->staging + i * c->cb());
    }
    // file: N+1 slots
    if (c->fd >= 0) {
        const uint64_t fbytes = file_bytes(c->n_slots, c->n, c->cb());
        struct stat st;
        if (fstat(c->fd, &st) == 0 && (uint64_t)st.st_size < fbytes && ftruncate(c->fd, (off_t)fbytes) != 0)
            return set_errno_error("ftruncate", errno);
        if (c->mapfile()) {
            c->map_bytes = fbytes;
            void *m = mmap(nullptr, fbytes, PROT_READ | PROT_WRITE, MAP_SHARED, c->fd, 0);
            if (m == MAP_FAILED) return set_errno_error("mmap", errno);
            c->map = static_cast<char *>(m);
            if ((e = cudaHostRegister(c->map, fbytes, cudaHostRegisterMapped | cudaHostRegisterPortable)) !=
                cudaSuccess) {
                munmap(c->map, fbytes);
                c->map = nullptr;
                return cuda_error(e, "cudaHostRegister(file mapping) — PCC_MAPFILE needs a DRAM-backed file "
                                     "(tmpfs, e.g. /dev/shm); use PWRITE mode (no MAPFILE) for disk files");
            }
            void *dp = nullptr;
            cudaHostGetDevicePointer(&dp, c->map, 0);
            c->map_dev = static_cast<char *>(dp);
        }
    }
    c->engine.reset(new CommitEngine());
    CommitEngine::Config ec;
    ec.fd = c->fd;
    ec.geom = c->sgeom;
    ec.n_inflight = c->cfg.max_inflight;
    ec.fsync = c->cfg.flags & PCC_FSYNC;
    ec.on_state = [c](uint64_t counter, int st) {
        // called under the engine lock; only touches the checkpoint table
        std::shared_ptr<Ckpt> ck;
        {
            std::lock_guard<std::mutex> lk(c->ck_mu);
            auto it = c->ckpts.find(counter);
            if (it == c->ckpts.end()) return;
            ck = it->second;
            ck->t_committed = c->now_us();
            ck->state.store(st);
        }
        c->ck_cv.notify_all();
    };
    if ((rc = c->engine->open(ec))) return rc;
    if ((e = cudaStreamSynchronize(c->pack_stream)) != cudaSuccess) return cuda_error(e, "register");
    c->registered = true;
    return PCC_OK;
}

static int dp_backpressure(pcc_ctx *c);

int pcc_checkpoint(pcc_ctx *c, uint64_t iter, void *train_stream, pcc_handle *out) {
    if (!c || !out) return set_error(PCC_EINVAL, "args");
    if (!c->registered) return set_error(PCC_ESTATE, "not registered");
    cudaStream_t ts = static_cast<cudaStream_t>(train_stream);
    gc_ckpts(c);
    auto ck = std::make_shared<Ckpt>();
    ck->t_call = c->now_us();
    // Listing 1 lines 3-11
    if (c->cfg.world > 1) {
        int rc = dp_backpressure(c);
        if (rc) return rc;
    }
    for (;;) {
        int rc = c->engine->begin(iter, &ck->t);
        if (rc == PCC_OK) break;
        if (rc != -PCC_EAGAIN) return rc;
        c->engine->wait_free(-1);  // the stall of L139 / Fig 6 when N checkpoints are in flight
    }
    cudaSetDevice(c->device);
    cudaEventCreateWithFlags(&ck->ev_train, cudaEventDisableTiming);
    cudaEventCreate(&ck->ev_begin);
    cudaEventCreate(&ck->ev_packed);
    cudaEventCreate(&ck->ev_landed);
    cudaEventCreate(&ck->ev_fin_k);
    cudaEventCreateWithFlags(&ck->ev_final, cudaEventDisableTiming);
    // the state as it is on the training stream now: K1 starts after this event
    cudaError_t e = cudaEventRecord(ck->ev_train, ts);
    if (e != cudaSuccess) {
        c->engine->fail(ck->t);
        destroy_ckpt_events(c, ck.get());
        return cuda_error(e, "event on the training stream");
    }
    ck->remaining = (uint32_t)c->n;
    ck->seq = ++c->issued_seq;
    {
        std::lock_guard<std::mutex> lk(c->ck_mu);
        c->ckpts[ck->t.counter] = ck;
    }
    c->guard_armed = true;
    if (!c->upfront()) c->jobs.push(ck);  // the orchestrator follows the K1 windows as they are published
    // K1: enqueued right here when nothing is queued ahead of it and the HBM ring already has room
    // for the whole slice (the usual case: the previous checkpoints drained within the interval);
    // otherwise the packer thread launches the windows as ring space frees.  Either way this call
    // never waits for ring space or for an earlier checkpoint's transfer.
    bool inline_pack = !c->zerocopy() && (int32_t)(c->packed_seq.load() - c->handed_seq) >= 0;
    if (inline_pack) {
        std::lock_guard<std::mutex> lk(c->ring_mu);
        inline_pack = c->ring_tail + c->ring_slots >= c->ring_head + c->n;
    }
    PCC_TRACE("ckpt %llu iter %llu seq %u: %s", (unsigned long long)ck->t.counter, (unsigned long long)iter, ck->seq,
              inline_pack ? "K1 inline" : "to the packer");
    if (inline_pack) {
        pack_one(c, ck);
    } else {
        c->handed_seq = ck->seq;
        c->packs.push(ck);
    }
    *out = ck->t.counter;
    return PCC_OK;
}

int pcc_guard(pcc_ctx *c, void *train_stream) {
    if (!c) return set_error(PCC_EINVAL, "ctx");
    if (!c->guard_armed) return PCC_OK;
    cudaStream_t ts = static_cast<cudaStream_t>(train_stream);
    const uint32_t want = c->issued_seq;
    // only when the packer thread still holds K1 windows of the newest checkpoint (ring space):
    // wait here, on the host and outside any CUDA call, until they are enqueued
    if ((int32_t)(c->packed_seq.load() - want) < 0) {
        PCC_TRACE("guard: seq %u waits for the packer", want);
        std::unique_lock<std::mutex> lk(c->pk_mu);
        c->pk_cv.wait(lk, [&] { return (int32_t)(c->packed_seq.load() - want) >= 0; });
        PCC_TRACE("guard: seq %u released", want);
    }
    cudaError_t e = cudaStreamWaitEvent(ts, c->ev_guard, 0);
    return e == cudaSuccess ? PCC_OK : cuda_error(e, "guard");
}

static std::shared_ptr<Ckpt> find_ck(pcc_ctx *c, pcc_handle h) {
    std::lock_guard<std::mutex> lk(c->ck_mu);
    auto it = c->ckpts.find(h);
    return it == c->ckpts.end() ? nullptr : it->second;
}

static bool terminal(int s) {
    return s == PCC_ST_LOCAL_COMMIT || s == PCC_ST_GLOBAL_COMMIT || s == PCC_ST_OBSOLETE || s == PCC_ST_FAILED;
}

// outcome of a pruned terminal handle (false: never issued)
static bool find_pruned(pcc_ctx *c, pcc_handle h, pcc_ctx::Outcome *o) {
    std::lock_guard<std::mutex> lk(c->ck_mu);
    auto it = c->pruned.find(h);
    if (it == c->pruned.end()) return false;
    *o = it->second;
    return true;
}

int pcc_poll(pcc_ctx *c, pcc_handle h, int *state) {
    if (!c || !state) return set_error(PCC_EINVAL, "args");
    auto ck = find_ck(c, h);
    if (!ck) {
        pcc_ctx::Outcome o;
        if (!find_pruned(c, h, &o)) return set_error(PCC_EINVAL, "unknown handle");
        int s = o.state;
        if (s == PCC_ST_LOCAL_COMMIT && c->cfg.world > 1) {
            uint64_t g = c->engine->global_iter();
            if (g != UINT64_MAX && g >= o.iter) s = PCC_ST_GLOBAL_COMMIT;
        }
        *state = s;
        return PCC_OK;
    }
    int s = ck->state.load();
    if (s == PCC_ST_PACKING && ck->packed_recorded.load() && cudaEventQuery(ck->ev_packed) == cudaSuccess)
        s = PCC_ST_PACKED;
    if (s == PCC_ST_LOCAL_COMMIT && c->cfg.world > 1) {
        uint64_t g = c->engine->global_iter();
        if (g != UINT64_MAX && g >= ck->t.iter) s = PCC_ST_GLOBAL_COMMIT;
    }
    *state = s;
    return PCC_OK;
}

int pcc_wait(pcc_ctx *c, pcc_handle h, int64_t timeout_us) {
    if (!c) return set_error(PCC_EINVAL, "ctx");
    auto ck = find_ck(c, h);
    if (!ck) {  // a pruned handle is terminal: its outcome
        pcc_ctx::Outcome o;
        if (!find_pruned(c, h, &o)) return set_error(PCC_EINVAL, "unknown handle");
        if (o.state == PCC_ST_FAILED) return o.err ? o.err : -PCC_EIO;
        return PCC_OK;
    }
    std::unique_lock<std::mutex> lk(c->ck_mu);
    auto pred = [&] { return terminal(ck->state.load()); };
    if (timeout_us < 0)
        c->ck_cv.wait(lk, pred);
    else if (!c->ck_cv.wait_for(lk, std::chrono::microseconds(timeout_us), pred))
        return set_error(PCC_ETIMEDOUT, "wait");
    if (ck->state.load() == PCC_ST_FAILED) return ck->err.load() ? ck->err.load() : -PCC_EIO;
    return PCC_OK;
}

int pcc_drain(pcc_ctx *c, int64_t timeout_us) {
    if (!c) return set_error(PCC_EINVAL, "ctx");
    std::unique_lock<std::mutex> lk(c->ck_mu);
    auto pred = [&] {
        for (auto &kv : c->ckpts)
            if (!terminal(kv.second->state.load())) return false;
        return true;
    };
    if (timeout_us < 0)
        c->ck_cv.wait(lk, pred);
    else if (!c->ck_cv.wait_for(lk, std::chrono::microseconds(timeout_us), pred))
        return set_error(PCC_ETIMEDOUT, "drain");
    return PCC_OK;
}

// In-place allreduce of int64 values over the library's NCCL communicator.  PCC_NOCOMM (one
// process measuring one rank's share alone) reduces over itself.
static int reduce_i64(pcc_ctx *c, int64_t *v, size_t n, NcclComm::Op op) {
    if (c->cfg.world == 1 || (c->cfg.flags & PCC_NOCOMM)) return PCC_OK;
    if (c->cfg.allreduce)
        return c->cfg.allreduce(c->cfg.coll_ctx, v, (uint32_t)n, op == NcclComm::kMax) ? set_error(PCC_ENCCL, "allreduce callback")
                                                                                      : PCC_OK;
    return c->nccl.allreduce_i64(v, n, op, c->red_dev, c->red_host, c->aux_stream);
}

// Collective backpressure (SURVEY §7 "hard parts"): a rank without a free slot cannot just
// block, because only a g-advance frees slots; every rank runs the same rounds of
// need = MAX(no free slot), g = MIN(L_r) until nobody needs.
static int dp_backpressure(pcc_ctx *c) {
    for (int round = 0;; ++round) {
        int64_t v[2] = {c->engine->has_free() ? 0 : 1, 0};
        int rc = reduce_i64(c, v, 1, NcclComm::kMax);
        if (rc) return rc;
        if (v[0] == 0) return PCC_OK;
        // let local persists progress, then advance g
        c->engine->wait_free(2000);
        uint64_t L = c->engine->local_latest();
        int64_t g[1] = {L == UINT64_MAX ? -1 : (int64_t)L};
        rc = reduce_i64(c, g, 1, NcclComm::kMin);
        if (rc) return rc;
        if (g[0] >= 0) c->engine->apply_global((uint64_t)g[0]);
    }
}

int pcc_commit(pcc_ctx *c, uint64_t *committed_iter) {
    if (!c) return set_error(PCC_EINVAL, "ctx");
    if (!c->registered) return set_error(PCC_ESTATE, "not registered");
    if (c->cfg.world == 1) {
        if (committed_iter) *committed_iter = c->engine->local_latest();
        return PCC_OK;
    }
    uint64_t L = c->engine->local_latest();
    int64_t g[1] = {L == UINT64_MAX ? -1 : (int64_t)L};
    int rc = reduce_i64(c, g, 1, NcclComm::kMin);
    if (rc) return rc;
    if (g[0] >= 0) rc = c->engine->apply_global((uint64_t)g[0]);
    if (committed_iter) *committed_iter = c->engine->global_iter();
    return rc;
}

int pcc_info(pcc_ctx *c, pcc_handle h, pcc_ckpt_info *info, uint32_t *crc, uint32_t crc_cap) {
    if (!c || !info) return set_error(PCC_EINVAL, "args");
    auto ck = find_ck(c, h);
    if (!ck) {
        pcc_ctx::Outcome o;
        return set_error(PCC_EINVAL, find_pruned(c, h, &o) ? "record pruned (pcc_info keeps the newest 64 terminal checkpoints)"
                                                          : "unknown handle");
    }
    std::memset(info, 0, sizeof(*info));
    info->iter = ck->t.iter;
    info->counter = ck->t.counter;
    info->slot = ck->t.slot;
    int st = 0;
    pcc_poll(c, h, &st);
    info->state = (uint32_t)st;
    info->n_chunks = (uint32_t)c->n;
    info->t_call_us = ck->t_call;
    if (terminal(ck->state.load()) || ck->state.load() == PCC_ST_PERSISTED) {
        info->digest = ck->digest;
        info->t_landed_us = ck->t_landed;
        info->t_persisted_us = ck->t_persisted;
        info->t_committed_us = ck->t_committed;
        info->pack_ms = ck->pack_ms;
        info->finalize_ms = ck->fin_ms;
        info->k1_busy_ms = ck->k1_busy_ms;
        info->snapshot_ms = ck->snap_ms;
        if (crc)
            for (uint32_t i = 0; i < crc_cap && i < ck->crc.size(); ++i) crc[i] = ck->crc[i];
    }
    return PCC_OK;
}

int pcc_geometry(pcc_ctx *c, uint64_t *n_chunks, uint64_t *first, uint64_t *count, uint64_t *end_bytes) {
    if (!c || !c->registered) return set_error(PCC_ESTATE, "not registered");
    if (n_chunks) *n_chunks = c->layout.C;
    if (first) *first = c->first;
    if (count) *count = c->n;
    if (end_bytes) *end_bytes = c->layout.end;
    return PCC_OK;
}

uint64_t pcc_kernel_launches(pcc_ctx *c) { return c ? c->launches.load() : 0; }

int pcc_nccl_unique_id(void *out128) {
    if (!out128) return set_error(PCC_EINVAL, "out");
    return pcc_nccl_unique_id_impl(out128);
}

int pcc_latest(const char *path, uint64_t *global_iter, uint64_t *local_iter) {
    if (!path) return set_error(PCC_EINVAL, "path");
    int fd = ::open(path, O_RDONLY);
    if (fd < 0) return set_error(PCC_ENOENT, "no file");
    alignas(4096) static thread_local uint8_t buf[kPage];
    PtrRecord best;
    for (int k = 0; k < 2; ++k) {
        if (::pread(fd, buf, kPage, k * kPage) != (ssize_t)kPage) continue;
        PtrRecord r = decode_ptr(buf);
        if (r.valid && (!best.valid || r.seq > best.seq)) best = r;
    }
    ::close(fd);
    if (!best.valid) return set_error(PCC_ENOENT, "no valid pointer record");
    if (global_iter) *global_iter = best.global_iter;
    if (local_iter) *local_iter = best.local_iter;
    return PCC_OK;
}

int pcc_close(pcc_ctx *c) {
    if (!c) return PCC_OK;
    pcc_drain(c, -1);
    c->packs.close();
    if (c->packer.joinable()) c->packer.join();
    c->jobs.close();
    if (c->orchestrator.joinable()) c->orchestrator.join();
    c->tasks.close();
    for (auto &t : c->persisters)
        if (t.joinable()) t.join();
    cudaSetDevice(c->device);
    cudaDeviceSynchronize();
    {
        std::lock_guard<std::mutex> lk(c->ck_mu);
        for (auto &kv : c->ckpts) destroy_ckpt_events(c, kv.second.get());
        c->ckpts.clear();
        c->pruned.clear();
    }
    free_registration(c);
    for (auto e : c->evpool) cudaEventDestroy(e);
    cudaEventDestroy(c->ev_guard);
    cudaStreamDestroy(c->pack_stream);
    cudaStreamDestroy(c->copy_stream);
    cudaStreamDestroy(c->aux_stream);
    c->nccl.destroy();
    if (c->red_dev) cudaFree(c->red_dev);
    if (c->red_host) cudaFreeHost(c->red_host);
    if (c->fd >= 0) ::close(c->fd);
    delete c;
    return PCC_OK;
}

}  // extern "C"

// ------------------------------------------------------------------------- restore
namespace {

int pread_full(int fd, char *p, uint64_t n, uint64_t off) {
    while (n) {
        ssize_t r = ::pread(fd, p, n, (off_t)off);
        if (r < 0) {
            if (errno == EINTR) continue;
            return set_errno_error("pread chunk", errno);
        }
        if (r == 0) return set_error(PCC_EIO, "short read (truncated file)");
        p += r;
        n -= (uint64_t)r;
        off += (uint64_t)r;
    }
    return PCC_OK;
}

// K2 over this rank's slice of the checkpoint in `slot`: H2D into the HBM ring, verify every
// chunk's CRC32C against the header table while scattering into the registered tensors.
int verify_scatter(pcc_ctx *c, uint32_t slot, std::vector<uint32_t> *bad_out) {
    const uint64_t n = c->n, cb = c->cb();
    bad_out->clear();
    if (n == 0) return PCC_OK;
    const uint64_t H = header_bytes(n);
    uint8_t *hdr = static_cast<uint8_t *>(std::aligned_alloc(kPage, H));
    int rc = pread_full(c->fd, reinterpret_cast<char *>(hdr), H, slot_offset(slot, n, cb));
    if (rc) {
        std::free(hdr);
        return rc;
    }
    HeaderView v = decode_header(hdr, c->sgeom, slot);
    if (!v.ok || !v.layout_ok) {
        std::free(hdr);
        return set_error(PCC_ELAYOUT, "slot header");
    }
    // restore runs with nothing in flight (pcc_restore drained): slot 0's scratch is free
    uint32_t *tile = c->tile_crc_dev[0], *crc = c->crc_dev[0], *scr = c->scratch_dev[0];
    uint32_t *expect = c->rexpect_dev, *bad = c->rbad_dev;
    cudaMemcpyAsync(expect, v.crc, n * 4, cudaMemcpyHostToDevice, c->pack_stream);
    cudaMemsetAsync(scr, 0, 16, c->pack_stream);
    const uint32_t digest = v.digest;
    cudaStreamSynchronize(c->pack_stream);  // hdr (the expect source) is freed below
    std::free(hdr);
    PCC_TRACE("restore: slot %u header ok t=%.0f us", slot, c->now_us());
    cudaError_t e = cudaSuccess;
    char *ring = c->ring;
    uint64_t R = c->ring_slots;
    bool own_ring = false;
    if (!ring) {  // zero-copy mode keeps no HBM ring
        R = std::min<uint64_t>(n, 16);
        if ((e = cudaMalloc(&ring, R * cb))) return cuda_error(e, "restore ring");
        own_ring = true;
    }
    SnapParams P{};
    P.rows = c->rows_dev;
    P.row_begin = c->row_begin_dev;
    P.tile_rows = c->tile_rows_dev;
    P.chunk_bytes = cb;
    P.tpc = c->geom.tpc;
    P.ring_base = ring;
    P.ring_slots = R;
    P.tile_crc = tile;
    P.tables = c->tables;
    P.consts = c->consts;
    // batches: H2D of batch b+1 overlaps K2 of batch b when the ring holds the whole slice
    const bool whole = R >= n;
    const uint64_t batch = whole ? std::max<uint64_t>(1, (n + 3) / 4) : R;
    cudaEvent_t ev_copy = get_event(c), ev_k2 = get_event(c);
    // timing (pcc_restore_stats): H2D span on the copy stream, each K2 launch and the finalize
    cudaEvent_t t_h2d[2], t_fin[2];
    for (auto *e2 : {t_h2d, t_fin}) {
        cudaEventCreate(&e2[0]);
        cudaEventCreate(&e2[1]);
    }
    std::vector<std::pair<cudaEvent_t, cudaEvent_t>> t_k2;
    double read_ms = 0;
    cudaEventRecord(t_h2d[0], c->copy_stream);
    const uint64_t data0 = c->slot_data_off(slot);
    for (uint64_t j0 = 0; j0 < n && rc == PCC_OK; j0 += batch) {
        const uint64_t k = std::min<uint64_t>(batch, n - j0);
        if (!whole && j0) cudaStreamWaitEvent(c->copy_stream, ev_k2, 0);  // ring slots reused
        for (uint64_t i = 0; i < k && rc == PCC_OK; ++i) {
            const uint64_t j = j0 + i;
            char *dst = ring + (whole ? j : i) * cb;
            if (c->mapfile()) {
                cudaMemcpyAsync(dst, c->map + data0 + j * cb, cb, cudaMemcpyHostToDevice, c->copy_stream);
            } else {  // pread into a pinned staging slot, then H2D (the slot is reused after the copy)
                char *st = c->staging + (i % c->staging_slots) * cb;
                if (i >= c->staging_slots) cudaStreamSynchronize(c->copy_stream);
                const auto tr0 = std::chrono::steady_clock::now();
                rc = pread_full(c->fd, st, cb, data0 + j * cb);
                read_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - tr0).count();
                if (rc == PCC_OK) cudaMemcpyAsync(dst, st, cb, cudaMemcpyHostToDevice, c->copy_stream);
            }
        }
        if (!c->mapfile()) cudaStreamSynchronize(c->copy_stream);  // staging reused next batch
        cudaEventRecord(ev_copy, c->copy_stream);
        cudaStreamWaitEvent(c->pack_stream, ev_copy, 0);
        P.first = (uint32_t)j0;
        P.count = (uint32_t)k;
        P.ring_head = whole ? 0 : (R - j0 % R) % R;
        std::pair<cudaEvent_t, cudaEvent_t> tk;
        cudaEventCreate(&tk.first);
        cudaEventCreate(&tk.second);
        t_k2.push_back(tk);
        cudaEventRecord(tk.first, c->pack_stream);
        if ((e = launch_unpack(P, snapshot_grid(c->device, (uint32_t)(k * P.tpc), 0, false), c->pack_stream)))
            rc = cuda_error(e, "K2");
        cudaEventRecord(tk.second, c->pack_stream);
        c->launches += 1;
        cudaEventRecord(ev_k2, c->pack_stream);
    }
    cudaEventRecord(t_h2d[1], c->copy_stream);
    PCC_TRACE("restore: copies + K2 issued t=%.0f us", c->now_us());
    FinalizeParams F{};
    F.tile_crc = tile;
    F.tables = c->tables;
    F.n = (uint32_t)n;
    F.tpc = c->geom.tpc;
    F.tile_shift = c->geom.tile_shift;
    F.chunk_shift = c->geom.chunk_shift;
    F.ff = c->geom.ff;
    F.crc_out = crc;
    F.expect = expect;
    F.bad = bad;
    F.scratch = scr;
    cudaEventRecord(t_fin[0], c->pack_stream);
    if (rc == PCC_OK && (e = launch_finalize(F, c->pack_stream))) rc = cuda_error(e, "finalize");
    cudaEventRecord(t_fin[1], c->pack_stream);
    c->launches += kFinalizeLaunches;
    std::vector<uint32_t> flags(n);
    uint32_t sc[4] = {0, 0, 0, 0};
    if (rc == PCC_OK) {
        cudaMemcpyAsync(flags.data(), bad, n * 4, cudaMemcpyDeviceToHost, c->pack_stream);
        cudaMemcpyAsync(sc, scr, 16, cudaMemcpyDeviceToHost, c->pack_stream);
        if ((e = cudaStreamSynchronize(c->pack_stream))) rc = cuda_error(e, "restore sync");
    }
    cudaStreamSynchronize(c->copy_stream);
    PCC_TRACE("restore: verified t=%.0f us", c->now_us());
    {
        pcc_restore_info &st = c->rstats;
        float ms = 0;
        st.attempts += 1;
        st.bytes += n * cb;
        st.read_ms += (float)read_ms;
        if (cudaEventElapsedTime(&ms, t_h2d[0], t_h2d[1]) == cudaSuccess) st.h2d_ms += ms;
        if (cudaEventElapsedTime(&ms, t_fin[0], t_fin[1]) == cudaSuccess) st.finalize_ms += ms;
        for (auto &tk : t_k2) {
            if (cudaEventElapsedTime(&ms, tk.first, tk.second) == cudaSuccess) st.k2_ms += ms;
            cudaEventDestroy(tk.first);
            cudaEventDestroy(tk.second);
        }
        for (auto *e2 : {t_h2d, t_fin}) {
            cudaEventDestroy(e2[0]);
            cudaEventDestroy(e2[1]);
        }
    }
    put_event(c, ev_copy);
    put_event(c, ev_k2);
    if (own_ring) cudaFree(ring);
    if (rc) return rc;
    for (uint64_t j = 0; j < n; ++j)
        if (flags[j]) bad_out->push_back((uint32_t)(c->first + j));
    if (!bad_out->empty()) return set_error(PCC_ECORRUPT, "chunk CRC32C mismatch");
    if (sc[3] != digest) return set_error(PCC_ECORRUPT, "slice digest mismatch");
    return PCC_OK;
}

// allgather of device buffers: NCCL on the library's communicator, or the caller's host
// callback (staged through pinned host memory)
static int allgather_dev(pcc_ctx *c, const void *send, void *recv, size_t bytes, cudaStream_t s) {
    if (!c->cfg.allgather) return c->nccl.allgather(send, recv, bytes, s);
    const size_t W = (size_t)c->cfg.world;
    char *hs = nullptr, *hr = nullptr;
    cudaError_t e;
    const size_t rbytes = W * bytes;
    if ((e = cudaMallocHost(&hs, bytes ? bytes : 1)) || (e = cudaMallocHost(&hr, rbytes ? rbytes : 1))) {
        cudaFreeHost(hs);
        return cuda_error(e, "allgather staging");
    }
    cudaMemcpyAsync(hs, send, bytes, cudaMemcpyDeviceToHost, s);
    int rc = PCC_OK;
    if ((e = cudaStreamSynchronize(s))) rc = cuda_error(e, "allgather d2h");
    if (rc == PCC_OK && c->cfg.allgather(c->cfg.coll_ctx, hs, hr, bytes)) rc = set_error(PCC_ENCCL, "allgather callback");
    PCC_TRACE("allgather: %zu B/rank, sent[0] %08x recv[0] %08x recv[last rank] %08x", bytes,
              bytes >= 4 ? *reinterpret_cast<uint32_t *>(hs) : 0u, bytes >= 4 ? *reinterpret_cast<uint32_t *>(hr) : 0u,
              bytes >= 4 ? *reinterpret_cast<uint32_t *>(hr + (W - 1) * bytes) : 0u);
    if (rc == PCC_OK) {
        cudaMemcpyAsync(recv, hr, W * bytes, cudaMemcpyHostToDevice, s);
        if ((e = cudaStreamSynchronize(s))) rc = cuda_error(e, "allgather h2d");
    }
    cudaFreeHost(hs);
    cudaFreeHost(hr);
    return rc;
}

// C3 of SURVEY §2.3: after every rank verified (and scattered) its own slice of iter g, the
// verified packed chunks cross NVLink with ncclAllGather in groups of G chunks per rank, and
// each rank K2-verifies + scatters the other ranks' chunks into its registered tensors (the
// CRC tables travel too, so a transfer fault is caught).  Uneven slices are padded to
// n_max = ceil(C / W) chunks per rank.
int dp_fanout(pcc_ctx *c, uint32_t slot) {
    const uint64_t cb = c->cb(), C = c->layout.C;
    const uint32_t W = (uint32_t)c->cfg.world, me = (uint32_t)c->cfg.rank;
    const uint64_t n_max = (C + W - 1) / W;
    if (C == 0) return PCC_OK;
    // full-image segment table (every chunk, not just this rank's slice)
    HostLayout full;
    if (build_layout(c->tensors.data(), (uint32_t)c->tensors.size(), c->cfg.align, cb, 0, -1, &full))
        return set_error(PCC_EINVAL, "full layout");
    build_tile_rows(&full, cb, kTile);
    SegRow *rows = nullptr;
    uint32_t *rb = nullptr, *tile = nullptr, *crc_mine = nullptr, *crc_all = nullptr, *crc_out = nullptr, *bad = nullptr,
             *scr = nullptr;
    uint2 *trows = nullptr;
    char *send = nullptr, *recv = nullptr;
    DevGeometry g2;
    cudaError_t e = cudaSuccess;
    int rc = PCC_OK;
    auto done = [&](int r) {
        cudaFree(rows); cudaFree(rb); cudaFree(tile); cudaFree(crc_mine); cudaFree(crc_all); cudaFree(crc_out);
        cudaFree(bad); cudaFree(scr); cudaFree(trows); cudaFree(send); cudaFree(recv);
        free_geometry(&g2);
        return r;
    };
    // group size: bounded by 4 GiB of receive buffer
    uint64_t G = std::max<uint64_t>(1, std::min<uint64_t>(n_max, (4ull << 30) / (W * cb)));
    const uint64_t nsub = tile_crc_words(c->geom.tpc);  // lane-CRC words per chunk
    if ((e = cudaMalloc(&rows, std::max<size_t>(1, full.rows.size()) * sizeof(SegRow))) ||
        (e = cudaMalloc(&rb, (C + 1) * 4)) || (e = cudaMalloc(&trows, std::max<size_t>(2, full.tile_rows.size()) * 4)) ||
        (e = cudaMalloc(&tile, C * nsub * 4)) || (e = cudaMalloc(&crc_mine, n_max * 4)) ||
        (e = cudaMalloc(&crc_all, W * n_max * 4)) || (e = cudaMalloc(&crc_out, C * 4)) || (e = cudaMalloc(&bad, C * 4)) ||
        (e = cudaMalloc(&scr, 16 * W)) || (e = cudaMalloc(&send, G * cb)) || (e = cudaMalloc(&recv, W * G * cb)))
        return done(cuda_error(e, "fanout buffers"));
    cudaStream_t ps = c->pack_stream;  // uploads ordered before the K2 launches on the same stream
    if (!full.rows.empty())
        cudaMemcpyAsync(rows, full.rows.data(), full.rows.size() * sizeof(SegRow), cudaMemcpyHostToDevice, ps);
    cudaMemcpyAsync(rb, full.row_begin.data(), (C + 1) * 4, cudaMemcpyHostToDevice, ps);
    if (!full.tile_rows.empty())
        cudaMemcpyAsync(trows, full.tile_rows.data(), full.tile_rows.size() * 4, cudaMemcpyHostToDevice, ps);
    if ((e = setup_geometry(&g2, cb, (uint32_t)n_max, c->pack_stream))) return done(cuda_error(e, "fanout geometry"));
    // this rank's CRC table (from its slot header) -> allgather
    {
        const uint64_t H = header_bytes(c->n);
        uint8_t *hdr = static_cast<uint8_t *>(std::aligned_alloc(kPage, H));
        rc = pread_full(c->fd, reinterpret_cast<char *>(hdr), H, slot_offset(slot, c->n, cb));
        std::vector<uint32_t> mine(n_max, 0);
        if (rc == PCC_OK) std::memcpy(mine.data(), hdr + 96, c->n * 4);
        std::free(hdr);
        if (rc) return done(rc);
        cudaMemcpyAsync(crc_mine, mine.data(), n_max * 4, cudaMemcpyHostToDevice, c->pack_stream);
        cudaStreamSynchronize(c->pack_stream);  // `mine` dies at the end of this scope
        PCC_TRACE("fanout: rank %u slot %u n %llu crc[0] %08x crc[n-1] %08x", me, slot, (unsigned long long)c->n,
                  mine[0], c->n ? mine[c->n - 1] : 0u);
    }
    if ((rc = allgather_dev(c, crc_mine, crc_all, n_max * 4, c->pack_stream))) return done(rc);
    const uint64_t data0 = c->slot_data_off(slot);
    std::vector<uint64_t> first_q(W), n_q(W);
    for (uint32_t q = 0; q < W; ++q) slice_of(C, q, W, &first_q[q], &n_q[q]);
    uint32_t launches = 0;
    for (uint64_t k0 = 0; k0 < n_max && rc == PCC_OK; k0 += G) {
        const uint64_t mine_k = n_q[me] > k0 ? std::min<uint64_t>(G, n_q[me] - k0) : 0;
        for (uint64_t i = 0; i < mine_k && rc == PCC_OK; ++i) {  // own verified chunks -> send buffer
            const char *src;
            if (c->mapfile()) {
                src = c->map + data0 + (k0 + i) * cb;
            } else {
                char *st = c->staging + (i % c->staging_slots) * cb;
                if (i >= c->staging_slots) cudaStreamSynchronize(c->copy_stream);
                rc = pread_full(c->fd, st, cb, data0 + (k0 + i) * cb);
                src = st;
            }
            if (rc == PCC_OK) cudaMemcpyAsync(send + i * cb, src, cb, cudaMemcpyHostToDevice, c->copy_stream);
        }
        cudaStreamSynchronize(c->copy_stream);
        if (rc) break;
        if ((rc = allgather_dev(c, send, recv, G * cb, c->pack_stream))) break;
        for (uint32_t q = 0; q < W; ++q) {
            if (q == me) continue;
            const uint64_t cnt = n_q[q] > k0 ? std::min<uint64_t>(G, n_q[q] - k0) : 0;
            if (!cnt) continue;
            const uint64_t j0 = first_q[q] + k0;  // global chunk index
            SnapParams P{};
            P.rows = rows;
            P.row_begin = rb;
            P.tile_rows = trows;
            P.chunk_bytes = cb;
            P.first = (uint32_t)j0;
            P.count = (uint32_t)cnt;
            P.tpc = c->geom.tpc;
            P.ring_base = recv + (uint64_t)q * G * cb;
            P.ring_slots = 1ull << 40;
            P.ring_head = P.ring_slots - j0;
            P.tile_crc = tile;
            P.tables = c->tables;
            P.consts = c->consts;
            if ((e = launch_unpack(P, snapshot_grid(c->device, (uint32_t)(cnt * P.tpc), 0, false), c->pack_stream))) {
                rc = cuda_error(e, "fanout K2");
                break;
            }
            FinalizeParams F{};
            F.tile_crc = tile + j0 * nsub;
            F.tables = c->tables;
            F.n = (uint32_t)cnt;
            F.tpc = c->geom.tpc;
            F.tile_shift = g2.tile_shift;
            F.chunk_shift = g2.chunk_shift;
            F.ff = g2.ff;
            F.crc_out = crc_out + j0;
            F.expect = crc_all + (uint64_t)q * n_max + k0;
            F.bad = bad + j0;
            F.scratch = scr + 4 * q;
            cudaMemsetAsync(F.scratch, 0, 16, c->pack_stream);
            if ((e = launch_finalize(F, c->pack_stream))) {
                rc = cuda_error(e, "fanout finalize");
                break;
            }
            launches += 1 + kFinalizeLaunches;
        }
        if ((e = cudaStreamSynchronize(c->pack_stream))) rc = cuda_error(e, "fanout sync");  // recv reused next group
        std::vector<uint32_t> sc(4 * W);
        cudaMemcpyAsync(sc.data(), scr, 16 * W, cudaMemcpyDeviceToHost, c->pack_stream);
        cudaStreamSynchronize(c->pack_stream);
        for (uint32_t q = 0; q < W && rc == PCC_OK; ++q) {
            if (!sc[4 * q + 2]) continue;
            if (trace_on()) {
                const uint64_t cnt = n_q[q] > k0 ? std::min<uint64_t>(G, n_q[q] - k0) : 0;
                std::vector<uint32_t> got(cnt), exp(cnt);
                cudaMemcpy(got.data(), crc_out + first_q[q] + k0, cnt * 4, cudaMemcpyDeviceToHost);
                cudaMemcpy(exp.data(), crc_all + q * n_max + k0, cnt * 4, cudaMemcpyDeviceToHost);
                for (uint64_t i = 0; i < cnt; ++i)
                    PCC_TRACE("fanout: rank %u chunk %llu crc %08x expect %08x", q,
                              (unsigned long long)(first_q[q] + k0 + i), got[i], exp[i]);
            }
            rc = set_error(PCC_ECORRUPT, "chunk corrupted in the NVLink fan-out");
        }
    }
    c->launches += launches;
    return done(rc);
}

}  // namespace

extern "C" int pcc_restore(pcc_ctx *c, uint64_t want_iter, uint32_t flags, uint64_t *restored_iter,
                           uint32_t *bad_chunks, uint32_t bad_cap, uint32_t *n_bad) {
    if (!c) return set_error(PCC_EINVAL, "ctx");
    if (!c->registered) return set_error(PCC_ESTATE, "not registered");
    if (n_bad) *n_bad = 0;
    if (c->fd < 0) return set_error(PCC_ENOENT, "no file (NULLSINK)");
    pcc_drain(c, -1);
    cudaSetDevice(c->device);
    const auto t_start = std::chrono::steady_clock::now();
    c->rstats = pcc_restore_info{};
    PCC_TRACE("restore: start t=%.0f us", c->now_us());
    SlotScan S;
    int rc = scan_rank_file(c->fd, c->sgeom, c->n_slots, &S);
    if (rc) return rc;
    PCC_TRACE("restore: scanned t=%.0f us", c->now_us());
    RestoreOps ops;
    if (c->cfg.world == 1) {
        ops.reduce = [](int64_t *, bool) { return PCC_OK; };
    } else {
        ops.reduce = [c](int64_t *v, bool is_max) { return reduce_i64(c, v, 1, is_max ? NcclComm::kMax : NcclComm::kMin); };
        if (!(c->cfg.flags & (PCC_NOCOMM | PCC_SHARDED)))
            ops.fanout = [c](uint64_t, uint32_t slot) {
                const auto t0 = std::chrono::steady_clock::now();
                int r = dp_fanout(c, slot);
                c->rstats.fanout_ms +=
                    (float)std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
                return r;
            };
    }
    ops.verify = [c](uint64_t, uint32_t slot, std::vector<uint32_t> *bad) { return verify_scatter(c, slot, bad); };
    uint64_t it = 0;
    std::vector<uint32_t> bad;
    rc = restore_agree(S, want_iter, flags, ops, &it, &bad);
    if (n_bad) *n_bad = (uint32_t)bad.size();
    for (size_t i = 0; i < bad.size() && i < bad_cap && bad_chunks; ++i) bad_chunks[i] = bad[i];
    if (rc == PCC_OK && restored_iter) *restored_iter = it;
    c->rstats.total_ms =
        (float)std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t_start).count();
    return rc;
}

extern "C" int pcc_restore_stats(pcc_ctx *c, pcc_restore_info *out) {
    if (!c || !out) return set_error(PCC_EINVAL, "args");
    *out = c->rstats;
    return PCC_OK;
}
