// commit.hpp — the crash-consistent metadata commit.
//
// Listing 1 (§4.1) on a file instead of PMEM:
//   begin()     lines 3-11: sample CHECK_ADDR, atomic_add(g_counter), free_space.deq()
//   filling()   reading R18: the reused slot's header becomes FILLING (+fdatasync) before data
//   complete()  lines 16-34: header COMPLETE (+fsync) = "persist the checkpoint", then the CAS
//               loop on CHECK_ADDR; BARRIER(CHECK_ADDR) = a monotone write of one of the two
//               CRC-protected pointer records (+fsync) (R7); enq the freed slot
// Data-parallel training (L152 §3.1, L283 §4.1) under readings R8, R9, R20: local commits
// in counter order, the caller reduces L_r = local_latest() with MIN across ranks and
// hands g to apply_global(), which writes global_iter and frees slots holding iters < g.
//
// Pure host C++ (no CUDA): the runtime drives it from its persist threads, and
// include/pccheck_host.h exposes it so CPU tests can drive it under gloo.
#pragma once
#include <atomic>
#include <condition_variable>
#include <cstdint>
#include <deque>
#include <functional>
#include <map>
#include <memory>
#include <mutex>
#include <vector>

#include "format.hpp"

namespace pcc {

struct CheckMeta {  // Listing 1 line 16: {data_location, counter} (+ iter)
    uint32_t data_location;
    uint64_t counter;
    uint64_t iter;
};

struct Ticket {
    uint64_t iter = 0, counter = 0;
    uint32_t slot = 0;
    CheckMeta *last_check = nullptr;  // line 3
};

class CommitEngine {
   public:
    struct Config {
        int fd = -1;                 // -1: no file (NULLSINK): in-memory commit only
        SlotGeom geom{};
        uint32_t n_inflight = 1;     // N; the file has N+1 slots
        bool fsync = false;
        // world > 1: called (under the engine's lock) for every checkpoint whose in-order
        // local commit happened, with PCC_ST_LOCAL_COMMIT or PCC_ST_FAILED
        std::function<void(uint64_t counter, int state)> on_state;
    };

    int open(const Config &c);       // reads existing pointer records / headers (resume)
    // lines 3-11.  -PCC_EAGAIN: no free slot (the caller spins / runs the DP backpressure loop)
    int begin(uint64_t iter, Ticket *t);
    int filling(const Ticket &t);
    // lines 16-34 after every chunk of t is durable.  *state = PCC_ST_LOCAL_COMMIT or OBSOLETE.
    int complete(const Ticket &t, const uint32_t *crc, uint32_t digest, int *state);
    void fail(const Ticket &t);      // I/O / CUDA error: pointer untouched, slot recycled
    uint64_t local_latest();         // L_r (PCC_NONE if nothing committed)
    uint64_t global_iter();
    int apply_global(uint64_t g);    // W > 1
    bool has_free();
    uint32_t free_count();
    bool wait_free(int64_t timeout_us);  // waits for a free slot (W = 1 stall, line 8-11)
    uint64_t last_iter() const { return last_iter_; }
    uint32_t n_slots() const { return n_slots_; }
    const SlotGeom &geom() const { return cfg_.geom; }
    int fd() const { return cfg_.fd; }
    int write_header(uint32_t slot, uint32_t state, uint64_t iter, uint64_t counter, uint32_t digest,
                     const uint32_t *crc);
    // held slots (iter -> slot) for tests / restore bookkeeping
    std::map<uint64_t, uint32_t> held();

   private:
    int write_pointer_locked();      // BARRIER(CHECK_ADDR): the current max, monotone seq
    int drain_locked(uint64_t self_counter, int *state);  // in-order DP commits (holds dp_mu_)
    void enq(uint32_t slot);

    Config cfg_;
    uint32_t n_slots_ = 0;
    std::mutex q_mu_;
    std::condition_variable q_cv_;
    std::deque<uint32_t> free_space_;          // the free-slot Queue (D4)
    std::atomic<CheckMeta *> check_addr_{nullptr};  // CHECK_ADDR (D5)
    std::atomic<uint64_t> g_counter_{0};       // D1
    std::deque<std::unique_ptr<CheckMeta>> metas_;
    std::mutex meta_mu_;
    std::mutex ptr_mu_;                        // serialises pointer-record writes
    uint64_t seq_ = 0;
    uint64_t last_iter_ = UINT64_MAX;          // R5: iters strictly increase
    // DP (world > 1)
    std::mutex dp_mu_;
    std::map<uint64_t, std::pair<Ticket, bool>> pending_;  // counter -> (ticket, ok) awaiting in-order commit
    uint64_t next_commit_ = 0;
    std::map<uint64_t, uint32_t> held_;        // committed iter -> slot, not yet freed
    uint64_t L_ = UINT64_MAX, g_ = UINT64_MAX;
    CheckMeta latest_local_{0, 0, 0};
    bool have_local_ = false;
    uint8_t *hdr_buf_ = nullptr;               // 4 KiB-aligned scratch (O_DIRECT-safe)
    uint8_t *ptr_buf_ = nullptr;
    std::mutex hdr_mu_;

   public:
    ~CommitEngine();
};

// ------------------------------------------------------------------ restore agreement
// What a rank file holds (FORMAT.md): the valid pointer record with the largest seq and the
// iters of COMPLETE, CRC-valid headers (split by whether they match the registration).
struct SlotScan {
    std::map<uint64_t, uint32_t> complete;    // iter -> slot
    std::map<uint64_t, uint32_t> bad_layout;  // iter -> slot, header valid but another registration
    PtrRecord best;
};
int scan_rank_file(int fd, const SlotGeom &g, uint32_t n_slots, SlotScan *S);

// The restore protocol of L287 (§4.2) with verification, for W ranks:
// every rank runs the same control flow, steered only by reduced values, so the collectives
// match.  W = 1 passes an identity reducer.
//   g = MAX_r(global_iter of the rank's best record)   (or want_iter)
//   loop: all = MIN_r(g is held COMPLETE here); if all: verify own slice (K2), err = MAX_r(err);
//         no error -> fanout (W > 1) -> done;  else (PCC_FALLBACK) g = MIN_r(max{h held < g})
struct RestoreOps {
    std::function<int(int64_t *v, bool is_max)> reduce;                           // in place, 1 value
    std::function<int(uint64_t iter, uint32_t slot, std::vector<uint32_t> *bad)> verify;  // own slice
    std::function<int(uint64_t iter, uint32_t slot)> fanout;                     // W > 1 (may be empty)
};
// Returns PCC_OK with *restored set, or the first candidate's error; *bad_first receives
// this rank's failing chunk indices of that first rejected candidate.
int restore_agree(const SlotScan &S, uint64_t want_iter, uint32_t flags, const RestoreOps &ops, uint64_t *restored,
                  std::vector<uint32_t> *bad_first);

}  // namespace pcc
