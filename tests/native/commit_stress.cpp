// commit_stress.cpp — the commit engine (include/pccheck_host.h) under concurrency, built with
// -fsanitize=thread by tests/test_commit_stress.py ("free-queue / CAS stress under
// -fsanitize=thread").  Test infrastructure only.
//
// Listing 1 (§4.1) is lock-free with N writer threads; the invariants of
// L229 checked here while they race:
//   * the pointer (local_latest) never moves backwards and only ever names a checkpoint whose
//     complete() already started (its header was written before the pointer, FORMAT.md);
//   * at most N+1 slots: free + held + in flight <= N+1, every begin eventually gets a slot;
//   * W > 1 (R20): with in-order local commits, every rank still holds g = MIN_r(L_r) after
//     apply_global(g) — the slot restore needs is never freed.
// Usage: commit_stress <dir> <N> <world> <checkpoints_per_rank> <seed> <layout_crc>
// (one registered tensor of kChunks*kCB bytes; layout_crc from oracle.layout_crc)
// Prints "OK <latest iter of rank 0> <global iter>" on success, "FAIL <what>" and exit 1 otherwise.
#include <nmmintrin.h>
#include <unistd.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <random>
#include <string>
#include <thread>
#include <vector>

#include "../../include/pccheck_host.h"

static std::atomic<bool> g_fail{false};
static void fail(const char *what, long a = 0, long b = 0) {
    if (!g_fail.exchange(true)) std::printf("FAIL %s (%ld, %ld)\n", what, a, b);
}

static const uint64_t kCB = 4096;
static const uint32_t kChunks = 6;  // whole image; each rank holds its slice
static const uint64_t kNone = UINT64_MAX;

// CRC32C of `n` zero bytes with the SSE4.2 instruction (the slot data is never written: the
// file is sparse, so every chunk reads back as zeros)
static uint32_t crc_zeros(uint64_t n) {
    uint64_t c = 0xFFFFFFFFu;
    for (uint64_t i = 0; i < n; i += 8) c = _mm_crc32_u64(c, 0);
    return (uint32_t)c ^ 0xFFFFFFFFu;
}

struct Rank {
    pcc_host *h = nullptr;
    uint32_t n = 0, n_slots = 0;
    std::mutex order_mu;          // begin() calls in strictly increasing iter (R5)
    uint64_t next_iter = 1;
    std::atomic<int> inflight{0};
    std::atomic<uint64_t> max_started{0};  // largest iter whose complete() has started
};

int main(int argc, char **argv) {
    if (argc < 7) return 2;
    const std::string dir = argv[1];
    const uint32_t N = (uint32_t)atoi(argv[2]), W = (uint32_t)atoi(argv[3]);
    const int per_rank = atoi(argv[4]);
    const unsigned seed = (unsigned)atoi(argv[5]);
    const uint32_t layout_crc = (uint32_t)strtoul(argv[6], nullptr, 0);
    std::vector<Rank> ranks(W);
    for (uint32_t r = 0; r < W; ++r) {
        std::string path = dir + "/rank" + std::to_string(r) + ".pcc";
        pcc_host_config cfg{};
        cfg.path = path.c_str();
        cfg.chunk_bytes = kCB;
        cfg.max_inflight = N;
        cfg.rank = r;
        cfg.world = W;
        cfg.total_chunks = kChunks;
        cfg.n_tensors = 1;
        cfg.align = 256;
        cfg.layout_crc = layout_crc;
        if (pcc_host_open(&cfg, &ranks[r].h) != 0) return fail("open"), 1;
        pcc_host_geometry(ranks[r].h, nullptr, &ranks[r].n, &ranks[r].n_slots);
    }
    std::atomic<int> done_writers{0};
    const int writers_per_rank = (int)N + 1;  // one more writer than in-flight slots: begin must stall
    std::vector<std::thread> th;
    for (uint32_t r = 0; r < W; ++r) {
        for (int w = 0; w < writers_per_rank; ++w) {
            th.emplace_back([&, r, w] {
                Rank &R = ranks[r];
                std::mt19937 rng(seed * 7919u + r * 131u + (unsigned)w);
                const uint32_t crc0 = crc_zeros(kCB), dig = crc_zeros(kCB * R.n);
                std::vector<uint32_t> crc(R.n, crc0);
                while (!g_fail) {
                    uint64_t counter = 0, iter = 0;
                    uint32_t slot = 0;
                    {
                        std::lock_guard<std::mutex> lk(R.order_mu);
                        iter = R.next_iter;
                        if ((int)iter > per_rank) break;
                        int rc = pcc_host_begin(R.h, iter, &counter, &slot);
                        if (rc == -PCC_EAGAIN) {  // all N+1 slots held: the paper's stall
                            std::this_thread::yield();
                            continue;
                        }
                        if (rc) return fail("begin", rc, (long)iter);
                        ++R.next_iter;
                    }
                    if (slot >= R.n_slots) return fail("slot out of range", slot);
                    int infl = ++R.inflight;
                    if ((uint32_t)infl > R.n_slots) fail("more in flight than slots", infl);
                    if (pcc_host_filling(R.h, counter)) return fail("filling");
                    std::this_thread::sleep_for(std::chrono::microseconds(rng() % 400));  // "persist"
                    uint64_t prev = R.max_started.load();
                    while (prev < iter && !R.max_started.compare_exchange_weak(prev, iter)) {
                    }
                    int st = 0;
                    if (pcc_host_complete(R.h, counter, crc.data(), dig, &st)) return fail("complete");
                    --R.inflight;
                    if (W == 1 && st != PCC_ST_LOCAL_COMMIT && st != PCC_ST_OBSOLETE) fail("W=1 state", st);
                }
                ++done_writers;
            });
        }
    }
    // checker / committer: pointer monotone, names a started checkpoint; W > 1: MIN + apply_global
    std::vector<uint64_t> last(W, kNone);
    uint64_t g_last = kNone;
    const int total_writers = (int)W * writers_per_rank;
    auto check_round = [&]() {
        uint64_t g = kNone;
        bool any_none = false;
        for (uint32_t r = 0; r < W; ++r) {
            const uint64_t L = pcc_host_local_latest(ranks[r].h);
            if (L != kNone) {
                if (last[r] != kNone && L < last[r]) fail("pointer moved backwards", (long)last[r], (long)L);
                if (L > ranks[r].max_started.load()) fail("pointer names an unfinished checkpoint", (long)L);
                last[r] = L;
                g = std::min(g, L);
            } else {
                any_none = true;
            }
            const uint32_t fr = pcc_host_free_slots(ranks[r].h);
            if (fr > ranks[r].n_slots) fail("free slots > N+1", fr);
        }
        if (W > 1 && !any_none && g != kNone) {
            if (g_last != kNone && g < g_last) fail("global iter moved backwards", (long)g_last, (long)g);
            for (uint32_t r = 0; r < W; ++r) {
                if (pcc_host_apply_global(ranks[r].h, g)) fail("apply_global");
                uint64_t it[64];
                uint32_t sl[64];
                const uint32_t k = pcc_host_held(ranks[r].h, it, sl, 64);
                bool has_g = false;
                for (uint32_t i = 0; i < k && i < 64; ++i) has_g |= it[i] == g;
                if (!has_g) fail("rank lost the global checkpoint's slot", (long)r, (long)g);
            }
            g_last = g;
        }
    };
    while (done_writers.load() < total_writers && !g_fail) {
        check_round();
        std::this_thread::sleep_for(std::chrono::microseconds(50));
    }
    for (auto &t : th) t.join();
    check_round();
    if (g_fail) return 1;
    const uint64_t L0 = pcc_host_local_latest(ranks[0].h);
    for (auto &R : ranks) pcc_host_close(R.h);
    std::printf("OK %llu %llu\n", (unsigned long long)L0, (unsigned long long)g_last);
    return 0;
}
