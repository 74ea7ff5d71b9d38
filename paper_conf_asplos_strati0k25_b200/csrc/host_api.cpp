// host_api.cpp — pccheck_host.h: the CommitEngine behind a C ABI (no CUDA).
#include <fcntl.h>
#include <sys/stat.h>
#include <unistd.h>

#include <cerrno>
#include <map>
#include <memory>
#include <mutex>

#include "../../include/pccheck_host.h"
#include "commit.hpp"
#include "errors.hpp"
#include "layout.hpp"

using namespace pcc;

struct pcc_host {
    CommitEngine engine;
    int fd = -1;
    uint64_t first = 0, n = 0, cb = 0;
    uint32_t n_slots = 0;
    std::mutex mu;
    std::map<uint64_t, Ticket> tickets;
    std::map<uint64_t, int> states;
};

extern "C" {

int pcc_host_open(const pcc_host_config *cfg, pcc_host **out) {
    if (!cfg || !out || cfg->world < 1 || cfg->rank >= cfg->world || cfg->max_inflight == 0 || !cfg->chunk_bytes)
        return set_error(PCC_EINVAL, "config");
    std::unique_ptr<pcc_host> h(new pcc_host());
    slice_of(cfg->total_chunks, cfg->rank, cfg->world, &h->first, &h->n);
    h->cb = cfg->chunk_bytes;
    h->n_slots = cfg->max_inflight + 1;
    if (cfg->path) {
        h->fd = ::open(cfg->path, O_RDWR | O_CREAT, 0644);
        if (h->fd < 0) return set_errno_error("open", errno);
        const uint64_t fb = file_bytes(h->n_slots, h->n, h->cb);
        struct stat st;
        if (fstat(h->fd, &st) == 0 && (uint64_t)st.st_size < fb && ftruncate(h->fd, (off_t)fb) != 0)
            return set_errno_error("ftruncate", errno);
    }
    CommitEngine::Config ec;
    ec.fd = h->fd;
    ec.geom = SlotGeom{cfg->chunk_bytes, cfg->rank, cfg->world, cfg->total_chunks, (uint32_t)h->first,
                       (uint32_t)h->n, cfg->n_tensors, cfg->align, cfg->layout_crc};
    ec.n_inflight = cfg->max_inflight;
    ec.fsync = cfg->fsync != 0;
    pcc_host *raw = h.get();
    // called under the engine's DP lock, from whichever thread's complete() drained the in-order
    // commits; h->mu orders it against pcc_host_begin / _state (no path holds h->mu while it
    // calls into the engine, so the two locks never nest the other way)
    ec.on_state = [raw](uint64_t counter, int st) {
        std::lock_guard<std::mutex> lk(raw->mu);
        raw->states[counter] = st;
    };
    int rc = h->engine.open(ec);
    if (rc) return rc;
    *out = h.release();
    return PCC_OK;
}

int pcc_host_begin(pcc_host *h, uint64_t iter, uint64_t *counter, uint32_t *slot) {
    Ticket t;
    int rc = h->engine.begin(iter, &t);
    if (rc) return rc;
    std::lock_guard<std::mutex> lk(h->mu);
    h->tickets[t.counter] = t;
    h->states[t.counter] = PCC_ST_QUEUED;
    *counter = t.counter;
    *slot = t.slot;
    return PCC_OK;
}

static Ticket *ticket(pcc_host *h, uint64_t counter) {
    std::lock_guard<std::mutex> lk(h->mu);
    auto it = h->tickets.find(counter);
    return it == h->tickets.end() ? nullptr : &it->second;
}

int pcc_host_filling(pcc_host *h, uint64_t counter) {
    Ticket *t = ticket(h, counter);
    return t ? h->engine.filling(*t) : set_error(PCC_EINVAL, "counter");
}

int pcc_host_complete(pcc_host *h, uint64_t counter, const uint32_t *crc, uint32_t digest, int *state) {
    Ticket *t = ticket(h, counter);
    if (!t) return set_error(PCC_EINVAL, "counter");
    int st = PCC_ST_FAILED;
    int rc = h->engine.complete(*t, crc, digest, &st);
    {
        std::lock_guard<std::mutex> lk(h->mu);
        if (h->engine.geom().world == 1 || st == PCC_ST_FAILED) h->states[counter] = st;
        if (state) *state = h->states[counter] == PCC_ST_QUEUED ? PCC_ST_PERSISTED : h->states[counter];
    }
    return rc;
}

int pcc_host_fail(pcc_host *h, uint64_t counter) {
    Ticket *t = ticket(h, counter);
    if (!t) return set_error(PCC_EINVAL, "counter");
    h->engine.fail(*t);
    std::lock_guard<std::mutex> lk(h->mu);
    h->states[counter] = PCC_ST_FAILED;
    return PCC_OK;
}

int pcc_host_state(pcc_host *h, uint64_t counter, int *state) {
    std::lock_guard<std::mutex> lk(h->mu);
    auto it = h->states.find(counter);
    if (it == h->states.end()) return set_error(PCC_EINVAL, "counter");
    *state = it->second;
    return PCC_OK;
}

uint64_t pcc_host_local_latest(pcc_host *h) { return h->engine.local_latest(); }
uint64_t pcc_host_global(pcc_host *h) { return h->engine.global_iter(); }
int pcc_host_apply_global(pcc_host *h, uint64_t g) { return h->engine.apply_global(g); }
uint32_t pcc_host_free_slots(pcc_host *h) { return h->engine.free_count(); }

int pcc_host_geometry(pcc_host *h, uint32_t *first, uint32_t *n, uint32_t *n_slots) {
    if (first) *first = (uint32_t)h->first;
    if (n) *n = (uint32_t)h->n;
    if (n_slots) *n_slots = h->n_slots;
    return PCC_OK;
}

uint64_t pcc_host_data_offset(pcc_host *h, uint32_t slot) { return slot_offset(slot, h->n, h->cb) + header_bytes(h->n); }

uint32_t pcc_host_held(pcc_host *h, uint64_t *iters, uint32_t *slots, uint32_t cap) {
    auto m = h->engine.held();
    uint32_t k = 0;
    for (auto &kv : m) {
        if (k < cap) {
            iters[k] = kv.first;
            slots[k] = kv.second;
        }
        ++k;
    }
    return k;
}

int pcc_host_restore_plan(pcc_host *h, uint64_t want_iter, uint32_t flags, pcc_reduce_fn reduce, pcc_verify_fn verify,
                          void *ctx, uint64_t *restored_iter) {
    if (!h || !reduce || !verify || h->fd < 0) return set_error(PCC_EINVAL, "args");
    SlotScan S;
    int rc = scan_rank_file(h->fd, h->engine.geom(), h->n_slots, &S);
    if (rc) return rc;
    RestoreOps ops;
    ops.reduce = [&](int64_t *v, bool is_max) { return reduce(ctx, v, is_max ? 1 : 0); };
    ops.verify = [&](uint64_t it, uint32_t slot, std::vector<uint32_t> *) {
        return verify(ctx, it, slot) == 0 ? PCC_OK : set_error(PCC_ECORRUPT, "verify callback");
    };
    uint64_t it = 0;
    rc = restore_agree(S, want_iter, flags, ops, &it, nullptr);
    if (rc == PCC_OK && restored_iter) *restored_iter = it;
    return rc;
}

int pcc_host_close(pcc_host *h) {
    if (!h) return PCC_OK;
    int fd = h->fd;
    delete h;
    if (fd >= 0) ::close(fd);
    return PCC_OK;
}

}  // extern "C"
