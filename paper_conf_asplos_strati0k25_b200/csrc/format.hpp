// format.hpp — the per-rank checkpoint file (FORMAT.md), product side.
//
// [pointer record A @0][pointer record B @4096][slot 0]...[slot N]; slot s at
// 8192 + s*stride; a slot = header (H = align_up(96+4n+4, 4096) bytes) + n chunks.
// The pointer records are the persisted CHECK_ADDR of Listing 1 (PAPER.md L229, L237,
// L253-L268; reading R7: two alternating CRC-protected records, written monotonically);
// the slot header is Check_meta (L227, L250) extended with the chunk CRC table (R4, R18).
//
// Host CRC32C for these 4 KiB metadata records uses the SSE4.2 crc32 instruction (the
// bulk data CRCs are computed on the GPU by K1).  Nothing here is shared with oracle/.
#pragma once
#include <cstdint>
#include <cstring>
#include <nmmintrin.h>

namespace pcc {

inline uint32_t host_crc32c(const void *data, uint64_t n) {
    const uint8_t *p = static_cast<const uint8_t *>(data);
    uint64_t c = 0xFFFFFFFFu;
    while (n >= 8) {
        uint64_t v;
        std::memcpy(&v, p, 8);
        c = _mm_crc32_u64(c, v);
        p += 8;
        n -= 8;
    }
    uint32_t c32 = static_cast<uint32_t>(c);
    while (n--) c32 = _mm_crc32_u8(c32, *p++);
    return c32 ^ 0xFFFFFFFFu;
}

constexpr uint64_t kPage = 4096;
constexpr uint32_t kStateFilling = 1, kStateComplete = 2, kVersion = 1;

inline uint64_t round_up(uint64_t x, uint64_t a) { return (x + a - 1) / a * a; }
inline uint64_t header_bytes(uint64_t n) { return round_up(96 + 4 * n + 4, kPage); }
inline uint64_t slot_stride(uint64_t n, uint64_t cb) { return round_up(header_bytes(n) + n * cb, kPage); }
inline uint64_t slot_offset(uint32_t s, uint64_t n, uint64_t cb) { return 2 * kPage + s * slot_stride(n, cb); }
inline uint64_t file_bytes(uint32_t n_slots, uint64_t n, uint64_t cb) { return 2 * kPage + n_slots * slot_stride(n, cb); }

template <class T>
inline void put(uint8_t *b, uint64_t off, T v) { std::memcpy(b + off, &v, sizeof(T)); }  // x86: little-endian
template <class T>
inline T get(const uint8_t *b, uint64_t off) {
    T v;
    std::memcpy(&v, b + off, sizeof(T));
    return v;
}

struct SlotGeom {  // what every header of this rank file carries
    uint64_t chunk_bytes;
    uint32_t rank, world, total_chunks, first_chunk, n, n_tensors, align, layout_crc;
};

// Fills a header of header_bytes(n) bytes (buffer zeroed by the caller).
inline void encode_header(uint8_t *h, const SlotGeom &g, uint32_t state, uint64_t iter, uint64_t counter,
                          uint32_t digest, uint32_t slot, const uint32_t *crc) {
    std::memcpy(h, "PCCSLOT1", 8);
    put<uint32_t>(h, 8, state);
    put<uint32_t>(h, 12, kVersion);
    put<uint64_t>(h, 16, iter);
    put<uint64_t>(h, 24, counter);
    put<uint64_t>(h, 32, g.chunk_bytes);
    put<uint32_t>(h, 40, g.rank);
    put<uint32_t>(h, 44, g.world);
    put<uint32_t>(h, 48, g.total_chunks);
    put<uint32_t>(h, 52, g.first_chunk);
    put<uint32_t>(h, 56, g.n);
    put<uint32_t>(h, 60, g.n_tensors);
    put<uint32_t>(h, 64, g.align);
    put<uint32_t>(h, 68, g.layout_crc);
    put<uint32_t>(h, 72, digest);
    put<uint32_t>(h, 76, slot);
    std::memset(h + 80, 0, 16);
    if (crc)
        std::memcpy(h + 96, crc, 4ull * g.n);
    else
        std::memset(h + 96, 0, 4ull * g.n);
    put<uint32_t>(h, 96 + 4ull * g.n, host_crc32c(h, 96 + 4ull * g.n));
}

struct PtrRecord {
    bool valid = false;
    uint32_t world = 0, rank = 0, local_slot = 0, n_slots = 0;
    uint64_t seq = 0, local_iter = 0, local_counter = 0, global_iter = 0;
};

inline void encode_ptr(uint8_t *b, const PtrRecord &r) {
    std::memset(b, 0, kPage);
    std::memcpy(b, "PCCPTR01", 8);
    put<uint32_t>(b, 8, kVersion);
    put<uint32_t>(b, 12, r.world);
    put<uint64_t>(b, 16, r.seq);
    put<uint64_t>(b, 24, r.local_iter);
    put<uint64_t>(b, 32, r.local_counter);
    put<uint32_t>(b, 40, r.local_slot);
    put<uint32_t>(b, 44, r.rank);
    put<uint64_t>(b, 48, r.global_iter);
    put<uint32_t>(b, 56, r.n_slots);
    put<uint32_t>(b, 4092, host_crc32c(b, 4092));
}

inline PtrRecord decode_ptr(const uint8_t *b) {
    PtrRecord r;
    if (std::memcmp(b, "PCCPTR01", 8) != 0 || get<uint32_t>(b, 8) != kVersion) return r;
    if (get<uint32_t>(b, 4092) != host_crc32c(b, 4092)) return r;
    r.valid = true;
    r.world = get<uint32_t>(b, 12);
    r.seq = get<uint64_t>(b, 16);
    r.local_iter = get<uint64_t>(b, 24);
    r.local_counter = get<uint64_t>(b, 32);
    r.local_slot = get<uint32_t>(b, 40);
    r.rank = get<uint32_t>(b, 44);
    r.global_iter = get<uint64_t>(b, 48);
    r.n_slots = get<uint32_t>(b, 56);
    return r;
}

struct HeaderView {
    bool ok = false;  // magic, version, hdr_crc, state COMPLETE
    bool layout_ok = false;
    uint64_t iter = 0, counter = 0;
    uint32_t digest = 0, slot = 0;
    const uint8_t *crc = nullptr;  // n little-endian u32
};

inline HeaderView decode_header(const uint8_t *h, const SlotGeom &g, uint32_t slot) {
    HeaderView v;
    if (std::memcmp(h, "PCCSLOT1", 8) != 0) return v;
    if (get<uint32_t>(h, 96 + 4ull * g.n) != host_crc32c(h, 96 + 4ull * g.n)) return v;
    if (get<uint32_t>(h, 8) != kStateComplete || get<uint32_t>(h, 12) != kVersion) return v;
    v.ok = true;
    v.iter = get<uint64_t>(h, 16);
    v.counter = get<uint64_t>(h, 24);
    v.digest = get<uint32_t>(h, 72);
    v.slot = get<uint32_t>(h, 76);
    v.crc = h + 96;
    v.layout_ok = get<uint64_t>(h, 32) == g.chunk_bytes && get<uint32_t>(h, 40) == g.rank &&
                  get<uint32_t>(h, 44) == g.world && get<uint32_t>(h, 48) == g.total_chunks &&
                  get<uint32_t>(h, 52) == g.first_chunk && get<uint32_t>(h, 56) == g.n &&
                  get<uint32_t>(h, 60) == g.n_tensors && get<uint32_t>(h, 64) == g.align &&
                  get<uint32_t>(h, 68) == g.layout_crc && v.slot == slot;
    return v;
}

// layout_crc = CRC32C(for each tensor: nbytes u64 ‖ dtype u32; then align u32 ‖ chunk_bytes u64)
inline uint32_t layout_crc(uint32_t n, const uint64_t *nbytes, const uint32_t *dtype, uint32_t align, uint64_t cb) {
    const uint64_t sz = 12ull * n + 12;
    uint8_t *b = new uint8_t[sz];
    for (uint32_t i = 0; i < n; ++i) {
        put<uint64_t>(b, 12ull * i, nbytes[i]);
        put<uint32_t>(b, 12ull * i + 8, dtype[i]);
    }
    put<uint32_t>(b, 12ull * n, align);
    put<uint64_t>(b, 12ull * n + 4, cb);
    const uint32_t c = host_crc32c(b, sz);
    delete[] b;
    return c;
}

}  // namespace pcc
