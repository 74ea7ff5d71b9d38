/*
 * pcc_oracle.c — the CPU ORACLE for the PCcheck snapshot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load, call or link this file.  The
 * product library (paper_conf_asplos_strati0k25_b200/) never includes, links or
 * calls it, and this file includes nothing from the product.
 *
 * What it computes is the plain definition of each step, single-threaded, one byte
 * at a time where a byte-level definition exists.  Citations are PAPER.md line
 * numbers ("L<n>") plus the section; readings the paper does not fix are the
 * numbered readings R1..R20 in DESIGN.md §3 (they follow SURVEY.md §8(c)).
 *
 *   O1 layout          R1 (§3.1/§4.1 "contiguous on storage")
 *   O2 pack            R1, R3
 *   O3 CRC32C          R4  (no checksum in the paper; BASELINE.json north_star)
 *   O4 digest          R4
 *   O5 on-file format  R7, R18 (Listing 1 L235-L268 Check_meta / CHECK_ADDR, L227-L229 §4.1)
 *   O7 restore         L287 §4.2; R10, R13
 *
 * Parity pins (tests/test_oracle_*.py): RFC 3720 §B.4 CRC32C vectors, the SSE4.2
 * crc32 instruction (an independent implementation), round-trip identity, brute
 * force on tiny registrations, fault injection.  No function here is unpinned.
 */
#include <stdint.h>
#include <stddef.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <fcntl.h>
#include <unistd.h>
#include <sys/stat.h>

#define ORC_EXPORT __attribute__((visibility("default")))

/* ------------------------------------------------------------------ O3 CRC32C */
/* CRC-32C (Castagnoli): reflected polynomial 0x82F63B78, init 0xFFFFFFFF,
 * xorout 0xFFFFFFFF (RFC 3720 §B.4).  Byte-at-a-time table (Sarwate); the table
 * entry for byte b is the CRC register after shifting b through 8 times. */
static uint32_t orc_table[256];
static int orc_table_ready = 0;

static void orc_init_table(void) {
    for (uint32_t b = 0; b < 256; ++b) {
        uint32_t r = b;
        for (int k = 0; k < 8; ++k) r = (r & 1u) ? (r >> 1) ^ 0x82F63B78u : (r >> 1);
        orc_table[b] = r;
    }
    orc_table_ready = 1;
}

/* raw register update: no init / xorout applied */
static uint32_t orc_crc_update(uint32_t reg, const uint8_t *p, uint64_t n) {
    if (!orc_table_ready) orc_init_table();
    for (uint64_t i = 0; i < n; ++i) reg = (reg >> 8) ^ orc_table[(reg ^ p[i]) & 0xFFu];
    return reg;
}

ORC_EXPORT uint32_t orc_crc32c(const uint8_t *p, uint64_t n) {
    return orc_crc_update(0xFFFFFFFFu, p, n) ^ 0xFFFFFFFFu;
}

/* CRC32C(A || B) from crc = CRC32C(A): undo the xorout, keep feeding bytes one at a time,
 * apply the xorout again.  The same byte loop as orc_crc32c, resumable, so a slice digest
 * (O4) of a multi-GB image can be computed in one pass over chunks handed in order. */
ORC_EXPORT uint32_t orc_crc32c_extend(uint32_t crc, const uint8_t *p, uint64_t n) {
    return orc_crc_update(crc ^ 0xFFFFFFFFu, p, n) ^ 0xFFFFFFFFu;
}

/* ------------------------------------------------------------------ O1 layout */
/* Tensors in registration order; off_0 = 0; off_i = align_up(off_{i-1} + nbytes_{i-1}, align);
 * end = off_last + nbytes_last; C = ceil(end / chunk_bytes).  (R1, R2, R3) */
static uint64_t align_up(uint64_t x, uint64_t a) { return (x + a - 1) / a * a; }

ORC_EXPORT int orc_layout(uint32_t n, const uint64_t *nbytes, uint32_t align, uint64_t chunk_bytes,
                          uint64_t *off, uint64_t *end_out, uint64_t *n_chunks_out) {
    if (align == 0 || chunk_bytes == 0) return -1;
    uint64_t end = 0;
    for (uint32_t i = 0; i < n; ++i) {
        uint64_t o = (i == 0) ? 0 : align_up(end, align);
        off[i] = o;
        end = o + nbytes[i];
    }
    *end_out = end;
    *n_chunks_out = (end + chunk_bytes - 1) / chunk_bytes;
    return 0;
}

/* Rank r of W owns chunks [floor(r*C/W), floor((r+1)*C/W)).  (§8(e); §3.1) */
ORC_EXPORT void orc_slice(uint64_t n_chunks, uint32_t rank, uint32_t world, uint64_t *first, uint64_t *count) {
    uint64_t a = n_chunks * rank / world, b = n_chunks * (rank + 1) / world;
    *first = a;
    *count = b - a;
}

/* -------------------------------------------------------------------- O2 pack */
/* Writes image bytes [first_chunk*CB, (first_chunk+count)*CB) into out:
 * image[off_i + k] = src_i[k] for every tensor i and 0 <= k < nbytes_i; every other
 * byte is 0.  Bytes are copied verbatim — no dtype interpretation.  (R1, R3) */
ORC_EXPORT void orc_pack(uint32_t n, const uint8_t *const *src, const uint64_t *nbytes, const uint64_t *off,
                         uint64_t chunk_bytes, uint64_t first_chunk, uint64_t count, uint8_t *out) {
    uint64_t lo = first_chunk * chunk_bytes, hi = (first_chunk + count) * chunk_bytes;
    for (uint64_t p = lo; p < hi; ++p) out[p - lo] = 0;
    for (uint32_t i = 0; i < n; ++i) {
        for (uint64_t k = 0; k < nbytes[i]; ++k) {
            uint64_t p = off[i] + k;
            if (p >= lo && p < hi) out[p - lo] = src[i][k];
        }
    }
}

/* crc[c] = CRC32C(chunk c) for each of `count` consecutive chunks of `img`.  (R4) */
ORC_EXPORT void orc_chunk_crcs(const uint8_t *img, uint64_t count, uint64_t chunk_bytes, uint32_t *crc) {
    for (uint64_t c = 0; c < count; ++c) crc[c] = orc_crc32c(img + c * chunk_bytes, chunk_bytes);
}

/* ----------------------------------------------------------- O5 on-file format */
static void put_u32(uint8_t *p, uint32_t v) { for (int i = 0; i < 4; ++i) p[i] = (uint8_t)(v >> (8 * i)); }
static void put_u64(uint8_t *p, uint64_t v) { for (int i = 0; i < 8; ++i) p[i] = (uint8_t)(v >> (8 * i)); }
static uint32_t get_u32(const uint8_t *p) { uint32_t v = 0; for (int i = 0; i < 4; ++i) v |= (uint32_t)p[i] << (8 * i); return v; }
static uint64_t get_u64(const uint8_t *p) { uint64_t v = 0; for (int i = 0; i < 8; ++i) v |= (uint64_t)p[i] << (8 * i); return v; }

/* layout_crc = CRC32C( for each tensor: nbytes u64 LE ‖ dtype u32 LE ; then align u32 LE ‖ chunk_bytes u64 LE ) */
ORC_EXPORT uint32_t orc_layout_crc(uint32_t n, const uint64_t *nbytes, const uint32_t *dtype, uint32_t align,
                                   uint64_t chunk_bytes) {
    uint32_t reg = 0xFFFFFFFFu;
    uint8_t b[12];
    for (uint32_t i = 0; i < n; ++i) {
        put_u64(b, nbytes[i]);
        put_u32(b + 8, dtype[i]);
        reg = orc_crc_update(reg, b, 12);
    }
    put_u32(b, align);
    put_u64(b + 4, chunk_bytes);
    reg = orc_crc_update(reg, b, 12);
    return reg ^ 0xFFFFFFFFu;
}

/* Slot header size H = align_up(96 + 4n + 4, 4096). */
ORC_EXPORT uint64_t orc_header_bytes(uint64_t n) { return align_up(96 + 4 * n + 4, 4096); }
ORC_EXPORT uint64_t orc_slot_stride(uint64_t n, uint64_t chunk_bytes) {
    return align_up(orc_header_bytes(n) + n * chunk_bytes, 4096);
}
ORC_EXPORT uint64_t orc_slot_offset(uint32_t slot, uint64_t n, uint64_t chunk_bytes) {
    return 8192 + (uint64_t)slot * orc_slot_stride(n, chunk_bytes);
}

/* The Check_meta of Listing 1 line 16 (L250), extended with the chunk CRC table.
 * Writes H bytes into out (caller provides orc_header_bytes(n) bytes). */
ORC_EXPORT void orc_slot_header(uint8_t *out, uint32_t state, uint64_t iter, uint64_t counter, uint64_t chunk_bytes,
                                uint32_t rank, uint32_t world, uint32_t total_chunks, uint32_t first_chunk,
                                uint32_t n, uint32_t n_tensors, uint32_t align, uint32_t layout_crc,
                                uint32_t digest, uint32_t slot, const uint32_t *crc) {
    uint64_t H = orc_header_bytes(n);
    memset(out, 0, H);
    memcpy(out, "PCCSLOT1", 8);
    put_u32(out + 8, state);
    put_u32(out + 12, 1);
    put_u64(out + 16, iter);
    put_u64(out + 24, counter);
    put_u64(out + 32, chunk_bytes);
    put_u32(out + 40, rank);
    put_u32(out + 44, world);
    put_u32(out + 48, total_chunks);
    put_u32(out + 52, first_chunk);
    put_u32(out + 56, n);
    put_u32(out + 60, n_tensors);
    put_u32(out + 64, align);
    put_u32(out + 68, layout_crc);
    put_u32(out + 72, digest);
    put_u32(out + 76, slot);
    for (uint32_t c = 0; c < n; ++c) put_u32(out + 96 + 4 * (uint64_t)c, crc ? crc[c] : 0);
    put_u32(out + 96 + 4 * (uint64_t)n, orc_crc32c(out, 96 + 4 * (uint64_t)n));
}

/* The persisted CHECK_ADDR (Listing 1 lines 3, 20-23; L229, L277), as one of two
 * alternating CRC-protected 4 KiB records (R7).  out must hold 4096 bytes. */
ORC_EXPORT void orc_ptr_record(uint8_t *out, uint32_t world, uint64_t seq, uint64_t local_iter,
                               uint64_t local_counter, uint32_t local_slot, uint32_t rank, uint64_t global_iter,
                               uint32_t n_slots) {
    memset(out, 0, 4096);
    memcpy(out, "PCCPTR01", 8);
    put_u32(out + 8, 1);
    put_u32(out + 12, world);
    put_u64(out + 16, seq);
    put_u64(out + 24, local_iter);
    put_u64(out + 32, local_counter);
    put_u32(out + 40, local_slot);
    put_u32(out + 44, rank);
    put_u64(out + 48, global_iter);
    put_u32(out + 56, n_slots);
    put_u32(out + 4092, orc_crc32c(out, 4092));
}

/* ------------------------------------------------------------ O7 restore (+R10) */
enum { ORC_OK = 0, ORC_ENOENT = 1, ORC_ECORRUPT = 2, ORC_ELAYOUT = 3, ORC_EIO = 4, ORC_EINVAL = 5 };

static int read_at(int fd, uint8_t *buf, uint64_t n, uint64_t off) {
    uint64_t done = 0;
    while (done < n) {
        ssize_t r = pread(fd, buf + done, n - done, (off_t)(off + done));
        if (r <= 0) return -1;  /* short file = missing bytes */
        done += (uint64_t)r;
    }
    return 0;
}

typedef struct {
    int valid;
    uint64_t seq, local_iter, local_counter, global_iter;
    uint32_t local_slot, world, rank, n_slots;
} orc_ptr;

static void parse_ptr(const uint8_t *b, orc_ptr *p) {
    memset(p, 0, sizeof(*p));
    if (memcmp(b, "PCCPTR01", 8) != 0) return;
    if (get_u32(b + 8) != 1) return;
    if (get_u32(b + 4092) != orc_crc32c(b, 4092)) return;
    p->valid = 1;
    p->world = get_u32(b + 12);
    p->seq = get_u64(b + 16);
    p->local_iter = get_u64(b + 24);
    p->local_counter = get_u64(b + 32);
    p->local_slot = get_u32(b + 40);
    p->rank = get_u32(b + 44);
    p->global_iter = get_u64(b + 48);
    p->n_slots = get_u32(b + 56);
}

/* Reads the two pointer records of a rank file and returns the valid one with the
 * larger seq (R7: a torn record falls back to the other).  0 = found. */
static int best_ptr(int fd, orc_ptr *out) {
    uint8_t b[4096];
    orc_ptr a, c;
    memset(&a, 0, sizeof a);
    memset(&c, 0, sizeof c);
    if (read_at(fd, b, 4096, 0) == 0) parse_ptr(b, &a);
    if (read_at(fd, b, 4096, 4096) == 0) parse_ptr(b, &c);
    if (!a.valid && !c.valid) return -1;
    if (a.valid && (!c.valid || a.seq > c.seq)) *out = a; else *out = c;
    return 0;
}

ORC_EXPORT int orc_latest(const char *path, uint64_t *global_iter, uint64_t *local_iter, uint64_t *seq) {
    int fd = open(path, O_RDONLY);
    if (fd < 0) return ORC_ENOENT;
    orc_ptr p;
    int r = best_ptr(fd, &p);
    close(fd);
    if (r) return ORC_ENOENT;
    *global_iter = p.global_iter;
    *local_iter = p.local_iter;
    *seq = p.seq;
    return ORC_OK;
}

/* Registration + geometry shared by every rank file of one restore. */
typedef struct {
    uint32_t n_tensors, align, world, n_slots;
    uint64_t chunk_bytes, n_chunks, layout_crc;
    const uint64_t *nbytes, *off;
} orc_geom;

/* Checks slot `s` of rank `r` as a holder of `iter`.  Returns ORC_OK and fills crc/digest,
 * ORC_ENOENT if the slot does not hold a COMPLETE header for iter, ORC_ELAYOUT on a
 * registration mismatch.  Data chunks are NOT checked here. */
static int check_header(int fd, const orc_geom *g, uint32_t rank, uint32_t slot, uint64_t iter,
                        uint64_t first, uint64_t n, uint8_t *hdr) {
    uint64_t H = orc_header_bytes(n);
    if (read_at(fd, hdr, H, orc_slot_offset(slot, n, g->chunk_bytes))) return ORC_ENOENT;
    if (memcmp(hdr, "PCCSLOT1", 8) != 0) return ORC_ENOENT;
    if (get_u32(hdr + 96 + 4 * n) != orc_crc32c(hdr, 96 + 4 * n)) return ORC_ENOENT;
    if (get_u32(hdr + 8) != 2 || get_u32(hdr + 12) != 1) return ORC_ENOENT;  /* R18: only COMPLETE */
    if (get_u64(hdr + 16) != iter) return ORC_ENOENT;
    if (get_u64(hdr + 32) != g->chunk_bytes || get_u32(hdr + 40) != rank || get_u32(hdr + 44) != g->world ||
        get_u32(hdr + 48) != g->n_chunks || get_u32(hdr + 52) != first || get_u32(hdr + 56) != n ||
        get_u32(hdr + 60) != g->n_tensors || get_u32(hdr + 64) != g->align || get_u32(hdr + 68) != g->layout_crc ||
        get_u32(hdr + 76) != slot)
        return ORC_ELAYOUT;
    return ORC_OK;
}

/* Lists the iters held by COMPLETE, CRC-valid headers of a rank file (the set H_r of §8(e)). */
static int list_iters(int fd, const orc_geom *g, uint32_t rank, uint64_t *iters, uint32_t *slots) {
    uint64_t first, n;
    orc_slice(g->n_chunks, rank, g->world, &first, &n);
    uint8_t *hdr = (uint8_t *)malloc(orc_header_bytes(n));
    int k = 0;
    for (uint32_t s = 0; s < g->n_slots; ++s) {
        uint64_t H = orc_header_bytes(n);
        if (read_at(fd, hdr, H, orc_slot_offset(s, n, g->chunk_bytes))) continue;
        if (memcmp(hdr, "PCCSLOT1", 8) != 0) continue;
        if (get_u32(hdr + 96 + 4 * n) != orc_crc32c(hdr, 96 + 4 * n)) continue;
        if (get_u32(hdr + 8) != 2) continue;
        iters[k] = get_u64(hdr + 16);
        slots[k] = s;
        ++k;
    }
    free(hdr);
    return k;
}

/* Restores the whole state from the W rank files of one checkpoint set.
 *   want_iter == UINT64_MAX: the newest globally committed iter (max over ranks of the
 *   pointer record's global_iter, §8(e) step 2); otherwise exactly want_iter.
 *   fallback != 0: on a rejected candidate, try the newest older iter held COMPLETE by
 *   every rank (R10).
 * Verification (R4, R13): header CRC, COMPLETE state, registration fields, every chunk's
 * CRC32C against the header table, and the slice digest.  Only an iter that passes on
 * every rank is scattered into dst (tensor i receives image[off_i, off_i + nbytes_i)).
 * bad[] receives (global chunk index) of every mismatching chunk of the first rejected
 * candidate.  Returns ORC_OK / ORC_ENOENT / ORC_ECORRUPT / ORC_ELAYOUT. */
ORC_EXPORT int orc_restore(uint32_t world, const char *const *paths, uint32_t n_slots, uint32_t n_tensors,
                           const uint64_t *nbytes, const uint32_t *dtype, uint32_t align, uint64_t chunk_bytes,
                           uint64_t want_iter, int fallback, uint8_t *const *dst, uint64_t *restored_iter,
                           uint32_t *bad, uint32_t bad_cap, uint32_t *n_bad) {
    *n_bad = 0;
    uint64_t *off = (uint64_t *)calloc(n_tensors ? n_tensors : 1, sizeof(uint64_t));
    uint64_t end, C;
    orc_layout(n_tensors, nbytes, align, chunk_bytes, off, &end, &C);
    orc_geom g = {n_tensors, align, world, n_slots, chunk_bytes, C,
                  orc_layout_crc(n_tensors, nbytes, dtype, align, chunk_bytes), nbytes, off};
    int *fds = (int *)calloc(world, sizeof(int));
    uint64_t *held = (uint64_t *)calloc((size_t)world * n_slots, sizeof(uint64_t));
    uint32_t *held_slot = (uint32_t *)calloc((size_t)world * n_slots, sizeof(uint32_t));
    int *n_held = (int *)calloc(world, sizeof(int));
    uint32_t *slot_of = (uint32_t *)calloc(world, sizeof(uint32_t));
    for (uint32_t r = 0; r < world; ++r) fds[r] = -1;
    int rc = ORC_ENOENT, first_reject = 0;
    uint64_t target = 0;
    int have_target = 0;
    for (uint32_t r = 0; r < world; ++r) {
        fds[r] = open(paths[r], O_RDONLY);
        if (fds[r] < 0) { rc = ORC_ENOENT; goto out; }
        n_held[r] = list_iters(fds[r], &g, r, held + (size_t)r * n_slots, held_slot + (size_t)r * n_slots);
        orc_ptr p;
        if (best_ptr(fds[r], &p) == 0) {
            if (!have_target || p.global_iter > target) target = p.global_iter;
            have_target = 1;
        }
    }
    if (want_iter != UINT64_MAX) { target = want_iter; have_target = 1; }
    if (!have_target) { rc = ORC_ENOENT; goto out; }
    /* candidates: target, then (fallback) iters < target held by every rank, newest first */
    for (;;) {
        int ok = 1;
        for (uint32_t r = 0; r < world && ok; ++r) {
            int found = 0;
            for (int k = 0; k < n_held[r]; ++k)
                if (held[(size_t)r * n_slots + k] == target) { slot_of[r] = held_slot[(size_t)r * n_slots + k]; found = 1; }
            if (!found) ok = 0;
        }
        int cand_rc = ok ? ORC_OK : ORC_ENOENT;
        if (ok) {
            /* header + chunk + digest verification on every rank */
            for (uint32_t r = 0; r < world; ++r) {
                uint64_t first, n;
                orc_slice(C, r, world, &first, &n);
                uint8_t *hdr = (uint8_t *)malloc(orc_header_bytes(n));
                int hr = check_header(fds[r], &g, r, slot_of[r], target, first, n, hdr);
                if (hr != ORC_OK) { cand_rc = hr; free(hdr); continue; }
                uint8_t *data = (uint8_t *)malloc(chunk_bytes ? chunk_bytes : 1);
                uint64_t base = orc_slot_offset(slot_of[r], n, chunk_bytes) + orc_header_bytes(n);
                uint32_t reg = 0xFFFFFFFFu;
                for (uint64_t c = 0; c < n; ++c) {
                    int miss = read_at(fds[r], data, chunk_bytes, base + c * chunk_bytes);
                    if (miss) memset(data, 0, chunk_bytes);
                    uint32_t crc = orc_crc32c(data, chunk_bytes);
                    reg = orc_crc_update(reg, data, chunk_bytes);
                    if (miss || crc != get_u32(hdr + 96 + 4 * c)) {
                        cand_rc = ORC_ECORRUPT;
                        if (!first_reject && *n_bad < bad_cap) bad[*n_bad] = (uint32_t)(first + c);
                        if (!first_reject) ++*n_bad;
                    }
                }
                if ((reg ^ 0xFFFFFFFFu) != get_u32(hdr + 72)) cand_rc = ORC_ECORRUPT;
                free(data);
                free(hdr);
            }
        }
        if (cand_rc == ORC_OK) {
            /* scatter: every rank's slice, byte by byte */
            for (uint32_t r = 0; r < world; ++r) {
                uint64_t first, n;
                orc_slice(C, r, world, &first, &n);
                uint64_t base = orc_slot_offset(slot_of[r], n, chunk_bytes) + orc_header_bytes(n);
                uint64_t lo = first * chunk_bytes, hi = (first + n) * chunk_bytes;
                uint8_t *img = (uint8_t *)malloc(hi - lo ? hi - lo : 1);
                if (hi > lo && read_at(fds[r], img, hi - lo, base)) { free(img); rc = ORC_EIO; goto out; }
                for (uint32_t i = 0; i < n_tensors; ++i)
                    for (uint64_t k = 0; k < nbytes[i]; ++k) {
                        uint64_t p = off[i] + k;
                        if (p >= lo && p < hi) dst[i][k] = img[p - lo];
                    }
                free(img);
            }
            *restored_iter = target;
            rc = ORC_OK;
            goto out;
        }
        if (!first_reject) { rc = cand_rc; first_reject = 1; }
        if (!fallback) goto out;
        /* next candidate: newest iter < target held by every rank */
        uint64_t next = 0;
        int found_next = 0;
        for (int k = 0; k < n_held[0]; ++k) {
            uint64_t h = held[k];
            if (h >= target) continue;
            int all = 1;
            for (uint32_t r = 1; r < world && all; ++r) {
                int f = 0;
                for (int j = 0; j < n_held[r]; ++j) if (held[(size_t)r * n_slots + j] == h) f = 1;
                all = f;
            }
            if (all && (!found_next || h > next)) { next = h; found_next = 1; }
        }
        if (!found_next) goto out;  /* rc stays the first rejection's code */
        target = next;
    }
out:
    for (uint32_t r = 0; r < world; ++r) if (fds[r] >= 0) close(fds[r]);
    free(slot_of);
    free(fds); free(held); free(held_slot); free(n_held); free(off);
    return rc;
}

/* ------------------------------------------------------- oracle-side file writer */
/* Writes one COMPLETE checkpoint of rank `rank` into slot `slot` of `path` (creating or
 * extending the file), then the pointer record for `seq` at offset 4096*(seq % 2).
 * The data region holds the slice's packed image (O2), the header its CRC table and
 * digest (O3, O4).  Used by tests to produce reference files; O6's fsync ordering is
 * irrelevant here because nothing crashes inside the oracle. */
ORC_EXPORT int orc_write_checkpoint(const char *path, uint32_t n_tensors, const uint8_t *const *src,
                                    const uint64_t *nbytes, const uint32_t *dtype, uint32_t align,
                                    uint64_t chunk_bytes, uint32_t rank, uint32_t world, uint32_t n_slots,
                                    uint32_t slot, uint64_t iter, uint64_t counter, uint64_t seq,
                                    uint64_t global_iter, int write_pointer) {
    uint64_t *off = (uint64_t *)calloc(n_tensors ? n_tensors : 1, sizeof(uint64_t));
    uint64_t end, C, first, n;
    orc_layout(n_tensors, nbytes, align, chunk_bytes, off, &end, &C);
    orc_slice(C, rank, world, &first, &n);
    uint8_t *img = (uint8_t *)malloc(n > 0 ? n * chunk_bytes : 1);
    orc_pack(n_tensors, src, nbytes, off, chunk_bytes, first, n, img);
    uint32_t *crc = (uint32_t *)calloc(n ? n : 1, sizeof(uint32_t));
    orc_chunk_crcs(img, n, chunk_bytes, crc);
    uint32_t digest = orc_crc32c(img, n * chunk_bytes);
    uint64_t H = orc_header_bytes(n);
    uint8_t *hdr = (uint8_t *)malloc(H);
    orc_slot_header(hdr, 2, iter, counter, chunk_bytes, rank, world, (uint32_t)C, (uint32_t)first, (uint32_t)n,
                    n_tensors, align, orc_layout_crc(n_tensors, nbytes, dtype, align, chunk_bytes), digest, slot, crc);
    int fd = open(path, O_RDWR | O_CREAT, 0644);
    int rc = fd < 0 ? ORC_EIO : ORC_OK;
    if (fd >= 0) {
        uint64_t total = 8192 + (uint64_t)n_slots * orc_slot_stride(n, chunk_bytes);
        struct stat st;
        if (fstat(fd, &st) == 0 && (uint64_t)st.st_size < total && ftruncate(fd, (off_t)total)) rc = ORC_EIO;
        uint64_t so = orc_slot_offset(slot, n, chunk_bytes);
        if (pwrite(fd, hdr, H, (off_t)so) != (ssize_t)H) rc = ORC_EIO;
        if (n && pwrite(fd, img, n * chunk_bytes, (off_t)(so + H)) != (ssize_t)(n * chunk_bytes)) rc = ORC_EIO;
        if (write_pointer) {
            uint8_t rec[4096];
            orc_ptr_record(rec, world, seq, iter, counter, slot, rank, global_iter, n_slots);
            if (pwrite(fd, rec, 4096, (off_t)(4096 * (seq % 2))) != 4096) rc = ORC_EIO;
        }
        close(fd);
    }
    free(off); free(img); free(crc); free(hdr);
    return rc;
}
