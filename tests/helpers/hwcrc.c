/* Independent CRC32C for tests: the x86 SSE4.2 `crc32` instruction (Intel SDM, CRC32 —
 * "Accumulate CRC32C Value", polynomial 0x11EDC6F41).  Shares nothing with oracle/ or the
 * CUDA path; it pins the oracle's table-driven CRC (pin P2). */
#include <stdint.h>
#include <stddef.h>
#include <string.h>
#include <nmmintrin.h>

uint32_t hw_crc32c(const uint8_t *p, size_t n) {
    uint64_t c = 0xFFFFFFFFu;
    while (n >= 8) { uint64_t v; memcpy(&v, p, 8); c = _mm_crc32_u64(c, v); p += 8; n -= 8; }
    uint32_t c32 = (uint32_t)c;
    while (n--) c32 = _mm_crc32_u8(c32, *p++);
    return c32 ^ 0xFFFFFFFFu;
}
