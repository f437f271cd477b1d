/* Test-only independent CRC32C: the x86 SSE4.2 `crc32` instruction (Castagnoli,
 * reflected). Shares nothing with oracle/ or the product; used to pin both. */
#include <nmmintrin.h>
#include <stddef.h>
#include <stdint.h>
#include <string.h>

uint32_t hw_crc32c(const uint8_t* p, size_t n) {
  uint64_t c = 0xFFFFFFFFu;
  while (n >= 8) {
    uint64_t w;
    memcpy(&w, p, 8);
    c = _mm_crc32_u64(c, w);
    p += 8;
    n -= 8;
  }
  uint32_t c32 = (uint32_t)c;
  while (n--) c32 = _mm_crc32_u8(c32, *p++);
  return c32 ^ 0xFFFFFFFFu;
}

/* CRC of each [offs[i], offs[i]+lens[i]) slice of base, for whole-image checks */
void hw_crc32c_many(const uint8_t* base, const uint64_t* offs, const uint64_t* lens, size_t n, uint32_t* out) {
  for (size_t i = 0; i < n; ++i) out[i] = hw_crc32c(base + offs[i], lens[i]);
}
