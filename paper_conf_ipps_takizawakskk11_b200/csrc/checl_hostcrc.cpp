// checl_hostcrc.cpp — host-side CRC32C of the product library, used only for the
// image's meta_crc (header + manifest + CRC table, FORMAT.md) and for validating
// it at restore. Payload chunks are never CRC'd on the host.
//
// x86-64 with SSE4.2: the crc32 instruction, 8 bytes at a time. Otherwise:
// slicing-by-8 with tables generated from the polynomial at first use.
#include <cstdint>
#include <cstring>
#include <mutex>

#include "checl_internal.h"

#if defined(__x86_64__)
#include <nmmintrin.h>
#endif

namespace checl {

namespace {

uint32_t g_tab[8][256];
std::once_flag g_tab_once;

void build_tables() {
  for (uint32_t e = 0; e < 256; ++e) {
    uint32_t r = e;
    for (int b = 0; b < 8; ++b) r = gf_mulx(r);
    g_tab[0][e] = r;
  }
  for (int k = 1; k < 8; ++k)
    for (uint32_t e = 0; e < 256; ++e) g_tab[k][e] = (g_tab[k - 1][e] >> 8) ^ g_tab[0][g_tab[k - 1][e] & 0xFFu];
}

// raw register update (no init / final xor)
uint32_t sw_update(uint32_t crc, const uint8_t* p, size_t n) {
  std::call_once(g_tab_once, build_tables);
  while (n && (reinterpret_cast<uintptr_t>(p) & 7u)) {
    crc = (crc >> 8) ^ g_tab[0][(crc ^ *p++) & 0xFFu];
    --n;
  }
  while (n >= 8) {
    uint64_t w;
    std::memcpy(&w, p, 8);
    const uint32_t lo = (uint32_t)w ^ crc, hi = (uint32_t)(w >> 32);
    crc = g_tab[7][lo & 0xFF] ^ g_tab[6][(lo >> 8) & 0xFF] ^ g_tab[5][(lo >> 16) & 0xFF] ^ g_tab[4][lo >> 24] ^
          g_tab[3][hi & 0xFF] ^ g_tab[2][(hi >> 8) & 0xFF] ^ g_tab[1][(hi >> 16) & 0xFF] ^ g_tab[0][hi >> 24];
    p += 8;
    n -= 8;
  }
  while (n--) crc = (crc >> 8) ^ g_tab[0][(crc ^ *p++) & 0xFFu];
  return crc;
}

#if defined(__x86_64__)
// Three interleaved crc32 streams over blocks of 3 x kLane bytes (the instruction
// has a 3-cycle latency and 1-cycle throughput): R(A||B||C, s) = R(A, s) x^(8*2L)
// + R(B, 0) x^(8L) + R(C, 0) (linearity; DESIGN.md §5 "GF(2) algebra"), the two
// shifts by nibble tables of the constants x^(8L), x^(16L).
constexpr size_t kLane = 1024;
struct ShiftTab {
  uint32_t t[8][16];
  explicit ShiftTab(uint64_t nbytes) {
    const uint32_t k = gf_x8n(nbytes);
    for (int j = 0; j < 8; ++j)
      for (uint32_t v = 0; v < 16; ++v) t[j][v] = gf_mul(v << (4 * j), k);
  }
  uint32_t mul(uint32_t r) const {
    uint32_t o = 0;
    for (int j = 0; j < 8; ++j) o ^= t[j][(r >> (4 * j)) & 15u];
    return o;
  }
};

__attribute__((target("sse4.2"))) uint32_t hw_update(uint32_t crc, const uint8_t* p, size_t n) {
  uint64_t c = crc;
  if (n >= 3 * kLane) {
    static const ShiftTab s1(kLane), s2(2 * kLane);
    while (n >= 3 * kLane) {
      uint64_t a = c, b = 0, d = 0;
      for (size_t i = 0; i < kLane; i += 8) {
        uint64_t wa, wb, wd;
        std::memcpy(&wa, p + i, 8);
        std::memcpy(&wb, p + kLane + i, 8);
        std::memcpy(&wd, p + 2 * kLane + i, 8);
        a = _mm_crc32_u64(a, wa);
        b = _mm_crc32_u64(b, wb);
        d = _mm_crc32_u64(d, wd);
      }
      c = s2.mul((uint32_t)a) ^ s1.mul((uint32_t)b) ^ (uint32_t)d;
      p += 3 * kLane;
      n -= 3 * kLane;
    }
  }
  while (n >= 8) {
    uint64_t w;
    std::memcpy(&w, p, 8);
    c = _mm_crc32_u64(c, w);
    p += 8;
    n -= 8;
  }
  uint32_t c32 = (uint32_t)c;
  while (n--) c32 = _mm_crc32_u8(c32, *p++);
  return c32;
}

bool have_sse42() {
  static const bool ok = __builtin_cpu_supports("sse4.2");
  return ok;
}
#endif

}  // namespace

// Raw CRC32C register update over n bytes.
uint32_t host_crc32c_update(uint32_t crc, const void* data, size_t n) {
  const uint8_t* p = static_cast<const uint8_t*>(data);
#if defined(__x86_64__)
  if (have_sse42()) return hw_update(crc, p, n);
#endif
  return sw_update(crc, p, n);
}

uint32_t host_crc32c(const void* data, size_t n) { return ~host_crc32c_update(0xFFFFFFFFu, data, n); }

}  // namespace checl
