/*
 * checl_oracle.c — TEST INFRASTRUCTURE ONLY (see checl_oracle.h).
 *
 * Plain definition of the CheCL device-state snapshot, written in the order of
 * the paper's procedure (§III-C) over the byte layout frozen in
 * FORMAT.md. Nothing here is blocked, fused or reordered: one loop per step.
 * Single-threaded, libc only. Shares no code with the product library.
 */
#include "checl_oracle.h"

#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------------ */
/* CRC32C (FORMAT.md "Payload and chunks"; north_star "CRC32C")               */
/* ------------------------------------------------------------------------ */

#define ORACLE_POLY_REFLECTED 0x82F63B78u /* Castagnoli 0x1EDC6F41, bit-reversed */

uint32_t oracle_crc32c_bitwise(const uint8_t* p, size_t n) {
  uint32_t crc = 0xFFFFFFFFu;
  for (size_t i = 0; i < n; ++i) {
    crc ^= p[i];
    for (int bit = 0; bit < 8; ++bit) {
      if (crc & 1u)
        crc = (crc >> 1) ^ ORACLE_POLY_REFLECTED;
      else
        crc = crc >> 1;
    }
  }
  return crc ^ 0xFFFFFFFFu;
}

static uint32_t oracle_table[256];
static int oracle_table_ready = 0;

static void oracle_build_table(void) {
  /* entry e = the register after shifting byte e through 8 bit steps */
  for (uint32_t e = 0; e < 256; ++e) {
    uint32_t r = e;
    for (int bit = 0; bit < 8; ++bit) r = (r & 1u) ? (r >> 1) ^ ORACLE_POLY_REFLECTED : (r >> 1);
    oracle_table[e] = r;
  }
  oracle_table_ready = 1;
}

uint32_t oracle_crc32c(const uint8_t* p, size_t n) {
  if (!oracle_table_ready) oracle_build_table();
  uint32_t crc = 0xFFFFFFFFu;
  for (size_t i = 0; i < n; ++i) crc = (crc >> 8) ^ oracle_table[(crc ^ p[i]) & 0xFFu];
  return crc ^ 0xFFFFFFFFu;
}

/* ------------------------------------------------------------------------ */
/* Little-endian field access                                                */
/* ------------------------------------------------------------------------ */

static void put_u32(uint8_t* p, uint32_t v) {
  for (int i = 0; i < 4; ++i) p[i] = (uint8_t)(v >> (8 * i));
}
static void put_u64(uint8_t* p, uint64_t v) {
  for (int i = 0; i < 8; ++i) p[i] = (uint8_t)(v >> (8 * i));
}
static uint32_t get_u32(const uint8_t* p) {
  uint32_t v = 0;
  for (int i = 0; i < 4; ++i) v |= (uint32_t)p[i] << (8 * i);
  return v;
}
static uint64_t get_u64(const uint8_t* p) {
  uint64_t v = 0;
  for (int i = 0; i < 8; ++i) v |= (uint64_t)p[i] << (8 * i);
  return v;
}

/* Format constants (FORMAT.md "Header"). */
#define O_HEADER 128u
#define O_CHUNK 65536u
#define O_ALIGN 256u
#define O_PAYLOAD_ALIGN 4096u
#define O_RECORD 48u

/* a + b with overflow detection; returns 0 on overflow */
static int add_ok(uint64_t a, uint64_t b, uint64_t* out) {
  if (a > UINT64_MAX - b) return 0;
  *out = a + b;
  return 1;
}
static int align_ok(uint64_t x, uint64_t a, uint64_t* out) {
  uint64_t t;
  if (!add_ok(x, a - 1, &t)) return 0;
  *out = t / a * a;
  return 1;
}
static uint64_t chunks_of(uint64_t size) { return size / O_CHUNK + (size % O_CHUNK ? 1 : 0); }

/* ------------------------------------------------------------------------ */
/* Checkpoint: walk the database in ascending handle id (L19), copy each     */
/* object's bytes into the image (L16 step 2), CRC each 64 KiB chunk.        */
/* ------------------------------------------------------------------------ */

static int cmp_handle(const void* a, const void* b) {
  const oracle_buffer* x = *(const oracle_buffer* const*)a;
  const oracle_buffer* y = *(const oracle_buffer* const*)b;
  return x->handle < y->handle ? -1 : (x->handle > y->handle ? 1 : 0);
}

/* sorted view of the registry; caller frees */
static const oracle_buffer** sorted_view(const oracle_buffer* bufs, size_t n, int* status) {
  const oracle_buffer** v = (const oracle_buffer**)malloc((n ? n : 1) * sizeof(*v));
  if (!v) {
    *status = ORACLE_OUT_OF_HOST_MEMORY;
    return NULL;
  }
  for (size_t i = 0; i < n; ++i) v[i] = &bufs[i];
  qsort(v, n, sizeof(*v), cmp_handle);
  for (size_t i = 0; i < n; ++i) {
    if (v[i]->handle == 0 || (i > 0 && v[i]->handle == v[i - 1]->handle) ||
        (v[i]->size > 0 && v[i]->data == NULL)) {
      free(v);
      *status = ORACLE_INVALID_VALUE;
      return NULL;
    }
  }
  *status = ORACLE_SUCCESS;
  return v;
}

static int layout_sorted(const oracle_buffer* const* v, size_t n, oracle_layout* L,
                         uint64_t* offs, uint64_t* firsts) {
  uint64_t off = 0, chunk = 0, end = 0;
  for (size_t b = 0; b < n; ++b) {
    if (b > 0 && !align_ok(end, O_ALIGN, &off)) return ORACLE_INVALID_VALUE;
    if (offs) offs[b] = off;
    if (firsts) firsts[b] = chunk;
    if (!add_ok(off, v[b]->size, &end)) return ORACLE_INVALID_VALUE;
    chunk += chunks_of(v[b]->size);
  }
  L->n_buffers = n;
  L->n_chunks = chunk;
  L->crc_off = O_HEADER + O_RECORD * (uint64_t)n;
  L->payload_bytes = n ? end : 0;
  if (!align_ok(L->crc_off + 4u * chunk, O_PAYLOAD_ALIGN, &L->payload_off)) return ORACLE_INVALID_VALUE;
  if (!add_ok(L->payload_off, L->payload_bytes, &L->image_bytes)) return ORACLE_INVALID_VALUE;
  return ORACLE_SUCCESS;
}

int oracle_layout_of(const oracle_buffer* bufs, size_t n, oracle_layout* out) {
  int st;
  if (!out || (n && !bufs)) return ORACLE_INVALID_VALUE;
  const oracle_buffer** v = sorted_view(bufs, n, &st);
  if (!v) return st;
  st = layout_sorted(v, n, out, NULL, NULL);
  free(v);
  return st;
}

static uint32_t meta_crc_of(const uint8_t* img, uint64_t payload_off) {
  /* CRC32C(image[0,124) || image[128, payload_off)) — one running register */
  if (!oracle_table_ready) oracle_build_table();
  uint32_t crc = 0xFFFFFFFFu;
  for (uint64_t i = 0; i < 124; ++i) crc = (crc >> 8) ^ oracle_table[(crc ^ img[i]) & 0xFFu];
  for (uint64_t i = O_HEADER; i < payload_off; ++i) crc = (crc >> 8) ^ oracle_table[(crc ^ img[i]) & 0xFFu];
  return crc ^ 0xFFFFFFFFu;
}

int oracle_checkpoint(const oracle_buffer* bufs, size_t n, int32_t device, uint64_t epoch,
                      uint8_t* out, size_t out_cap) {
  int st;
  if (!out || (n && !bufs)) return ORACLE_INVALID_VALUE;
  const oracle_buffer** v = sorted_view(bufs, n, &st);
  if (!v) return st;
  uint64_t* offs = (uint64_t*)malloc((n ? n : 1) * sizeof(uint64_t));
  uint64_t* firsts = (uint64_t*)malloc((n ? n : 1) * sizeof(uint64_t));
  oracle_layout L;
  if (!offs || !firsts) {
    st = ORACLE_OUT_OF_HOST_MEMORY;
    goto done;
  }
  st = layout_sorted(v, n, &L, offs, firsts);
  if (st) goto done;
  if (out_cap < L.image_bytes) {
    st = ORACLE_INVALID_VALUE;
    goto done;
  }
  /* everything not written below is zero: reserved fields, padding, gaps */
  memset(out, 0, L.image_bytes);

  /* Step 2 of L16: copy every object's bytes to host, in database order. */
  for (size_t b = 0; b < n; ++b)
    if (v[b]->size) memcpy(out + L.payload_off + offs[b], v[b]->data, v[b]->size);

  /* CRC table: one independent CRC32C per 64 KiB chunk of each buffer. */
  for (size_t b = 0; b < n; ++b) {
    uint64_t nch = chunks_of(v[b]->size);
    for (uint64_t k = 0; k < nch; ++k) {
      uint64_t lo = k * O_CHUNK;
      uint64_t len = v[b]->size - lo < O_CHUNK ? v[b]->size - lo : O_CHUNK;
      put_u32(out + L.crc_off + 4u * (firsts[b] + k), oracle_crc32c(v[b]->data + lo, len));
    }
  }

  /* Manifest records. */
  for (size_t b = 0; b < n; ++b) {
    uint8_t* r = out + O_HEADER + O_RECORD * b;
    put_u64(r + 0, v[b]->handle);
    put_u64(r + 8, v[b]->size);
    put_u64(r + 16, offs[b]);
    put_u64(r + 24, firsts[b]);
    put_u32(r + 32, v[b]->flags);
    put_u32(r + 36, (uint32_t)device);
  }

  /* Header, then meta_crc over everything that is not payload. */
  memcpy(out, "CHECLIM1", 8);
  put_u32(out + 8, 1);
  put_u32(out + 12, O_HEADER);
  put_u32(out + 16, O_CHUNK);
  put_u32(out + 20, O_ALIGN);
  put_u64(out + 24, L.n_buffers);
  put_u64(out + 32, L.n_chunks);
  put_u64(out + 40, O_HEADER);
  put_u64(out + 48, L.crc_off);
  put_u64(out + 56, L.payload_off);
  put_u64(out + 64, L.payload_bytes);
  put_u64(out + 72, L.image_bytes);
  put_u32(out + 80, (uint32_t)device);
  put_u32(out + 84, 0);
  put_u64(out + 88, epoch);
  put_u32(out + 124, meta_crc_of(out, L.payload_off));
  st = ORACLE_SUCCESS;
done:
  free(offs);
  free(firsts);
  free(v);
  return st;
}

/* ------------------------------------------------------------------------ */
/* Restart (L16 restart steps 2-3)                                           */
/* ------------------------------------------------------------------------ */

static void report_init(oracle_report* rep) {
  memset(rep, 0, sizeof(*rep));
  rep->first_bad_chunk = UINT64_MAX;
}

int oracle_validate(const uint8_t* img, size_t len, oracle_report* rep) {
  oracle_report local;
  if (!rep) rep = &local;
  report_init(rep);
  if (!img || len < O_HEADER) return ORACLE_BAD_IMAGE;
  if (memcmp(img, "CHECLIM1", 8) != 0) return ORACLE_BAD_IMAGE;
  if (get_u32(img + 8) != 1 || get_u32(img + 12) != O_HEADER || get_u32(img + 16) != O_CHUNK ||
      get_u32(img + 20) != O_ALIGN || get_u64(img + 40) != O_HEADER || get_u32(img + 84) != 0)
    return ORACLE_BAD_IMAGE;
  for (int i = 96; i < 124; ++i)
    if (img[i] != 0) return ORACLE_BAD_IMAGE;
  uint64_t n = get_u64(img + 24), nch = get_u64(img + 32);
  uint64_t crc_off = get_u64(img + 48), payload_off = get_u64(img + 56);
  uint64_t payload_bytes = get_u64(img + 64), image_bytes = get_u64(img + 72);
  int32_t device = (int32_t)get_u32(img + 80);
  /* closed-form region offsets, with overflow checks */
  if (n > (UINT64_MAX - O_HEADER) / O_RECORD) return ORACLE_BAD_IMAGE;
  if (crc_off != O_HEADER + O_RECORD * n) return ORACLE_BAD_IMAGE;
  if (nch > (UINT64_MAX - crc_off) / 4u) return ORACLE_BAD_IMAGE;
  uint64_t want_payload_off;
  if (!align_ok(crc_off + 4u * nch, O_PAYLOAD_ALIGN, &want_payload_off)) return ORACLE_BAD_IMAGE;
  if (payload_off != want_payload_off) return ORACLE_BAD_IMAGE;
  uint64_t want_image;
  if (!add_ok(payload_off, payload_bytes, &want_image) || image_bytes != want_image) return ORACLE_BAD_IMAGE;
  if ((uint64_t)len < image_bytes) return ORACLE_BAD_IMAGE;
  if (get_u32(img + 124) != meta_crc_of(img, payload_off)) return ORACLE_BAD_IMAGE;
  for (uint64_t i = crc_off + 4u * nch; i < payload_off; ++i)
    if (img[i] != 0) return ORACLE_BAD_IMAGE;
  /* records */
  uint64_t off = 0, end = 0, chunk = 0, prev = 0;
  for (uint64_t b = 0; b < n; ++b) {
    const uint8_t* r = img + O_HEADER + O_RECORD * b;
    uint64_t h = get_u64(r), size = get_u64(r + 8);
    if (h == 0 || (b > 0 && h <= prev)) return ORACLE_BAD_IMAGE;
    if (b > 0 && !align_ok(end, O_ALIGN, &off)) return ORACLE_BAD_IMAGE;
    if (get_u64(r + 16) != off || get_u64(r + 24) != chunk) return ORACLE_BAD_IMAGE;
    if ((int32_t)get_u32(r + 36) != device || get_u64(r + 40) != 0) return ORACLE_BAD_IMAGE;
    if (!add_ok(off, size, &end)) return ORACLE_BAD_IMAGE;
    chunk += chunks_of(size);
    prev = h;
  }
  if (chunk != nch) return ORACLE_BAD_IMAGE;
  if (payload_bytes != (n ? end : 0)) return ORACLE_BAD_IMAGE;
  rep->n_buffers = n;
  rep->payload_bytes = payload_bytes;
  rep->n_chunks = nch;
  return ORACLE_SUCCESS;
}

int oracle_restore(const uint8_t* img, size_t len, uint8_t* out_bytes, size_t out_bytes_cap,
                   uint64_t* out_handles, uint64_t* out_sizes, uint32_t* out_flags, size_t out_cap,
                   oracle_report* rep) {
  oracle_report local;
  if (!rep) rep = &local;
  /* Step r1: header + manifest */
  int st = oracle_validate(img, len, rep);
  if (st) return st;
  uint64_t n = rep->n_buffers;
  uint64_t crc_off = get_u64(img + 48), payload_off = get_u64(img + 56);
  uint64_t payload_bytes = rep->payload_bytes;
  const uint8_t* payload = img + payload_off;

  /* Step r4 (verify): every chunk's CRC, and the padding its buffer's last
   * chunk owns, before anything is handed out (all-or-nothing). */
  for (uint64_t b = 0; b < n; ++b) {
    const uint8_t* r = img + O_HEADER + O_RECORD * b;
    uint64_t h = get_u64(r), size = get_u64(r + 8), off = get_u64(r + 16), first = get_u64(r + 24);
    uint64_t nch = chunks_of(size);
    uint64_t pad_end = (b + 1 < n) ? get_u64(r + O_RECORD + 16) : payload_bytes;
    for (uint64_t k = 0; k < nch; ++k) {
      uint64_t lo = k * O_CHUNK;
      uint64_t clen = size - lo < O_CHUNK ? size - lo : O_CHUNK;
      int bad = oracle_crc32c(payload + off + lo, clen) != get_u32(img + crc_off + 4u * (first + k));
      if (k == nch - 1)
        for (uint64_t i = off + size; i < pad_end; ++i)
          if (payload[i] != 0) bad = 1;
      if (bad) {
        if (rep->n_bad_chunks == 0) {
          rep->first_bad_chunk = first + k;
          rep->first_bad_handle = h;
        }
        rep->n_bad_chunks++;
      }
    }
  }
  if (rep->n_bad_chunks) return ORACLE_CRC_MISMATCH;

  /* Steps r2/r3/r5: re-create every buffer with its bytes, in manifest order. */
  if (n > out_cap) return ORACLE_INVALID_VALUE;
  uint64_t total = 0;
  for (uint64_t b = 0; b < n; ++b) total += get_u64(img + O_HEADER + O_RECORD * b + 8);
  if (total > out_bytes_cap || (total && !out_bytes)) return ORACLE_INVALID_VALUE;
  uint64_t pos = 0;
  for (uint64_t b = 0; b < n; ++b) {
    const uint8_t* r = img + O_HEADER + O_RECORD * b;
    uint64_t size = get_u64(r + 8), off = get_u64(r + 16);
    if (out_handles) out_handles[b] = get_u64(r);
    if (out_sizes) out_sizes[b] = size;
    if (out_flags) out_flags[b] = get_u32(r + 32);
    if (size) memcpy(out_bytes + pos, payload + off, size);
    pos += size;
  }
  return ORACLE_SUCCESS;
}
