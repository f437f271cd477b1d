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

/* Span of chunk j of manifest record b (FORMAT.md "Span of a chunk"): its bytes
 * plus, for a buffer's last chunk, the padding it owns, in full-payload offsets. */
static void chunk_span(const uint8_t* img, uint64_t n, uint64_t b, uint64_t j, uint64_t full_payload,
                       uint64_t* start, uint64_t* stop) {
  const uint8_t* r = img + O_HEADER + O_RECORD * b;
  uint64_t size = get_u64(r + 8), off = get_u64(r + 16);
  *start = off + (uint64_t)O_CHUNK * j;
  if (j + 1 < chunks_of(size))
    *stop = *start + O_CHUNK;
  else
    *stop = b + 1 < n ? get_u64(r + O_RECORD + 16) : full_payload;
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
  uint32_t flags = get_u32(img + 84); /* 0 = full, 1 = incremental */
  if (get_u32(img + 8) != 1 || get_u32(img + 12) != O_HEADER || get_u32(img + 16) != O_CHUNK ||
      get_u32(img + 20) != O_ALIGN || get_u64(img + 40) != O_HEADER || flags > 1)
    return ORACLE_BAD_IMAGE;
  for (int i = 96; i < 124; ++i) {
    /* base_epoch, base_table_crc, dirty_rule, n_present */
    int used = flags == 1 && ((i >= 96 && i < 108) || (i >= 108 && i < 112) || (i >= 112 && i < 120));
    if (!used && img[i] != 0) return ORACLE_BAD_IMAGE;
  }
  if (flags == 1 && get_u32(img + 108) > 1) return ORACLE_BAD_IMAGE; /* dirty_rule 0 or 1 */
  uint64_t n = get_u64(img + 24), nch = get_u64(img + 32);
  uint64_t crc_off = get_u64(img + 48), payload_off = get_u64(img + 56);
  uint64_t payload_bytes = get_u64(img + 64), image_bytes = get_u64(img + 72);
  int32_t device = (int32_t)get_u32(img + 80);
  /* closed-form region offsets, with overflow checks */
  if (n > (UINT64_MAX - O_HEADER) / O_RECORD) return ORACLE_BAD_IMAGE;
  if (crc_off != O_HEADER + O_RECORD * n) return ORACLE_BAD_IMAGE;
  if (nch > (UINT64_MAX - crc_off) / 4u) return ORACLE_BAD_IMAGE;
  uint64_t map_bytes = flags == 1 ? nch / 8 + (nch % 8 ? 1 : 0) : 0; /* present bitmap */
  uint64_t want_payload_off;
  if (!align_ok(crc_off + 4u * nch + map_bytes, O_PAYLOAD_ALIGN, &want_payload_off)) return ORACLE_BAD_IMAGE;
  if (payload_off != want_payload_off) return ORACLE_BAD_IMAGE;
  uint64_t want_image;
  if (!add_ok(payload_off, payload_bytes, &want_image) || image_bytes != want_image) return ORACLE_BAD_IMAGE;
  if ((uint64_t)len < image_bytes) return ORACLE_BAD_IMAGE;
  if (get_u32(img + 124) != meta_crc_of(img, payload_off)) return ORACLE_BAD_IMAGE;
  for (uint64_t i = crc_off + 4u * nch + map_bytes; i < payload_off; ++i)
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
  uint64_t full_payload = n ? end : 0;
  if (flags == 0 && payload_bytes != full_payload) return ORACLE_BAD_IMAGE;
  if (flags == 1) {
    /* present bitmap: unused bits zero, popcount = n_present, spans sum to payload_bytes */
    const uint8_t* map = img + crc_off + 4u * nch;
    for (uint64_t k = nch; k < map_bytes * 8; ++k)
      if (map[k / 8] & (1u << (k % 8))) return ORACLE_BAD_IMAGE;
    uint64_t n_present = 0, sum = 0;
    for (uint64_t b = 0; b < n; ++b) {
      uint64_t nb = chunks_of(get_u64(img + O_HEADER + O_RECORD * b + 8));
      uint64_t first = get_u64(img + O_HEADER + O_RECORD * b + 24);
      for (uint64_t j = 0; j < nb; ++j) {
        if (!(map[(first + j) / 8] & (1u << ((first + j) % 8)))) continue;
        uint64_t start, stop;
        chunk_span(img, n, b, j, full_payload, &start, &stop);
        n_present++;
        sum += stop - start;
      }
    }
    if (n_present != get_u64(img + 112) || sum != payload_bytes) return ORACLE_BAD_IMAGE;
  }
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
  if (get_u32(img + 84) != 0) return ORACLE_BAD_IMAGE; /* a delta restores only through merge */
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

/* ------------------------------------------------------------------------ */
/* Incremental checkpoint (FORMAT.md "Incremental images"; PAPER.md L45      */
/* §IV-D future work: write only what was updated since the last checkpoint) */
/* ------------------------------------------------------------------------ */

static uint32_t table_crc_of(const uint8_t* img) {
  uint64_t nch = get_u64(img + 32), crc_off = get_u64(img + 48);
  return oracle_crc32c(img + crc_off, 4u * nch);
}

int oracle_checkpoint_incremental(const oracle_buffer* bufs, size_t n, int32_t device, uint64_t epoch,
                                  const uint8_t* base, size_t base_len, uint8_t* out, size_t out_cap,
                                  uint64_t* out_len) {
  return oracle_checkpoint_incremental_rule(bufs, n, device, epoch, base, base_len, NULL, 0, 0, out, out_cap,
                                            out_len);
}

/* Is chunk j of manifest record b "updated" (FORMAT.md "Present set")?
 * rule 0: its CRC32C in the table of `full` (now) differs from base's entry
 *         (reading 21);
 * rule 1: its bytes in `full` differ from its bytes in `base_full`, the full image of
 *         the base's state (reading 25) — the plain definition of L45's
 *         "updated since the last checkpoint". */
static int chunk_updated(const uint8_t* full, const uint8_t* base, const uint8_t* base_full, uint32_t rule,
                         uint64_t b, uint64_t j) {
  uint64_t crc_off = get_u64(full + 48);
  const uint8_t* r = full + O_HEADER + O_RECORD * b;
  uint64_t k = get_u64(r + 24) + j;
  if (rule == 0) return get_u32(full + crc_off + 4u * k) != get_u32(base + crc_off + 4u * k);
  uint64_t size = get_u64(r + 8), off = get_u64(r + 16);
  uint64_t lo = j * O_CHUNK;
  uint64_t len = size - lo < O_CHUNK ? size - lo : O_CHUNK;
  return memcmp(full + get_u64(full + 56) + off + lo, base_full + get_u64(base_full + 56) + off + lo, len) != 0;
}

int oracle_checkpoint_incremental_rule(const oracle_buffer* bufs, size_t n, int32_t device, uint64_t epoch,
                                       const uint8_t* base, size_t base_len, const uint8_t* base_full,
                                       size_t base_full_len, uint32_t dirty_rule, uint8_t* out, size_t out_cap,
                                       uint64_t* out_len) {
  oracle_report brep, frep;
  int st;
  if (!out_len || dirty_rule > 1) return ORACLE_INVALID_VALUE;
  /* the base must be a valid image (full or incremental) */
  st = oracle_validate(base, base_len, &brep);
  if (st) return st;
  if (dirty_rule == 1) {
    /* base_full: a valid full image of the base's state: same epoch, manifest and
     * CRC table as the base */
    if (!base_full || oracle_validate(base_full, base_full_len, &frep) || get_u32(base_full + 84) != 0)
      return ORACLE_INVALID_VALUE;
    uint64_t bco = get_u64(base + 48), bnch = get_u64(base + 32);
    if (get_u64(base_full + 88) != get_u64(base + 88) || get_u64(base_full + 32) != bnch ||
        get_u64(base_full + 48) != bco || memcmp(base_full + O_HEADER, base + O_HEADER, bco + 4u * bnch - O_HEADER) != 0)
      return ORACLE_INVALID_VALUE;
  }

  /* Step 1: the full image of the registry now (the definition of its content). */
  oracle_layout L;
  st = oracle_layout_of(bufs, n, &L);
  if (st) return st;
  uint8_t* full = (uint8_t*)malloc(L.image_bytes ? L.image_bytes : 1);
  if (!full) return ORACLE_OUT_OF_HOST_MEMORY;
  st = oracle_checkpoint(bufs, n, device, epoch, full, L.image_bytes);
  if (st) {
    free(full);
    return st;
  }

  /* Step 2: same layout as the base? (manifest, chunk count, device) — else full. */
  int same = get_u64(base + 32) == L.n_chunks && get_u64(base + 48) == L.crc_off &&
             get_u32(base + 80) == (uint32_t)device &&
             memcmp(base + O_HEADER, full + O_HEADER, L.crc_off - O_HEADER) == 0;
  if (!same) {
    *out_len = L.image_bytes;
    if (out_cap < L.image_bytes || !out) {
      free(full);
      return ORACLE_INVALID_VALUE;
    }
    memcpy(out, full, L.image_bytes);
    free(full);
    return ORACLE_SUCCESS;
  }

  /* Step 3: chunk k is present iff it was updated (chunk_updated, by the rule). */
  uint64_t nch = L.n_chunks, crc_off = L.crc_off;
  uint64_t map_bytes = nch / 8 + (nch % 8 ? 1 : 0);
  uint64_t n_present = 0, payload = 0;
  for (uint64_t b = 0; b < L.n_buffers; ++b) {
    uint64_t nb = chunks_of(get_u64(full + O_HEADER + O_RECORD * b + 8));
    for (uint64_t j = 0; j < nb; ++j) {
      if (!chunk_updated(full, base, base_full, dirty_rule, b, j)) continue;
      uint64_t start, stop;
      chunk_span(full, L.n_buffers, b, j, L.payload_bytes, &start, &stop);
      n_present++;
      payload += stop - start;
    }
  }

  /* Step 4: layout of the delta. */
  uint64_t payload_off = 0;
  if (!align_ok(crc_off + 4u * nch + map_bytes, O_PAYLOAD_ALIGN, &payload_off)) {
    free(full);
    return ORACLE_INVALID_VALUE;
  }
  uint64_t image_bytes = payload_off + payload;
  *out_len = image_bytes;
  if (out_cap < image_bytes || !out) {
    free(full);
    return ORACLE_INVALID_VALUE;
  }
  memset(out, 0, image_bytes);

  /* Step 5: header (the full image's, then the incremental fields), manifest,
   * CRC table of every chunk, bitmap, and the present spans in ascending order. */
  memcpy(out, full, O_HEADER);
  put_u64(out + 56, payload_off);
  put_u64(out + 64, payload);
  put_u64(out + 72, image_bytes);
  put_u32(out + 84, 1);
  put_u64(out + 96, get_u64(base + 88));
  put_u32(out + 104, table_crc_of(base));
  put_u32(out + 108, dirty_rule);
  put_u64(out + 112, n_present);
  memcpy(out + O_HEADER, full + O_HEADER, crc_off - O_HEADER);
  memcpy(out + crc_off, full + crc_off, 4u * nch);
  uint8_t* map = out + crc_off + 4u * nch;
  uint64_t pos = payload_off;
  for (uint64_t b = 0; b < L.n_buffers; ++b) {
    uint64_t nb = chunks_of(get_u64(full + O_HEADER + O_RECORD * b + 8));
    uint64_t first = get_u64(full + O_HEADER + O_RECORD * b + 24);
    for (uint64_t j = 0; j < nb; ++j) {
      uint64_t k = first + j;
      if (!chunk_updated(full, base, base_full, dirty_rule, b, j)) continue;
      uint64_t start, stop;
      chunk_span(full, L.n_buffers, b, j, L.payload_bytes, &start, &stop);
      map[k / 8] |= (uint8_t)(1u << (k % 8));
      memcpy(out + pos, full + L.payload_off + start, stop - start);
      pos += stop - start;
    }
  }
  put_u32(out + 124, meta_crc_of(out, payload_off));
  free(full);
  return ORACLE_SUCCESS;
}

int oracle_merge(const uint8_t* full, size_t full_len, const uint8_t* delta, size_t delta_len, uint8_t* out,
                 size_t out_cap, uint64_t* out_len) {
  oracle_report fr, dr;
  if (!out_len) return ORACLE_INVALID_VALUE;
  if (oracle_validate(full, full_len, &fr) || oracle_validate(delta, delta_len, &dr)) return ORACLE_BAD_IMAGE;
  if (get_u32(full + 84) != 0 || get_u32(delta + 84) != 1) return ORACLE_BAD_IMAGE;
  /* the link: base epoch, base CRC-table CRC, identical manifest and device */
  uint64_t crc_off = get_u64(full + 48), nch = get_u64(full + 32);
  if (get_u64(delta + 96) != get_u64(full + 88) || get_u32(delta + 104) != table_crc_of(full) ||
      get_u64(delta + 32) != nch || get_u64(delta + 48) != crc_off || get_u32(delta + 80) != get_u32(full + 80) ||
      memcmp(delta + O_HEADER, full + O_HEADER, crc_off - O_HEADER) != 0)
    return ORACLE_BAD_IMAGE;
  uint64_t image_bytes = get_u64(full + 72), payload_off = get_u64(full + 56), payload_bytes = get_u64(full + 64);
  *out_len = image_bytes;
  if (out_cap < image_bytes || !out) return ORACLE_INVALID_VALUE;
  /* F's bytes, then D's header with flags 0 and the full-image fields, D's CRC table */
  memcpy(out, full, image_bytes);
  memcpy(out, delta, O_HEADER);
  put_u32(out + 84, 0);
  put_u64(out + 56, payload_off);
  put_u64(out + 64, payload_bytes);
  put_u64(out + 72, image_bytes);
  memset(out + 96, 0, 28);
  memcpy(out + crc_off, delta + crc_off, 4u * nch);
  /* every present chunk's span replaced by D's, in ascending order */
  const uint8_t* map = delta + crc_off + 4u * nch;
  uint64_t n = get_u64(full + 24), pos = get_u64(delta + 56);
  for (uint64_t b = 0; b < n; ++b) {
    uint64_t nb = chunks_of(get_u64(full + O_HEADER + O_RECORD * b + 8));
    uint64_t first = get_u64(full + O_HEADER + O_RECORD * b + 24);
    for (uint64_t j = 0; j < nb; ++j) {
      uint64_t k = first + j;
      if (!(map[k / 8] & (1u << (k % 8)))) continue;
      uint64_t start, stop;
      chunk_span(full, n, b, j, payload_bytes, &start, &stop);
      memcpy(out + payload_off + start, delta + pos, stop - start);
      pos += stop - start;
    }
  }
  put_u32(out + 124, meta_crc_of(out, payload_off));
  return ORACLE_SUCCESS;
}
