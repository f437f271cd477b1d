/*
 * checl_oracle.h — TEST INFRASTRUCTURE ONLY.
 *
 * The plain, slow, obviously-correct CPU definition of the CheCL device-state
 * snapshot (checkpoint = pack + per-chunk CRC32C, restore = validate + verify +
 * scatter). Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library. The product (libchecl.so under
 * paper_conf_ipps_takizawakskk11_b200/) shares no code, header, table or
 * constant generator with it, and neither includes the other.
 *
 * Paper anchors (PAPER.md line, section):
 *   L16 §III-C checkpoint step 2 "Copy all the user data in the device memory to
 *       the host memory"; restart step 3 "Send the user data back to the device".
 *   L19 §III-C "a database is managed to hold the pointers to all CheCL objects
 *       ... CheCL copies the data of every OpenCL object to the host memory".
 *   L15 §III-B the CheCL handle stays stable while the real handle changes.
 * The byte layout and the CRC32C chunking come from BASELINE.json north_star and
 * are frozen in FORMAT.md (the paper is silent on both).
 */
#ifndef CHECL_ORACLE_H
#define CHECL_ORACLE_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Status values mirror include/checl.h numerically (written out again here on
 * purpose: the oracle includes nothing from the product). */
#define ORACLE_SUCCESS 0
#define ORACLE_INVALID_VALUE (-1)
#define ORACLE_OUT_OF_HOST_MEMORY (-5)
#define ORACLE_BAD_IMAGE (-6)
#define ORACLE_CRC_MISMATCH (-7)

/* CRC32C by the bit-serial definition: reflected poly 0x82F63B78, init and
 * final XOR 0xFFFFFFFF (FORMAT.md "Payload and chunks"). */
uint32_t oracle_crc32c_bitwise(const uint8_t* p, size_t n);
/* Same function, Sarwate byte-at-a-time with a 256-entry table that is built at
 * first use from oracle_crc32c_bitwise's shift rule. */
uint32_t oracle_crc32c(const uint8_t* p, size_t n);

/* One live registry entry ("CheCL object" of a cl_mem, L15/L19): handle id,
 * size, flags, device, and a host copy of its bytes. */
typedef struct {
  uint64_t handle;
  uint64_t size;
  uint32_t flags;
  int32_t device;
  const uint8_t* data; /* size bytes (may be NULL when size == 0) */
} oracle_buffer;

/* Layout of the image the given registry produces (FORMAT.md). Buffers may be
 * given in any order; the layout sorts them by handle. */
typedef struct {
  uint64_t n_buffers, n_chunks, crc_off, payload_off, payload_bytes, image_bytes;
} oracle_layout;

int oracle_layout_of(const oracle_buffer* bufs, size_t n, oracle_layout* out);

/* Checkpoint (L16 steps 1-2, L19): writes the whole image into out[0, image_bytes).
 * out_cap must be >= image_bytes. Returns ORACLE_INVALID_VALUE on duplicate or
 * zero handles, or when out_cap is too small. */
int oracle_checkpoint(const oracle_buffer* bufs, size_t n, int32_t device,
                      uint64_t epoch, uint8_t* out, size_t out_cap);

/* Restore report (same fields as checl_report). first_bad_* = UINT64_MAX / 0
 * when there is no bad chunk. */
typedef struct {
  uint64_t n_buffers, payload_bytes, n_chunks, n_bad_chunks;
  uint64_t first_bad_handle, first_bad_chunk;
} oracle_report;

/* Header + manifest validation only (FORMAT.md "Validation order" step 1), for
 * full (flags 0) and incremental (flags 1) images. */
int oracle_validate(const uint8_t* img, size_t len, oracle_report* rep);

/* Restart (L16 restart steps 2-3) of a full image (an incremental image alone is
 * ORACLE_BAD_IMAGE: chains restore through oracle_merge): validate, verify every chunk, and on success
 * copy every buffer's bytes, in manifest order, into out_bytes (concatenated,
 * no padding) and the records into out_handles / out_sizes / out_flags (each
 * n_buffers long). Capacities are checked: ORACLE_INVALID_VALUE when too small.
 * On CRC_MISMATCH nothing is written to the outputs. */
int oracle_restore(const uint8_t* img, size_t len, uint8_t* out_bytes,
                   size_t out_bytes_cap, uint64_t* out_handles, uint64_t* out_sizes,
                   uint32_t* out_flags, size_t out_cap, oracle_report* rep);

/* ---- Incremental images (FORMAT.md "Incremental images") ----
 * PAPER.md L45 §IV-D (future work): "only the OpenCL objects updated since the
 * last checkpoint need to be written". Unit = 64 KiB chunk; updated = its CRC32C
 * differs from the base image's entry (reading 21), or, with dirty rule 1,
 * its bytes differ from the base state's (reading 25). */

/* Writes into out[0, *out_len) the incremental image of the registry at `epoch`
 * relative to `base` (a full or incremental image). When base's manifest, chunk
 * count or device differ from this registry's, the output is the full image
 * (flags 0) instead. ORACLE_BAD_IMAGE if base does not validate;
 * ORACLE_INVALID_VALUE if out_cap < the size needed (*out_len is set to it). */
int oracle_checkpoint_incremental(const oracle_buffer* bufs, size_t n, int32_t device, uint64_t epoch,
                                  const uint8_t* base, size_t base_len, uint8_t* out, size_t out_cap,
                                  uint64_t* out_len);

/* Same, with the rule that decides which chunks were updated (FORMAT.md "Present
 * set", written to the delta's dirty_rule field):
 *   0: the chunk's CRC32C differs from base's CRC-table entry (reading 21;
 *      base_full unused, may be NULL) — oracle_checkpoint_incremental;
 *   1: the chunk's bytes differ from its bytes in the base's state (DESIGN.md reading
 *      25). base_full = the full image of that state: base itself when base is full,
 *      else merge(...merge(F, D1)..., base). It must validate, be full, and carry
 *      base's epoch, manifest and CRC table (ORACLE_INVALID_VALUE otherwise).
 * ORACLE_INVALID_VALUE also for a rule > 1. */
int oracle_checkpoint_incremental_rule(const oracle_buffer* bufs, size_t n, int32_t device, uint64_t epoch,
                                       const uint8_t* base, size_t base_len, const uint8_t* base_full,
                                       size_t base_full_len, uint32_t dirty_rule, uint8_t* out, size_t out_cap,
                                       uint64_t* out_len);

/* merge(F, D): the full image of D's epoch from full image F and delta D whose
 * link names F. ORACLE_BAD_IMAGE if either does not validate, F is not full, D is
 * not incremental, or the link (base epoch, base table CRC, manifest) does not
 * match; ORACLE_INVALID_VALUE if out_cap is too small (*out_len set). */
int oracle_merge(const uint8_t* full, size_t full_len, const uint8_t* delta, size_t delta_len, uint8_t* out,
                 size_t out_cap, uint64_t* out_len);

#ifdef __cplusplus
}
#endif
#endif
