// checl_internal.h — internal types of libchecl (product code; no oracle code).
//
// Format constants are FORMAT.md's; the CRC32C arithmetic is GF(2)[x] modulo the
// Castagnoli polynomial in the reflected bit order CRC registers use (bit 31 of a
// 32-bit value is the coefficient of x^0, bit 0 that of x^31).
#pragma once

#include <cstddef>
#include <cstdint>

#ifdef __CUDACC__
#define CHECL_HD __host__ __device__ __forceinline__
#else
#define CHECL_HD inline
#endif

namespace checl {

constexpr uint32_t kChunkBytes = 65536;     // FORMAT.md chunk_bytes
constexpr uint32_t kBufferAlign = 256;      // payload_align
constexpr uint32_t kHeaderBytes = 128;      // header_bytes
constexpr uint32_t kRecordBytes = 48;       // manifest record
constexpr uint32_t kPayloadAlign = 4096;    // payload_off alignment
constexpr uint32_t kPolyRefl = 0x82F63B78u; // x^32 + ... (Castagnoli), low terms, reflected
constexpr uint32_t kOne = 0x80000000u;      // the polynomial 1 (x^0) in reflected order
constexpr uint32_t kX = 0x40000000u;        // the polynomial x

// One chunk of the flat work list (16 bytes). `ptr` is the registered buffer's
// address of the chunk (pack: source; restore: destination). The chunk's payload
// offset is img_off_256 * 256 (chunks start on 256-byte boundaries: buffers are
// 256-aligned and chunks are 64 KiB apart inside a buffer). len in [1, 65536];
// pad = zero bytes owned after the chunk (< 256, non-zero only for a buffer's
// last chunk).
struct ChunkDesc {
  uint64_t ptr;
  uint32_t img_off_256;
  uint32_t len_pad;  // len | pad << 24
};
static_assert(sizeof(ChunkDesc) == 16, "ChunkDesc is 16 bytes");

// One buffer of a plan (48 bytes); the GPU expands records into ChunkDescs.
// ptr = the buffer's device address (pack: source; restore: destination),
// off = payload offset (256-aligned), first_chunk = global index of its chunk 0,
// first_round = global index of its first 4 KiB round (rounds of the chunk list
// enumerated in order: a chunk of len bytes has ceil(len / 4096) rounds).
struct BufferRecord {
  uint64_t ptr, size, off, first_chunk, first_round, reserved;
};
static_assert(sizeof(BufferRecord) == 48, "BufferRecord is 48 bytes");

CHECL_HD uint32_t desc_len(const ChunkDesc& d) { return d.len_pad & 0x1FFFFu; }
CHECL_HD uint32_t desc_pad(const ChunkDesc& d) { return d.len_pad >> 24; }
CHECL_HD uint32_t make_len_pad(uint32_t len, uint32_t pad) { return len | (pad << 24); }

// a * x mod P: one zero bit through the CRC register.
CHECL_HD uint32_t gf_mulx(uint32_t a) { return (a >> 1) ^ ((a & 1u) ? kPolyRefl : 0u); }

// a * x^-1 mod P (x is invertible: P has a constant term). Inverse of gf_mulx:
// bit 31 of gf_mulx(a) equals bit 0 of a because kPolyRefl has bit 31 set.
CHECL_HD uint32_t gf_divx(uint32_t r) {
  uint32_t b = r >> 31;
  return ((r ^ (b ? kPolyRefl : 0u)) << 1) | b;
}

// a * b mod P.
CHECL_HD uint32_t gf_mul(uint32_t a, uint32_t b) {
  uint32_t p = 0;
  for (int i = 0; i < 32; ++i) {
    if (a & (kOne >> i)) p ^= b;
    b = gf_mulx(b);
  }
  return p;
}

// x^(2^k) mod P.
CHECL_HD uint32_t gf_x_pow2k(int k) {
  uint32_t r = kX;
  for (int i = 0; i < k; ++i) r = gf_mul(r, r);
  return r;
}

// x^(8n) mod P (shift of a CRC register over n zero bytes), square-and-multiply.
CHECL_HD uint32_t gf_x8n(uint64_t n) {
  uint32_t r = kOne, sq = gf_mul(kX, kX);  // x^2
  sq = gf_mul(sq, sq);                     // x^4
  sq = gf_mul(sq, sq);                     // x^8
  while (n) {
    if (n & 1u) r = gf_mul(r, sq);
    sq = gf_mul(sq, sq);
    n >>= 1;
  }
  return r;
}

// Kernel geometry: one warp per chunk, rounds of 4 KiB of
// contiguous bytes, lane l CRCs the 128-byte segment 32r + l of round r.
constexpr int kRoundBytes = 4096;
constexpr int kSegBytes = 128;                   // per lane per round
constexpr int kRowPitch = kSegBytes + 16;        // padded smem row: conflict-free LDS.128
#ifndef CHECL_WARPS
#define CHECL_WARPS 10  // measured best of 4..16 (tools/exp_sweep2.sh): fewer warps contend less for the LSU/MIO
#endif
constexpr int kWarpsPerCta = CHECL_WARPS;
constexpr int kThreadsPerCta = kWarpsPerCta * 32;
constexpr int kFoldLevels = 5;
#ifndef CHECL_PREFETCH
#define CHECL_PREFETCH 1
#endif
constexpr int kPrefetch = CHECL_PREFETCH;  // rounds of loads in flight per warp (registers)
static_assert(kPrefetch == 1 || kPrefetch == 2, "prefetch depth 1 or 2");

// What one launch does with each chunk of its list (the same data path serves
// every step that streams chunks):
//   kOpPack   a3  K1: buffer -> image, CRC -> table, zero the owned padding
//   kOpVerify r4  K2: image -> buffer, CRC == table and owned padding zero
//   kOpCrc    f1  CRC only (no copy): the table of the current contents
//   kOpCheck  f1  CRC only, compared with the table (in-place verify of a restore)
//   kOpCopy   f1  buffer -> image without CRC (gather of an incremental image)
//   kOpScatter f1 image -> buffer without CRC, owned padding included (a delta's
//                 chunks over a restored base; the result is checked by kOpCheck)
enum : int { kOpPack = 0, kOpVerify = 1, kOpCrc = 2, kOpCheck = 3, kOpCopy = 4, kOpScatter = 5 };

// Lane-private lookup tables, computed once per device into global memory and
// bulk-copied (cp.async.bulk) into shared memory by every CTA. Word offsets:
constexpr int kTabWords = 4 * 256 * 32;          // slicing-by-4, 128 KiB
constexpr int kHornerWords = 8 * 16 * 32;       // x^(8*3968) nibble tables, 16 KiB
constexpr int kFoldWords = kFoldLevels * 8 * 16; // fold nibble tables, 2.5 KiB
constexpr int kPosWords = 8 * 16 * 32;          // sweep: lane-position nibble tables, 16 KiB
constexpr int kUnitWords = 16 * 32;             // sweep: x^(8*4096*k) * x^i, 2 KiB
// TMA kernel (column CRC): lane l takes word l of every 128-byte row
// in kColChains independent chains (chain c: the rows = c mod kColChains), so a
// chain's step is v -> v * x^(8*128*kColChains) (slicing-by-4 tables of that shift,
// same lane-private layout); a lane's chains are combined with the shift x^(-1024)
// (fold level kFoldLevels) and the lanes with shifts x^(-32*2^k).
#ifndef CHECL_COL_CHAINS
#define CHECL_COL_CHAINS 4
#endif
constexpr int kColChains = CHECL_COL_CHAINS;
static_assert(kColChains == 1 || kColChains == 2 || kColChains == 4 || kColChains == 8, "chains divide 32 rows");
constexpr int kColFoldLevels = kFoldLevels + 1;  // + x^(-32*32): one row of the tile
constexpr int kColWords = 4 * 256 * 32;          // 128 KiB
constexpr int kColFoldWords = kColFoldLevels * 8 * 16;  // 3 KiB
constexpr int kTabOff = 0;
constexpr int kHornerOff = kTabOff + kTabWords;
constexpr int kFoldOff = kHornerOff + kHornerWords;
constexpr int kPosOff = kFoldOff + kFoldWords;
constexpr int kUnitOff = kPosOff + kPosWords;
constexpr int kColOff = kUnitOff + kUnitWords;
constexpr int kColFoldOff = kColOff + kColWords;
constexpr int kTableWords = kColFoldOff + kColFoldWords;
static_assert((kPosOff * 4) % 16 == 0 && (kFoldOff * 4 + kFoldWords * 4) % 16 == 0, "bulk-copy alignment");

// Constants the table builder needs (computed on the host).
struct TableParams {
  uint32_t fold[kFoldLevels];  // x^(8 * 128 * 2^k) mod P
  uint32_t horner;             // x^(8 * (kRoundBytes - kSegBytes)) mod P
  uint32_t lanepow[32];        // x^(8 * 128 * (31 - l)) mod P
  uint32_t unitpow[16];        // x^(8 * 4096 * k) mod P
  uint32_t col_shift;          // x^(8 * 128 * kColChains) mod P
  uint32_t col_fold[kColFoldLevels];  // x^(-32 * 2^k) mod P
};

// Parameters of one launch over the chunk range [c0, c1) of `desc`. Payload byte
// o of the image lives at image + o - image_base for the chunks of this launch.
struct LaunchParams {
  const ChunkDesc* desc;
  uint64_t c0, c1;
  uint8_t* image;           // pack/copy: destination slot; verify: source (may be a peer address)
  uint64_t image_base;      // payload offset that maps to image[0]
  uint32_t* crc;            // pack/crc: output table (global chunk index); verify/check: reference table
  uint32_t* crc_mirror;     // pack/crc: optional second copy of the table in mapped pinned host memory
  const uint32_t* inv_z;    // kRoundBytes entries, x^(-8z) mod P
  const uint32_t* tables;   // kTableWords words (build_tables)
  const uint32_t* round_base;  // per chunk: global index of its round 0 (+ one past the end);
                               // nullptr: the launch runs the grid-stride kernels
  unsigned long long* status;  // verify/check: [0] = first bad chunk (atomicMin), [1] = bad count,
                               // [2] = CTAs finished (publishing launches)
  // verify/check: the launch that closes a restore copies status[0..1] here (mapped
  // pinned host memory) from its last CTA and resets status to {~0, 0, 0}; nullptr:
  // status is left as accumulated
  unsigned long long* status_host;
  // the image is not this GPU's HBM: 1 = a peer GPU's memory (NVLink), 2 = mapped
  // pinned host memory (PCIe). Rounds from it take the register path (16-byte loads),
  // except peer images when remote_bulk is set (experiments build, CHECL_PEER_BULK=1:
  // cp.async.bulk straight from the peer's HBM, for A/B on a box with two GPUs)
  int image_remote;
  int remote_bulk;
  // diagnostics (CHECL_WARP_TRACE): per warp {start, tables ready, end, smid}
  unsigned long long* warp_trace;
  // balanced / TMA kernels: the first static_permille/1000 of the rounds go to the
  // warps in equal contiguous stretches, the rest in blocks of dyn_block rounds to
  // whichever warp is free, from the counter work[0] (work[1] counts finished CTAs;
  // the last one resets both: zero between launches). work == nullptr: all static.
  unsigned long long* work;
  uint32_t static_permille, dyn_block;
  // sweep kernel (one 4 KiB unit per warp-iteration)
  unsigned long long* unit_acc;  // per chunk: low 32 = XOR of unit terms, high = finished-unit mask (zeroed)
};

}  // namespace checl
