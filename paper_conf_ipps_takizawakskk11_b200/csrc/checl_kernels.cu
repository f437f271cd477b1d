// checl_kernels.cu — sm_100a kernels of the CheCL snapshot hot path.
//
//  K1 pack_gather_crc  (checkpoint step 2, §III-C; north_star "gather
//     ... into one contiguous checkpoint image carrying a per-64 KiB CRC32C")
//  K2 verify_scatter   (restart step 3, L16 §III-C; north_star "every chunk is
//     CRC-verified, and its bytes are scattered into freshly re-created buffers")
//  f1 incremental: CRC-only pass, present-set scan + compaction, gather / scatter
//  plan expansion (a2 / r2), lookup-table builder, K6 debug fill / compare
//
// K1, K2 and the incremental passes are one data path templated on the op
// (kOp* in checl_internal.h) in three work splits: balanced_kernel (default: equal
// contiguous stretches of 4 KiB rounds per warp), snapshot_kernel (one warp per
// chunk, grid-stride) and sweep_kernel (4 KiB units, grid-stride). A chunk is moved
// in rounds of 4 KiB of contiguous bytes: eight coalesced 16-byte global loads per
// lane (each warp instruction = 512 contiguous bytes), a coalesced 16-byte store of
// the same registers to the destination, and a transposition through a padded
// 32 x 144 B shared tile so that lane l then reads "its" 128-byte segment (segment
// 32r + l of the chunk) with conflict-free 16-byte shared loads. Each lane runs a
// slicing-by-4 CRC over its segments, carrying its register from round to round
// with a Horner step (multiply by x^(8*3968) mod P: skip the other 31 lanes'
// segments). Lookup tables are lane-private in shared memory (every lane reads its
// own bank: conflict-free on any data). At the end the 32 lane registers are folded
// with a 5-level warp-shuffle tree (multiply by x^(8*128*2^k)); a chunk whose length
// is not a multiple of 4 KiB was CRC'd zero-padded and is corrected with one
// multiply by x^(-8 zp). The next round's loads are issued before the current
// round's CRC so that HBM latency hides under the table lookups.
// DESIGN.md §5 derives the resource budget and the GF(2) identities.
#include <cstdlib>

#include <cuda_runtime.h>

#include "checl_internal.h"

namespace checl {

constexpr int kStageBytes = 32 * kRowPitch;      // per warp
constexpr int kSnapTabWords = kPosOff;           // snapshot kernel: tab | horner | fold
constexpr size_t kTileOff = (size_t)kSnapTabWords * 4;
constexpr size_t kMbarOff = kTileOff + (size_t)kWarpsPerCta * kStageBytes;
constexpr size_t kSmemBytes = kMbarOff + 16;
static_assert(kSmemBytes <= 232448, "fits the 227 KiB opt-in shared memory");

// Global loads are volatile asm: a plain asm has no side effects for the compiler,
// which then may execute it speculatively outside its branch (it hoisted the next
// part's first loads above their `if`, with a null source: an illegal address).
__device__ __forceinline__ uint4 ld_stream_v4(const void* p) {
  uint4 r;
  asm volatile("ld.global.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
      : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
      : "l"(p));
  return r;
}

// One 16-byte global store. Written as a PTX vector store: with a plain uint4
// assignment ptxas split the balanced kernel's verify stores into 64- and 32-bit
// pieces (register tuples it could not keep aligned), 2.7x the store requests.
__device__ __forceinline__ void st_stream_v4(void* p, uint4 v) {
  asm volatile("st.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}

__device__ __forceinline__ uint32_t ld_stream_u32(const void* p) {
  uint32_t r;
  asm volatile("ld.global.L1::no_allocate.u32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}

// n (< 16) bytes at p, zero-extended into a 16-byte granule.
__device__ __forceinline__ uint4 ld_partial(const uint8_t* p, uint32_t n) {
  uint32_t w[4] = {0u, 0u, 0u, 0u};
#pragma unroll
  for (int i = 0; i < 16; ++i)
    if ((uint32_t)i < n) w[i >> 2] |= (uint32_t)p[i] << (8 * (i & 3));
  return make_uint4(w[0], w[1], w[2], w[3]);
}

// A full 16-byte granule at any alignment: mode 0 = 16-byte aligned, 1 = 4-byte
// aligned, 2 = byte aligned (registered tensor views may carry a storage offset).
__device__ __forceinline__ uint4 ld_granule(const uint8_t* p, int mode) {
  if (mode == 0) return ld_stream_v4(p);
  if (mode == 1)
    return make_uint4(ld_stream_u32(p), ld_stream_u32(p + 4), ld_stream_u32(p + 8), ld_stream_u32(p + 12));
  return ld_partial(p, 16);
}

__device__ __forceinline__ void st_partial(uint8_t* p, uint4 v, uint32_t n) {
  const uint32_t w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
  for (int i = 0; i < 16; ++i)
    if ((uint32_t)i < n) p[i] = (uint8_t)(w[i >> 2] >> (8 * (i & 3)));
}

// Lane-private slicing-by-4 tables, laid out as two "super-tables" of 256 rows x
// 256 B: row e of A = [T3[e] x 32 lanes | T2[e] x 32 lanes], row e of B = [T1[e] |
// T0[e]]. The byte address of T_k[e] for lane l is base + e*256 + half*128 + 4l, so
// one PRMT builds the whole in-table offset from the data word and l4 = 4l:
// result byte 0 = l4, byte 1 = the selected data byte, bytes 2-3 = 0. Every lane
// reads its own bank (bank = l): conflict-free on any data.
__device__ __forceinline__ uint32_t tab_ld(const uint8_t* tb, uint32_t off) {
  return *reinterpret_cast<const uint32_t*>(tb + off);
}

// One slicing-by-4 step over the little-endian word w.
__device__ __forceinline__ uint32_t crc_step4(uint32_t crc, uint32_t w, const uint8_t* tb, uint32_t l4) {
  const uint32_t x = crc ^ w;
  return tab_ld(tb, __byte_perm(x, l4, 0x5504)) ^ tab_ld(tb + 128, __byte_perm(x, l4, 0x5514)) ^
         tab_ld(tb + 65536, __byte_perm(x, l4, 0x5524)) ^ tab_ld(tb + 65536 + 128, __byte_perm(x, l4, 0x5534));
}

__device__ __forceinline__ uint32_t crc_step1(uint32_t crc, uint32_t b, const uint8_t* tb, uint32_t l4) {
  return (crc >> 8) ^ tab_ld(tb + 65536 + 128, __byte_perm(crc ^ b, l4, 0x5504));
}

__device__ __forceinline__ uint32_t crc_step16(uint32_t crc, uint4 q, const uint8_t* tb, uint32_t l4) {
  crc = crc_step4(crc, q.x, tb, l4);
  crc = crc_step4(crc, q.y, tb, l4);
  crc = crc_step4(crc, q.z, tb, l4);
  return crc_step4(crc, q.w, tb, l4);
}

// f * x^(8*128*2^level) mod P via 8 nibble lookups (shared table, once per chunk).
__device__ __forceinline__ uint32_t fold_mul(uint32_t f, const uint32_t* ft) {
  uint32_t r = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) r ^= ft[j * 16 + ((f >> (4 * j)) & 15u)];
  return r;
}

// s * x^(8*3968) mod P (advance a lane's register over the 31 segments of the
// other lanes) via 8 lane-private nibble lookups: entry (j, v) of lane l at byte
// j*2048 + v*128 + 4l, bank = l.
__device__ __forceinline__ uint32_t horner_mul(uint32_t s, const uint8_t* hb, uint32_t l4) {
  uint32_t r = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) r ^= tab_ld(hb + j * 2048, (((s >> (4 * j)) & 15u) << 7) | l4);
  return r;
}

// What each op does (kOp* in checl_internal.h).
template <int kOp>
struct OpT {
  static constexpr bool kSrcImg = kOp == kOpVerify || kOp == kOpScatter;  // read the image, write the buffer
  static constexpr bool kStore = kOp == kOpPack || kOp == kOpVerify || kOp == kOpCopy || kOp == kOpScatter;
  static constexpr bool kCrc = kOp != kOpCopy && kOp != kOpScatter;
  static constexpr bool kCompare = kOp == kOpVerify || kOp == kOpCheck;  // vs table + owned padding zero
  static constexpr bool kZeroPad = kOp == kOpPack || kOp == kOpCopy;     // destination is the image
  static constexpr bool kCopyPad = kOp == kOpScatter;                    // padding copied as is
  static constexpr bool kExactTail = kOp == kOpVerify || kOp == kOpScatter;  // destination is a buffer
};

__device__ __forceinline__ uint32_t warp_xor(uint32_t v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v ^= __shfl_xor_sync(0xFFFFFFFFu, v, o);
  return v;
}

__device__ __forceinline__ uint32_t smem_addr(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// Bulk-copies `n` regions of the global table image into shared memory (one
// elected thread issues cp.async.bulk, everyone waits on one mbarrier). Sizes and
// addresses are multiples of 16.
struct TableCopy {
  uint32_t dst_off, src_word, bytes;
};
__device__ __forceinline__ void wait_tables(uint64_t* mbar) {
  asm volatile(
      "{\n .reg .pred p;\n WAIT_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n"
      " @!p bra WAIT_%=;\n}" ::"r"(smem_addr(mbar))
      : "memory");
}

// kWait = false: the caller overlaps its first global loads with the table copy
// and calls wait_tables before the first lookup.
template <int N, bool kWait = true>
__device__ __forceinline__ void load_tables(uint8_t* smem, const uint32_t* gtab, const TableCopy (&cp)[N],
                                            uint64_t* mbar) {
  const uint32_t mb = smem_addr(mbar);
  if (threadIdx.x == 0) {
    uint32_t total = 0;
#pragma unroll
    for (int i = 0; i < N; ++i) total += cp[i].bytes;
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(mb) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"(total) : "memory");
#pragma unroll
    for (int i = 0; i < N; ++i) {
      for (uint32_t o = 0; o < cp[i].bytes; o += 32768u) {
        const uint32_t n = cp[i].bytes - o < 32768u ? cp[i].bytes - o : 32768u;
        asm volatile(
            "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                smem_addr(smem + cp[i].dst_off + o)),
            "l"(reinterpret_cast<const uint8_t*>(gtab + cp[i].src_word) + o), "r"(n), "r"(mb)
            : "memory");
      }
    }
  }
  __syncthreads();  // the barrier is initialised before anyone waits on it
  if (kWait) wait_tables(mbar);
}

// Loads granule set of round `r` (8 x 16 B per lane) of a chunk of `len` bytes.
__device__ __forceinline__ void load_round(uint4 (&v)[8], const uint8_t* src, uint32_t len, int mode, int r,
                                           uint32_t lane_off) {
  const uint32_t base = (uint32_t)r * kRoundBytes + lane_off;
  if (mode == 0 && (uint32_t)(r + 1) * kRoundBytes <= len) {  // warp-uniform fast path
    const uint8_t* s = src + base;
#pragma unroll
    for (int i = 0; i < 8; ++i) v[i] = ld_stream_v4(s + i * 4 * kSegBytes);
  } else {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const uint32_t o = base + (uint32_t)i * 4 * kSegBytes;
      if (o + 16 <= len)
        v[i] = ld_granule(src + o, mode);
      else if (o < len)
        v[i] = ld_partial(src + o, len - o);
      else
        v[i] = make_uint4(0u, 0u, 0u, 0u);  // past the chunk: CRC'd as zeros, corrected at the end
    }
  }
}

// Stores round r to the destination (if the op stores) and into the warp's tile.
template <int kOp>
__device__ __forceinline__ void store_round(const uint4 (&v)[8], uint8_t* dst, uint32_t len, int r, uint32_t lane_off,
                                            uint8_t* tile_w) {
  using O = OpT<kOp>;
  const uint32_t base = (uint32_t)r * kRoundBytes + lane_off;
  if ((uint32_t)(r + 1) * kRoundBytes <= len) {  // warp-uniform fast path
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      if (O::kStore) st_stream_v4(dst + base + i * 4 * kSegBytes, v[i]);
      if (O::kCrc) *reinterpret_cast<uint4*>(tile_w + i * 4 * kRowPitch) = v[i];
    }
  } else {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const uint32_t o = base + (uint32_t)i * 4 * kSegBytes;
      if (O::kStore && o < len) {
        if (!O::kExactTail || o + 16 <= len)
          st_stream_v4(dst + o, v[i]);  // image destination: zeros past len are owned padding
        else
          st_partial(dst + o, v[i], len - o);
      }
      if (O::kCrc) *reinterpret_cast<uint4*>(tile_w + i * 4 * kRowPitch) = v[i];
    }
  }
}

// End of a chunk: the owned padding (zeroed in the image, or checked), and the CRC
// word (written to the table, or compared). `f` = the chunk register before the
// zero-padding correction, valid in lane 0.
template <int kOp>
__device__ __forceinline__ void finish_chunk(const LaunchParams& p, uint64_t c, const uint8_t* src, uint8_t* dst,
                                             uint32_t len, uint32_t pad, int nrounds, uint32_t f, int lane) {
  using O = OpT<kOp>;
  uint32_t pad_bad = 0;
  if (pad) {
    if (O::kZeroPad) {
      const uint32_t start = (len + 15u) & ~15u, end = len + pad;
      for (uint32_t o = start + lane * 16u; o < end; o += 512u)
        *reinterpret_cast<uint4*>(dst + o) = make_uint4(0u, 0u, 0u, 0u);
    } else if (O::kCompare) {
      for (uint32_t o = len + lane; o < len + pad; o += 32u) pad_bad |= src[o];
    } else if (O::kCopyPad) {
      for (uint32_t o = len + lane; o < len + pad; o += 32u) dst[o] = src[o];
    }
  }
  if (O::kCompare) pad_bad = __any_sync(0xFFFFFFFFu, pad_bad != 0);
  if (O::kCrc && lane == 0) {
    const uint32_t zp = (uint32_t)nrounds * kRoundBytes - len;
    const uint32_t out = ~(zp ? gf_mul(f, p.inv_z[zp]) : f);
    if (!O::kCompare) {
      p.crc[c] = out;
      if (p.crc_mirror) p.crc_mirror[c] = out;  // posted write into the image's pinned host mirror
    } else if (out != p.crc[c] || pad_bad) {
      atomicMin(&p.status[0], (unsigned long long)c);
      atomicAdd(&p.status[1], 1ull);
    }
  }
}

// End of a publishing verify/check launch (p.status_host set): the last CTA to
// finish copies the status words to the pinned host mirror and resets them to
// {~0, 0, 0}, so the host reads the result without a D2H copy and the next restore
// needs no initialisation launch. (Each CTA's atomics are ordered before its
// arrival by __threadfence; the last arrival then sees every CTA's updates.)
template <int kOp>
__device__ __forceinline__ void publish_status(const LaunchParams& p) {
  if (!OpT<kOp>::kCompare || !p.status_host) return;
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    if (atomicAdd(&p.status[2], 1ull) == gridDim.x - 1) {
      __threadfence();
      const unsigned long long first = atomicExch(&p.status[0], ~0ull);
      const unsigned long long n_bad = atomicExch(&p.status[1], 0ull);
      atomicExch(&p.status[2], 0ull);
      volatile unsigned long long* h = p.status_host;
      h[0] = first;
      h[1] = n_bad;
    }
  }
}

// diagnostics (experiments build only, CHECL_WARP_TRACE): lane 0 of every warp
// records {start, tables ready, end}; the product build compiles both to nothing
#ifdef CHECL_EXPERIMENTS
__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ void warp_trace(const LaunchParams& p, int k, unsigned long long t) {
  if (p.warp_trace && (threadIdx.x & 31) == 0)
    p.warp_trace[((uint64_t)blockIdx.x * kWarpsPerCta + (threadIdx.x >> 5)) * 4 + k] = t;
}
#else
__device__ __forceinline__ unsigned long long gtimer() { return 0; }
__device__ __forceinline__ void warp_trace(const LaunchParams&, int, unsigned long long) {}
#endif

template <int kOp>
__device__ __forceinline__ void chunk_ptrs(const LaunchParams& p, const ChunkDesc& d, const uint8_t*& src,
                                           uint8_t*& dst, int& mode) {
  using O = OpT<kOp>;
  uint8_t* img = p.image + ((uint64_t)d.img_off_256 * kBufferAlign - p.image_base);
  uint8_t* buf = reinterpret_cast<uint8_t*>(d.ptr);
  src = O::kSrcImg ? img : buf;
  dst = O::kSrcImg ? buf : img;
  mode = O::kSrcImg ? 0 : ((d.ptr & 15u) == 0 ? 0 : ((d.ptr & 3u) == 0 ? 1 : 2));
}

template <int kOp>
__global__ void __launch_bounds__(kThreadsPerCta, 1) snapshot_kernel(const LaunchParams p) {
  using O = OpT<kOp>;
  extern __shared__ __align__(128) uint8_t smem[];
  if (O::kCrc) {
    const TableCopy cp[1] = {{0u, (uint32_t)kTabOff, (uint32_t)kSnapTabWords * 4u}};
    // (waited for before the first CRC: the first chunk's loads overlap the copy)
    load_tables<1, false>(smem, p.tables, cp, reinterpret_cast<uint64_t*>(smem + kMbarOff));
  }
  bool tables_ready = false;
  const uint8_t* tb = smem + kTabOff * 4;
  const uint8_t* hb = smem + kHornerOff * 4;
  const uint32_t* ftab = reinterpret_cast<const uint32_t*>(smem + kFoldOff * 4);

  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint8_t* stage = smem + kTileOff + warp * kStageBytes;
  const uint32_t l4 = (uint32_t)lane * 4u;
  const uint64_t nwarps = (uint64_t)gridDim.x * kWarpsPerCta;
  const unsigned full = 0xFFFFFFFFu;
  // instruction i of a round: lane l moves granule l%8 of segment 4i + l/8 (each
  // warp instruction = 512 contiguous bytes = four full 128-byte lines)
  const int g_lane = lane & 7, s_lane = lane >> 3;
  const uint32_t lane_off = (uint32_t)s_lane * kSegBytes + (uint32_t)g_lane * 16;
  uint8_t* tile_w = stage + s_lane * kRowPitch + g_lane * 16;  // this lane's slot, instruction 0

  for (uint64_t c = p.c0 + (uint64_t)blockIdx.x * kWarpsPerCta + warp; c < p.c1; c += nwarps) {
    const ChunkDesc d = p.desc[c];
    const uint32_t len = desc_len(d), pad = desc_pad(d);
    const uint8_t* src;
    uint8_t* dst;
    int mode;
    chunk_ptrs<kOp>(p, d, src, dst, mode);
    const int nrounds = (int)((len + kRoundBytes - 1) / kRoundBytes);
    uint32_t ch = lane == 0 ? 0xFFFFFFFFu : 0u;

    // one round: store + stage it, issue the loads of round r + kPrefetch into the
    // registers just stored, then CRC the staged round while those loads fly
    auto round = [&](uint4 (&v)[8], int r) {
      store_round<kOp>(v, dst, len, r, lane_off, tile_w);
      __syncwarp();
      if (r + kPrefetch < nrounds) load_round(v, src, len, mode, r + kPrefetch, lane_off);
      if (O::kCrc && !tables_ready) {
        wait_tables(reinterpret_cast<uint64_t*>(smem + kMbarOff));
        tables_ready = true;
      }
      if (O::kCrc) {
        // lane l: segment 32r + l; Horner step over the rest of the round first
        if (r > 0) ch = horner_mul(ch, hb, l4);
        const uint4* row = reinterpret_cast<const uint4*>(stage + lane * kRowPitch);
#pragma unroll
        for (int g = 0; g < 8; ++g) ch = crc_step16(ch, row[g], tb, l4);
      }
      __syncwarp();
    };
#if CHECL_PREFETCH == 2
    uint4 va[8], vb[8];
    load_round(va, src, len, mode, 0, lane_off);
    if (nrounds > 1) load_round(vb, src, len, mode, 1, lane_off);
    for (int r = 0; r < nrounds; r += 2) {
      round(va, r);
      if (r + 1 < nrounds) round(vb, r + 1);
    }
#else
    uint4 v[8];
    load_round(v, src, len, mode, 0, lane_off);
    for (int r = 0; r < nrounds; ++r) round(v, r);
#endif

    // Fold the lanes: at level k, lane l (l % 2^(k+1) == 0) shifts its group past
    // the 128*2^k bytes of the group to its right and adds it. The result is the
    // register of the chunk zero-padded to nrounds*4096 bytes (corrected in
    // finish_chunk with one multiply by x^(-8 zp)).
    uint32_t f = ch;
    if (O::kCrc) {
#pragma unroll
      for (int k = 0; k < kFoldLevels; ++k) {
        const uint32_t o = __shfl_down_sync(full, f, 1 << k);
        if ((lane & ((2 << k) - 1)) == 0) f = fold_mul(f, ftab + k * 128) ^ o;
      }
    }
    finish_chunk<kOp>(p, c, src, dst, len, pad, nrounds, f, lane);
  }
  // no warp exits while the table copy into its CTA's shared memory is in flight
  if (O::kCrc && !tables_ready) wait_tables(reinterpret_cast<uint64_t*>(smem + kMbarOff));
  publish_status<kOp>(p);
}

// ---- work of the balanced and TMA kernels --------------------------------------
// The rounds [R0, R0 + R) of the launch's chunks (round_base) are handed out in two
// phases (guided self-scheduling): the first Rs rounds in equal contiguous stretches,
// one per warp, then blocks of B rounds taken from a launch-wide counter by whichever
// warp is free. Measured (CHECL_WARP_TRACE): with static stretches only, warps on the
// 3-warp SM sub-partitions finish ~8 us after those on 2-warp ones, and bulk-copy
// throughput differs by SM position by up to 25%; the dynamic tail absorbs both.
struct Sched {
  uint64_t R0, R, Rs, nblk;
  uint32_t B;
  bool near;  // few short chunks: find_chunk's first probe settles every search
};

__device__ __forceinline__ Sched make_sched(const LaunchParams& p) {
  Sched s;
  s.R0 = p.round_base[p.c0];
  s.R = p.round_base[p.c1] - s.R0;
  s.B = p.dyn_block ? p.dyn_block : 1u;
  s.Rs = p.work ? s.R * p.static_permille / 1000u : s.R;
  s.nblk = (s.R - s.Rs + s.B - 1) / s.B;
  // rounds missing against 16 per chunk; below 16 * 30 the chunk holding any round is
  // within 31 chunks of find_chunk's lower bound
  s.near = (p.c1 - p.c0) * (kChunkBytes / kRoundBytes) - s.R < 16 * 30;
  return s;
}

// The chunk holding round g: the last c in [c0, c1) with round_base[c] <= g. A chunk
// has at most 16 rounds, so round_base[c] <= R0 + 16 (c - c0) and the answer is at
// least lo = c0 + (g - R0) / 16, and at most ~(missing rounds) / 16 chunks above it.
// With few short chunks (s.near: C1, C2, C4) one coalesced probe of the 32 chunks from
// lo settles it (one dependent load instead of three or four); otherwise a 32-way
// search over [c0, c1) (one probe per lane; with 10 000 short chunks the first probe
// would only add a load: C3 measured 8-12 us slower with it).
__device__ __forceinline__ uint64_t find_chunk(const LaunchParams& p, uint64_t g, const Sched& s, int lane) {
  constexpr uint64_t kRoundsPerChunk = kChunkBytes / kRoundBytes;
  uint64_t lo = p.c0, hi = p.c1;  // invariant: round_base[lo] <= g, answer in [lo, hi)
  if (s.near) {
    lo += (g - s.R0) / kRoundsPerChunk;
    const uint64_t idx = lo + (uint64_t)lane;
    const unsigned m = __ballot_sync(0xFFFFFFFFu, idx < hi && p.round_base[idx] <= g);
    if (m != 0xFFFFFFFFu) return lo + (uint64_t)(31 - __clz(m));
    lo += 31;
  }
  while (hi - lo > 1) {
    const uint64_t step = (hi - lo + 31) / 32, idx = lo + lane * step;
    const unsigned m = __ballot_sync(0xFFFFFFFFu, idx < hi && p.round_base[idx] <= g);
    lo += (uint64_t)(31 - __clz(m)) * step;
    hi = hi < lo + step ? hi : lo + step;
  }
  return lo;
}

// Next dynamic block [g, ge) and its first chunk; false when the counter ran out.
__device__ __forceinline__ bool next_block(const LaunchParams& p, const Sched& s, int lane, uint64_t& g, uint64_t& ge,
                                           uint64_t& c) {
  if (!p.work) return false;
  unsigned long long b = 0;
  if (lane == 0) b = atomicAdd(&p.work[0], 1ull);
  b = __shfl_sync(0xFFFFFFFFu, b, 0);
  if (b >= s.nblk) return false;
  g = s.R0 + s.Rs + b * s.B;
  ge = g + s.B < s.R0 + s.R ? g + s.B : s.R0 + s.R;
  c = find_chunk(p, g, s, lane);
  return true;
}

// End of a scheduled launch: the last CTA resets the work counter for the next one.
__device__ __forceinline__ void release_work(const LaunchParams& p) {
  if (!p.work) return;
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    if (atomicAdd(&p.work[1], 1ull) == gridDim.x - 1) {
      atomicExch(&p.work[0], 0ull);
      atomicExch(&p.work[1], 0ull);
    }
  }
}

// ---- balanced kernel: an equal contiguous stretch of rounds per warp ---------
//
// The rounds of the launch's chunks, enumerated in order (round_base), are split
// into one contiguous stretch per warp of the grid, equal to within one round. That
// removes the wave quantisation of the grid-stride chunk loop (7070 C2 chunks over
// 1480 warps leave its last wave 78% full; measured C2 pack 168 -> 163 us; a variant
// taking whole waves first and splitting only the last one measured 168 us). A
// stretch covers whole chunks and at most a partial chunk at each end. A part [r0, r1) of a chunk of n
// rounds is CRC'd exactly like a whole chunk (lane chains with Horner steps, lane
// fold) from a zero register (the CRC init only when r0 = 0), giving F = the
// register of those rounds; the chunk register is XOR_parts F * x^(8*4096*(n - r1)).
// Whole chunks finish directly; split ones XOR their term into the chunk's 64-bit
// accumulator together with their rounds' bits of a completion mask (the sweep
// kernel's scheme): the part that completes the mask holds the chunk register.
// Small launches degenerate to about one round per warp.
constexpr size_t kBalUnitOff = kTileOff;                         // x^(8*4096*k)*x^i table
constexpr size_t kBalTileOff = kBalUnitOff + (size_t)kUnitWords * 4;
constexpr size_t kBalMbarOff = kBalTileOff + (size_t)kWarpsPerCta * kStageBytes;
constexpr size_t kBalSmemBytes = kBalMbarOff + 16;
static_assert(kBalSmemBytes <= 232448, "fits the 227 KiB opt-in shared memory");

template <int kOp>
__global__ void __launch_bounds__(kThreadsPerCta, 1) balanced_kernel(const LaunchParams p) {
  using O = OpT<kOp>;
  extern __shared__ __align__(128) uint8_t smem[];
  const unsigned long long t_start = gtimer();
  if (O::kCrc) {
    const TableCopy cp[2] = {{0u, (uint32_t)kTabOff, (uint32_t)kSnapTabWords * 4u},
                             {(uint32_t)kBalUnitOff, (uint32_t)kUnitOff, (uint32_t)kUnitWords * 4u}};
    load_tables<2, false>(smem, p.tables, cp, reinterpret_cast<uint64_t*>(smem + kBalMbarOff));
  }
  bool tables_ready = !O::kCrc;
  const uint8_t* tb = smem + kTabOff * 4;
  const uint8_t* hb = smem + kHornerOff * 4;
  const uint32_t* ftab = reinterpret_cast<const uint32_t*>(smem + kFoldOff * 4);
  const uint32_t* utab = reinterpret_cast<const uint32_t*>(smem + kBalUnitOff);

  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint8_t* stage = smem + kBalTileOff + warp * kStageBytes;
  const uint32_t l4 = (uint32_t)lane * 4u;
  const unsigned full = 0xFFFFFFFFu;
  const int g_lane = lane & 7, s_lane = lane >> 3;
  const uint32_t lane_off = (uint32_t)s_lane * kSegBytes + (uint32_t)g_lane * 16;
  uint8_t* tile_w = stage + s_lane * kRowPitch + g_lane * 16;

  const uint64_t nw = (uint64_t)gridDim.x * kWarpsPerCta, wid = (uint64_t)blockIdx.x * kWarpsPerCta + warp;
  const Sched sc = make_sched(p);
  uint64_t g = sc.R0 + sc.Rs * wid / nw, g_end = sc.R0 + sc.Rs * (wid + 1) / nw;
  uint64_t lo = g < g_end ? find_chunk(p, g, sc, lane) : p.c0;
  for (bool more = true; more;) {
  // the next dynamic block is fetched (and its chunk found) while the first loads of
  // this stretch are in flight
  uint64_t ng = 0, nge = 0, nlo = 0;
  bool fetched = false, nmore = false;
  auto prefetch = [&]() {
    if (!fetched) {
      fetched = true;
      nmore = next_block(p, sc, lane, ng, nge, nlo);
    }
  };
  for (uint64_t cur = lo; g < g_end; ++cur) {
    const uint64_t rb = p.round_base[cur];
    const ChunkDesc d = p.desc[cur];
    const uint32_t len = desc_len(d), pad = desc_pad(d);
    const uint8_t* src;
    uint8_t* dst;
    int mode;
    chunk_ptrs<kOp>(p, d, src, dst, mode);
    const int nrounds = (int)((len + kRoundBytes - 1) / kRoundBytes);
    const int r0 = (int)(g - rb);
    const int r1 = (int)(g_end - rb < (uint64_t)nrounds ? g_end - rb : (uint64_t)nrounds);
    g = rb + (uint64_t)r1;
    uint32_t ch = (lane == 0 && r0 == 0) ? 0xFFFFFFFFu : 0u;

    // one round: store + stage it, issue the loads of round r + kPrefetch into the
    // registers just stored, then CRC the staged round while those loads fly
    auto round = [&](uint4 (&v)[8], int r) {
      store_round<kOp>(v, dst, len, r, lane_off, tile_w);
      __syncwarp();
      if (r + kPrefetch < r1) load_round(v, src, len, mode, r + kPrefetch, lane_off);
      if (O::kCrc) {
        if (r > r0) ch = horner_mul(ch, hb, l4);
        const uint4* row = reinterpret_cast<const uint4*>(stage + lane * kRowPitch);
#pragma unroll
        for (int q = 0; q < 8; ++q) ch = crc_step16(ch, row[q], tb, l4);
      }
      __syncwarp();
    };
#if CHECL_PREFETCH == 2
    uint4 va[8], vb[8];
    load_round(va, src, len, mode, r0, lane_off);
    if (r0 + 1 < r1) load_round(vb, src, len, mode, r0 + 1, lane_off);
    if (!tables_ready) {
      wait_tables(reinterpret_cast<uint64_t*>(smem + kBalMbarOff));
      tables_ready = true;
    }
    for (int r = r0; r < r1; r += 2) {
      round(va, r);
      if (r + 1 < r1) round(vb, r + 1);
    }
#else
    uint4 v[8];
    load_round(v, src, len, mode, r0, lane_off);
    if (!tables_ready) {  // the first loads are in flight; the tables have landed by now
      wait_tables(reinterpret_cast<uint64_t*>(smem + kBalMbarOff));
      tables_ready = true;
      warp_trace(p, 1, gtimer());
    }
    prefetch();
    for (int r = r0; r < r1; ++r) round(v, r);
#endif
    uint32_t f = ch;
    if (O::kCrc) {
#pragma unroll
      for (int k = 0; k < kFoldLevels; ++k) {
        const uint32_t o = __shfl_down_sync(full, f, 1 << k);
        if ((lane & ((2 << k) - 1)) == 0) f = fold_mul(f, ftab + k * 128) ^ o;
      }
    }
    if (!O::kCrc || (r0 == 0 && r1 == nrounds)) {
      if (O::kCrc || r1 == nrounds) finish_chunk<kOp>(p, cur, src, dst, len, pad, nrounds, f, lane);
      continue;
    }
    // split chunk: this part's term, shifted past the rounds after it
    f = __shfl_sync(full, f, 0);
    const int k = nrounds - r1;
    const uint32_t term = warp_xor(((f >> (31 - lane)) & 1u) ? utab[k * 32 + lane] : 0u);
    const unsigned long long mine =
        (unsigned long long)term | ((((1ull << (r1 - r0)) - 1ull) << r0) << 32);
    unsigned long long old = 0;
    if (lane == 0) old = atomicXor(&p.unit_acc[cur - p.c0], mine);
    const unsigned long long now = __shfl_sync(full, old, 0) ^ mine;
    if ((now >> 32) == (1ull << nrounds) - 1) {
      if (lane == 0) p.unit_acc[cur - p.c0] = 0ull;  // zero again for the next launch
      finish_chunk<kOp>(p, cur, src, dst, len, pad, nrounds, (uint32_t)now, lane);
    }
  }
  prefetch();
  more = nmore;
  g = ng;
  g_end = nge;
  lo = nlo;
  }
  // a warp without rounds still waits: the CTA must not exit under the table copy
  if (!tables_ready) wait_tables(reinterpret_cast<uint64_t*>(smem + kBalMbarOff));
  release_work(p);
  warp_trace(p, 0, t_start);
  warp_trace(p, 2, gtimer());
  {
    unsigned smid;
    asm("mov.u32 %0, %%smid;" : "=r"(smid));
    warp_trace(p, 3, smid);
  }
  publish_status<kOp>(p);
}

// ---- TMA kernel: bulk copies through a contiguous tile, column CRC -----------
//
// Same work split as balanced_kernel (equal stretches of 4 KiB rounds per warp,
// split chunks combined through the atomic accumulator), different data path: a
// full round of a 16-byte-aligned source is moved global -> shared by one bulk
// copy (cp.async.bulk, mbarrier completion) and shared -> global by one bulk store,
// two tiles per warp (the next round's copy is in flight during this round's CRC);
// the LSU carries only the CRC's shared loads. Partial, misaligned or remote rounds
// take the register path (16-byte loads, stores from registers, exact tails) and
// are written into the same tile. The tile is contiguous, so the CRC reads it by
// columns: lane l reads word l of every 128-byte row (conflict-free LDS.32) and
// chains it, a column of stride 128 B that runs across rounds unchanged:
//   h <- (h ^ w) * x^(8*128)
// With D = the part's bytes zero-padded to whole rounds, n = |D|, word i = l + 32k,
//   R(D, s) = XOR_i R(w_i, 0) x^(8(n - 4i - 4)) = XOR_l h_l x^(-32 l),
// (s folded into lane 0's first word), the lanes combined by a shuffle tree with
// shifts x^(-32*2^k). The column is split into kColChains independent chains (rows
// = c mod kColChains, step x^(8*128*kColChains), slicing-by-4 over tables of that
// shift) so that a lane has kColChains lookups in flight instead of one:
//   h_l = XOR_c ch_c x^(-1024 c). The rest (zero-padding correction, split-chunk terms) is the
// balanced kernel's.
constexpr int kTmaTiles = 2;
constexpr size_t kTmaColOff = 0;
constexpr size_t kTmaFoldOff = (size_t)kColWords * 4;
constexpr size_t kTmaUnitOff = kTmaFoldOff + (size_t)kColFoldWords * 4;
constexpr size_t kTmaTileOff = (kTmaUnitOff + (size_t)kUnitWords * 4 + 127) / 128 * 128;
constexpr size_t kTmaMbarOff = kTmaTileOff + (size_t)kWarpsPerCta * kTmaTiles * kRoundBytes;
constexpr size_t kTmaSmemBytes = kTmaMbarOff + (size_t)(kWarpsPerCta * kTmaTiles + 1) * 8;
static_assert(kTmaSmemBytes <= 232448, "fits the 227 KiB opt-in shared memory");
static_assert(kColFoldOff == kColOff + kColWords, "column tables and their fold tables are contiguous");

__device__ __forceinline__ void mbar_init(uint32_t mb) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(mb) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t mb, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n TW_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      " @!p bra TW_%=;\n}" ::"r"(mb),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void bulk_load(uint32_t dst, const void* src, uint32_t bytes, uint32_t mb) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"(bytes) : "memory");
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
               "l"(src), "r"(bytes), "r"(mb)
               : "memory");
}
__device__ __forceinline__ void bulk_store(void* dst, uint32_t src, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(src), "r"(bytes)
               : "memory");
  asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
__device__ __forceinline__ void bulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

__device__ __forceinline__ void cluster_sync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

// Table prologue of a 2-CTA cluster (kernel 4, CHECL_TABLE_MC): the table image is
// cut into 32 KiB pieces and each CTA issues every other piece as one bulk copy
// multicast to both CTAs (same shared offset in each), so L2 serves each table byte
// once per SM pair instead of once per SM. Each CTA's table mbarrier expects all the
// bytes; the cluster barrier orders both CTAs' barrier initialisations before any
// multicast can complete on them (and synchronises the CTA like load_tables).
template <int N>
__device__ __forceinline__ void load_tables_mc(uint8_t* smem, const uint32_t* gtab, const TableCopy (&cp)[N],
                                               uint64_t* mbar) {
  const uint32_t mb = smem_addr(mbar);
  uint32_t rank;
  asm("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(mb) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  cluster_sync();
  if (threadIdx.x == 0) {
    uint32_t total = 0;
#pragma unroll
    for (int i = 0; i < N; ++i) total += cp[i].bytes;
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"(total) : "memory");
    const uint16_t both = 0x3;
    uint32_t k = 0;
#pragma unroll
    for (int i = 0; i < N; ++i) {
      for (uint32_t o = 0; o < cp[i].bytes; o += 32768u, ++k) {
        if ((k & 1u) != rank) continue;
        const uint32_t n = cp[i].bytes - o < 32768u ? cp[i].bytes - o : 32768u;
        asm volatile(
            "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.multicast::cluster [%0], [%1], %2, [%3], "
            "%4;" ::"r"(smem_addr(smem + cp[i].dst_off + o)),
            "l"(reinterpret_cast<const uint8_t*>(gtab + cp[i].src_word) + o), "r"(n), "r"(mb), "h"(both)
            : "memory");
      }
    }
  }
}

// kMc: launched as 2-CTA clusters; the table prologue is multicast (load_tables_mc)
template <int kOp, bool kMc>
__global__ void __launch_bounds__(kThreadsPerCta, 1) tma_kernel(const LaunchParams p) {
  using O = OpT<kOp>;
  extern __shared__ __align__(128) uint8_t smem[];
  const unsigned long long t_start = gtimer();
  uint64_t* mbars = reinterpret_cast<uint64_t*>(smem + kTmaMbarOff);  // [warp][tile], then the tables'
  if (threadIdx.x == 0)
    for (int i = 0; i < kWarpsPerCta * kTmaTiles; ++i) mbar_init(smem_addr(mbars + i));
  {  // (load_tables fences the barrier initialisations and synchronises the CTA)
    const TableCopy cp[2] = {{(uint32_t)kTmaColOff, (uint32_t)kColOff, (uint32_t)(kColWords + kColFoldWords) * 4u},
                             {(uint32_t)kTmaUnitOff, (uint32_t)kUnitOff, (uint32_t)kUnitWords * 4u}};
    if constexpr (kMc)
      load_tables_mc<2>(smem, p.tables, cp, mbars + kWarpsPerCta * kTmaTiles);
    else
      load_tables<2, false>(smem, p.tables, cp, mbars + kWarpsPerCta * kTmaTiles);
  }
  bool tables_ready = false;
  const uint8_t* tb = smem + kTmaColOff;
  const uint32_t* ftab = reinterpret_cast<const uint32_t*>(smem + kTmaFoldOff);
  const uint32_t* utab = reinterpret_cast<const uint32_t*>(smem + kTmaUnitOff);

  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint8_t* tiles = smem + kTmaTileOff + (size_t)warp * kTmaTiles * kRoundBytes;
  const uint32_t tile_sa = smem_addr(tiles), mb_sa = smem_addr(mbars + warp * kTmaTiles);
  uint32_t phase = 0;  // bit t: parity of tile t's next completion
  const uint32_t l4 = (uint32_t)lane * 4u;
  const unsigned full = 0xFFFFFFFFu;
  // register path: instruction i of a round = 512 contiguous bytes; lane l moves
  // the 16 bytes at lane_off + 512 i (the same offset in the contiguous tile)
  const uint32_t lane_off = (uint32_t)(lane >> 3) * kSegBytes + (uint32_t)(lane & 7) * 16;

  // A part = the rounds [r0, r1) of one chunk inside a stretch. The first round of
  // the next part (next chunk of the stretch, or first chunk of the next stretch) is
  // issued during this part's last round, so a warp's copy pipeline never drains at
  // chunk or stretch boundaries.
  struct Part {
    uint64_t c, rb;  // chunk, its round_base
    const uint8_t* src;
    uint8_t* dst;
    uint32_t len, pad;
    int mode, nrounds, r0, r1;
    bool bulk_ok;
  };
  auto open_part = [&](uint64_t c, uint64_t rb, const ChunkDesc d, uint64_t g, uint64_t ge) {
    Part q;
    q.c = c;
    q.rb = rb;
    q.len = desc_len(d);
    q.pad = desc_pad(d);
    chunk_ptrs<kOp>(p, d, q.src, q.dst, q.mode);
    q.nrounds = (int)((q.len + kRoundBytes - 1) / kRoundBytes);
    q.r0 = (int)(g - rb);
    q.r1 = (int)(ge - rb < (uint64_t)q.nrounds ? ge - rb : (uint64_t)q.nrounds);
    q.bulk_ok = q.mode == 0 && ((reinterpret_cast<uintptr_t>(q.src) & 15u) == 0) &&
                (!O::kStore || (reinterpret_cast<uintptr_t>(q.dst) & 15u) == 0) && !(O::kSrcImg && p.image_remote && !(p.image_remote == 1 && p.remote_bulk));
    return q;
  };
  auto is_bulk = [&](const Part& q, int r) { return q.bulk_ok && (uint32_t)(r + 1) * kRoundBytes <= q.len; };
  uint4 v[8];  // the register path's round in flight
  auto issue = [&](const Part& q, int r, int tt) {
    if (is_bulk(q, r)) {
      if (lane == 0) bulk_load(tile_sa + tt * kRoundBytes, q.src + (size_t)r * kRoundBytes, kRoundBytes, mb_sa + tt * 8);
    } else {
      load_round(v, q.src, q.len, q.mode, r, lane_off);
    }
  };

  const uint64_t nw = (uint64_t)gridDim.x * kWarpsPerCta, wid = (uint64_t)blockIdx.x * kWarpsPerCta + warp;
  const Sched sc = make_sched(p);
  uint64_t g = sc.R0 + sc.Rs * wid / nw, g_end = sc.R0 + sc.Rs * (wid + 1) / nw, c = 0;
  bool have = g < g_end, fetched = false, nmore = false;
  if (have) {
    c = find_chunk(p, g, sc, lane);
  } else {  // no static rounds: straight to the dynamic blocks (the block taken here is
            // the current stretch; its successor is fetched during its first round)
    have = next_block(p, sc, lane, g, g_end, c);
  }
  uint64_t ng = 0, nge = 0, nlo = 0;  // the next stretch (dynamic block), once fetched
  int t = 0;                          // tile of the round being consumed
#ifdef CHECL_TRACE_LOOPEND  // experiment: slot 2 = the warp's last round done, slot 3 = smid | rounds << 32
  unsigned long long n_done = 0;
#endif
  Part cur{};
  if (have) {
    cur = open_part(c, p.round_base[c], p.desc[c], g, g_end);
    issue(cur, cur.r0, t);
  }
#ifdef CHECL_TRACE_SETUP  // experiment: slot 1 = first round issued (schedule set up)
  warp_trace(p, 1, gtimer());
#endif
  // (the tables are waited for just before the first CRC: by then the first two rounds
  // are in flight)
  while (have) {
    // successor inside this stretch: its descriptor loads fly during this part's rounds
    const uint64_t cur_end = cur.rb + (uint64_t)cur.r1;
    const bool same = cur_end < g_end;
    bool succ = same, s_known = same || fetched;
    uint64_t s_c = cur.c + 1, s_g = cur_end, s_ge = g_end;
    ChunkDesc sd{};
    uint64_t srb = 0;
    if (!same && fetched && nmore) {
      succ = true;
      s_c = nlo, s_g = ng, s_ge = nge;
    }
    if (succ) {
      sd = p.desc[s_c];
      srb = p.round_base[s_c];
    }
    Part nxt = cur;
    uint32_t ch[kColChains];  // chain c: rows = c mod kColChains (the CRC init enters row 0)
    ch[0] = (lane == 0 && cur.r0 == 0) ? 0xFFFFFFFFu : 0u;
#pragma unroll
    for (int c = 1; c < kColChains; ++c) ch[c] = 0u;
    for (int r = cur.r0; r < cur.r1; ++r) {
      uint8_t* tile = tiles + t * kRoundBytes;
      // the bulk stores of earlier rounds have finished reading their tiles
      if (lane == 0) bulk_wait_read();
      __syncwarp();
      const bool bulk = is_bulk(cur, r);
      if (!bulk) {  // register round: into the tile, and to the destination from registers
#pragma unroll
        for (int i = 0; i < 8; ++i) *reinterpret_cast<uint4*>(tile + lane_off + i * 512) = v[i];
        if (O::kStore) {
          const uint32_t base = (uint32_t)r * kRoundBytes + lane_off;
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            const uint32_t o = base + (uint32_t)i * 512;
            if (o < cur.len) {
              if (!O::kExactTail || o + 16 <= cur.len)
                st_stream_v4(cur.dst + o, v[i]);  // image destination: zeros past len are owned padding
              else
                st_partial(cur.dst + o, v[i], cur.len - o);
            }
          }
        }
        __syncwarp();
      }
      if (r + 1 < cur.r1) issue(cur, r + 1, t ^ 1);
      // the next dynamic block, fetched (and its chunk found) once per stretch while
      // this stretch's first rounds are in flight
      if (!fetched) {
        fetched = true;
        nmore = next_block(p, sc, lane, ng, nge, nlo);
      }
      if (!s_known) {  // the successor is the next block's first part
        s_known = true;
        if (nmore) {
          succ = true;
          s_c = nlo, s_g = ng, s_ge = nge;
          sd = p.desc[s_c];
          srb = p.round_base[s_c];
        }
      }
      if (r + 1 == cur.r1 && succ) {
        nxt = open_part(s_c, srb, sd, s_g, s_ge);
        issue(nxt, nxt.r0, t ^ 1);
      }
      if (!tables_ready) {
        wait_tables(mbars + kWarpsPerCta * kTmaTiles);
        tables_ready = true;
#ifndef CHECL_TRACE_SETUP
        warp_trace(p, 1, gtimer());
#endif
      }
      if (bulk) {
        mbar_wait(mb_sa + t * 8, (phase >> t) & 1u);
        phase ^= 1u << t;
        if (O::kStore && lane == 0)
          bulk_store(cur.dst + (size_t)r * kRoundBytes, tile_sa + t * kRoundBytes, kRoundBytes);
      }
      if (O::kCrc) {
#pragma unroll
        for (int q = 0; q < 32; ++q)
          ch[q % kColChains] =
              crc_step4(ch[q % kColChains], *reinterpret_cast<const uint32_t*>(tile + q * kSegBytes + l4), tb, l4);
      }
      fence_proxy_async();  // this round's shared reads before the next bulk copy into the tile
      __syncwarp();
      t ^= 1;
#ifdef CHECL_TRACE_LOOPEND
      ++n_done;
#endif
    }
    // chain c stepped every row it holds by x^(1024*kColChains), i.e. c rows too far:
    // h = XOR_c ch[c] * x^(-1024 c) (Horner), then the lanes as before
    uint32_t f = ch[kColChains - 1];
    if (O::kCrc) {
#pragma unroll
      for (int c = kColChains - 2; c >= 0; --c) f = fold_mul(f, ftab + kFoldLevels * 128) ^ ch[c];
#pragma unroll
      for (int k = 0; k < kFoldLevels; ++k) {
        const uint32_t o = __shfl_down_sync(full, f, 1 << k);
        if ((lane & ((2 << k) - 1)) == 0) f ^= fold_mul(o, ftab + k * 128);
      }
    }
    if (!O::kCrc || (cur.r0 == 0 && cur.r1 == cur.nrounds)) {
      if (O::kCrc || cur.r1 == cur.nrounds)
        finish_chunk<kOp>(p, cur.c, cur.src, cur.dst, cur.len, cur.pad, cur.nrounds, f, lane);
    } else {
      f = __shfl_sync(full, f, 0);
      const int k = cur.nrounds - cur.r1;
      const uint32_t term = warp_xor(((f >> (31 - lane)) & 1u) ? utab[k * 32 + lane] : 0u);
      const unsigned long long mine =
          (unsigned long long)term | ((((1ull << (cur.r1 - cur.r0)) - 1ull) << cur.r0) << 32);
      unsigned long long old = 0;
      if (lane == 0) old = atomicXor(&p.unit_acc[cur.c - p.c0], mine);
      const unsigned long long now = __shfl_sync(full, old, 0) ^ mine;
      if ((now >> 32) == (1ull << cur.nrounds) - 1) {
        if (lane == 0) p.unit_acc[cur.c - p.c0] = 0ull;
        finish_chunk<kOp>(p, cur.c, cur.src, cur.dst, cur.len, cur.pad, cur.nrounds, (uint32_t)now, lane);
      }
    }
    if (!succ) break;
    if (!same) {  // into the next stretch: its successor is fetched at the top
      g_end = nge;
      fetched = false;
      nmore = false;
    }
    cur = nxt;
  }
#ifdef CHECL_TRACE_LOOPEND
  warp_trace(p, 2, gtimer());
#endif
  if (!tables_ready) wait_tables(mbars + kWarpsPerCta * kTmaTiles);
  if (lane == 0) bulk_wait_all();  // the bulk stores have landed before the kernel ends
  release_work(p);
  if constexpr (kMc) cluster_sync();  // neither CTA exits while a multicast it issued is in flight
  warp_trace(p, 0, t_start);
#ifndef CHECL_TRACE_LOOPEND
  warp_trace(p, 2, gtimer());
#endif
  {
    unsigned smid;
    asm("mov.u32 %0, %%smid;" : "=r"(smid));
#ifdef CHECL_TRACE_LOOPEND
    warp_trace(p, 3, smid | (n_done << 32));
#else
    warp_trace(p, 3, smid);
#endif
  }
  publish_status<kOp>(p);
}

// ---- sweep kernel: one 4 KiB unit per warp-iteration ------------------------
//
// Same data path and CRC tables as snapshot_kernel, different work split: the
// work units are the 4 KiB rounds of all chunks (unit u = round u%16 of chunk
// u/16), taken grid-stride, so that at any time the warps of the whole GPU touch
// neighbouring 4 KiB blocks of the payload (the access pattern a plain copy needs
// to run near the HBM roofline) and a chunk's latency is one unit, not 16.
// Lane l CRCs segment l of its unit (zero init; lane 0 of round 0 takes the CRC
// init), then the unit register is  XOR_l  reg_l * x^(8*128*(31-l))  — one
// lane-private nibble-table multiply per lane and a shuffle-XOR reduction. The
// unit's term reg * x^(8*4096*(n-1-r)) is XORed into a per-chunk 64-bit word
// whose high half is a mask of finished units; the unit that completes the mask
// holds the chunk register: CRC = ~( XOR_u term_u * x^(-8 zp) ), zp = 4096 n - len.
// The next unit's loads are issued before the current unit's CRC.

// s * x^(8*128*(31-l)) mod P via 8 lane-private nibble lookups (lane l's constant).
__device__ __forceinline__ uint32_t lanepos_mul(uint32_t s, const uint8_t* pb, uint32_t l4) {
  uint32_t r = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) r ^= tab_ld(pb + j * 2048, (((s >> (4 * j)) & 15u) << 7) | l4);
  return r;
}


template <int kOp>
__global__ void __launch_bounds__(kThreadsPerCta, 1) sweep_kernel(const LaunchParams p) {
  using O = OpT<kOp>;
  extern __shared__ __align__(128) uint8_t smem[];
  // shared layout: tab | pos | unit | (unused) | tiles | mbarrier
  constexpr uint32_t kPosSm = (uint32_t)kTabWords * 4u;
  constexpr uint32_t kUnitSm = kPosSm + (uint32_t)kPosWords * 4u;
  static_assert(kUnitSm + kUnitWords * 4u <= kTileOff, "sweep tables fit before the tiles");
  if (O::kCrc) {
    const TableCopy cp[2] = {{0u, (uint32_t)kTabOff, (uint32_t)kTabWords * 4u},
                             {kPosSm, (uint32_t)kPosOff, (uint32_t)(kPosWords + kUnitWords) * 4u}};
    // (waited for after the first unit's loads are issued: the two overlap)
    load_tables<2, false>(smem, p.tables, cp, reinterpret_cast<uint64_t*>(smem + kMbarOff));
  }
  const uint8_t* tb = smem;
  const uint8_t* pb = smem + kPosSm;
  const uint32_t* utab = reinterpret_cast<const uint32_t*>(smem + kUnitSm);

  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint8_t* stage = smem + kTileOff + warp * kStageBytes;
  const uint32_t l4 = (uint32_t)lane * 4u;
  const int g_lane = lane & 7, s_lane = lane >> 3;
  const uint32_t lane_off = (uint32_t)s_lane * kSegBytes + (uint32_t)g_lane * 16;
  uint8_t* tile_w = stage + s_lane * kRowPitch + g_lane * 16;
  const uint64_t nunits = (p.c1 - p.c0) * 16;
  const uint64_t nw = (uint64_t)gridDim.x * kWarpsPerCta;

  struct Unit {
    uint64_t c;
    int r, nrounds, mode;
    uint32_t len, pad;
    const uint8_t* src;
    uint8_t* dst;
    bool on;
  };
  auto get_unit = [&](uint64_t u) {
    Unit x;
    x.on = false;
    if (u >= nunits) return x;
    x.c = p.c0 + (u >> 4);
    x.r = (int)(u & 15);
    const ChunkDesc d = p.desc[x.c];
    x.len = desc_len(d);
    x.pad = desc_pad(d);
    x.nrounds = (int)((x.len + kRoundBytes - 1) / kRoundBytes);
    if (x.r >= x.nrounds) return x;
    chunk_ptrs<kOp>(p, d, x.src, x.dst, x.mode);
    x.on = true;
    return x;
  };
  uint4 v[8];

  uint64_t u = (uint64_t)blockIdx.x * kWarpsPerCta + warp;
  Unit cur = get_unit(u);
  if (cur.on) load_round(v, cur.src, cur.len, cur.mode, cur.r, lane_off);
  if (O::kCrc) wait_tables(reinterpret_cast<uint64_t*>(smem + kMbarOff));
  for (; u < nunits; u += nw) {
    const Unit nxt = get_unit(u + nw);
    if (cur.on) store_round<kOp>(v, cur.dst, cur.len, cur.r, lane_off, tile_w);
    __syncwarp();
    if (nxt.on) load_round(v, nxt.src, nxt.len, nxt.mode, nxt.r, lane_off);  // in flight during this unit's CRC
    if (cur.on) {
      if (!O::kCrc) {
        if (cur.r == cur.nrounds - 1) finish_chunk<kOp>(p, cur.c, cur.src, cur.dst, cur.len, cur.pad, cur.nrounds, 0u, lane);
      } else {
        uint32_t crc = (lane == 0 && cur.r == 0) ? 0xFFFFFFFFu : 0u;
        const uint4* row = reinterpret_cast<const uint4*>(stage + lane * kRowPitch);
#pragma unroll
        for (int g = 0; g < 8; ++g) crc = crc_step16(crc, row[g], tb, l4);
        const uint32_t reg = warp_xor(lanepos_mul(crc, pb, l4));
        // the unit's term in the chunk register: reg * x^(8*4096*(n-1-r)), lane i
        // adding the x^i coefficient of reg times utab[k][i] = x^(8*4096*k) * x^i
        const int k = cur.nrounds - 1 - cur.r;
        const uint32_t term = warp_xor(((reg >> (31 - lane)) & 1u) ? utab[k * 32 + lane] : 0u);
        // one 64-bit atomicXor carries the term (low half) and this unit's bit in the
        // finished-unit mask (high half): the unit that completes the mask holds the
        // chunk register — no fence, no second pass
        const unsigned long long mine = (unsigned long long)term | (1ull << (32 + cur.r));
        unsigned long long old = 0;
        if (lane == 0) old = atomicXor(&p.unit_acc[cur.c - p.c0], mine);
        const unsigned long long now = __shfl_sync(0xFFFFFFFFu, old, 0) ^ mine;
        if ((now >> 32) == (1ull << cur.nrounds) - 1) {
          // every unit of the chunk has arrived: reset its word for the next launch
          // (the accumulators are all zero between launches; no memset)
          if (lane == 0) p.unit_acc[cur.c - p.c0] = 0ull;
          finish_chunk<kOp>(p, cur.c, cur.src, cur.dst, cur.len, cur.pad, cur.nrounds, (uint32_t)now, lane);
        }
      }
    }
    __syncwarp();
    cur = nxt;
  }
  publish_status<kOp>(p);
}

// ---- lookup tables: built once per device (DevState::init) -------------------
// T_k[e] = CRC register of byte e followed by k zero bytes (zero init); H[j][v] =
// (v << 4j) * x^(8*3968); fold[lvl][j][v] = (v << 4j) * x^(8*128*2^lvl); the sweep
// kernel's position tables (v << 4j) * x^(8*128*(31-l)) and unit powers
// x^(8*4096*k) * x^i. Lane-private copies: entry e of lane l at word e*32 + l.
__global__ void build_tables_kernel(const TableParams tp, uint32_t* __restrict__ out) {
  __shared__ uint32_t scratch[1024 + 128];
  for (int e = threadIdx.x; e < 256; e += blockDim.x) {
    uint32_t r = (uint32_t)e;
    for (int b = 0; b < 8; ++b) r = gf_mulx(r);
    scratch[e] = r;
  }
  for (int i = threadIdx.x; i < 128; i += blockDim.x) scratch[1024 + i] = gf_mul((uint32_t)(i & 15) << (4 * (i >> 4)), tp.horner);
  __syncthreads();
  for (int e = threadIdx.x; e < 256; e += blockDim.x) {
    uint32_t r = scratch[e];
    for (int k = 1; k < 4; ++k) {
      r = (r >> 8) ^ scratch[r & 0xFFu];
      scratch[k * 256 + e] = r;
    }
  }
  __syncthreads();
  // slicing-by-4 super-tables: row-half h = (super-table, row e, half); A = [T3|T2], B = [T1|T0]
  for (int i = threadIdx.x; i < 1024 * 32; i += blockDim.x) {
    const int h = i >> 5, st = h >> 9, e = (h >> 1) & 255, half = h & 1;
    const int k = 3 - (2 * st + half);
    out[kTabOff + i] = scratch[k * 256 + e];
  }
  for (int i = threadIdx.x; i < 128 * 32; i += blockDim.x) out[kHornerOff + i] = scratch[1024 + (i >> 5)];
  for (int i = threadIdx.x; i < kFoldWords; i += blockDim.x) {
    const int lvl = i >> 7, j = (i >> 4) & 7, v = i & 15;
    out[kFoldOff + i] = gf_mul((uint32_t)v << (4 * j), tp.fold[lvl]);
  }
  // position tables: entry (j, v) of lane l = (v << 4j) * C_l, from the four
  // single-bit products C_l * x^(31-4j-t) (bit 4j+t of a reflected value is x^(31-4j-t))
  for (int t = threadIdx.x; t < 8 * 32; t += blockDim.x) {
    const int j = t >> 5, l = t & 31;
    uint32_t b = tp.lanepow[l];
    for (int m = 0; m < 31 - 4 * j - 3; ++m) b = gf_mulx(b);  // b = C * x^(28-4j)
    uint32_t bit[4];
    bit[3] = b;  // v bit 3 sits at position 4j+3 -> x^(28-4j)
    for (int q = 2; q >= 0; --q) bit[q] = gf_mulx(bit[q + 1]);
    for (int v = 0; v < 16; ++v) {
      uint32_t e = 0;
      for (int q = 0; q < 4; ++q)
        if (v & (1 << q)) e ^= bit[q];
      out[kPosOff + (j * 16 + v) * 32 + l] = e;
    }
  }
  for (int t = threadIdx.x; t < kUnitWords; t += blockDim.x) {
    uint32_t b = tp.unitpow[t >> 5];
    for (int m = 0; m < (t & 31); ++m) b = gf_mulx(b);
    out[kUnitOff + t] = b;
  }
  // column tables (TMA kernel): C_j[e] = (e << 8j) * x^(8*128*kColChains), byte j of
  // the register, in the super-table layout (A = [C_0 | C_1], B = [C_2 | C_3]); fold
  // tables of the shifts x^(-32*2^k), k <= kFoldLevels (the last one combines chains)
  __syncthreads();
  for (int e = threadIdx.x; e < 1024; e += blockDim.x) scratch[e] = gf_mul((uint32_t)(e & 255) << (8 * (e >> 8)), tp.col_shift);
  __syncthreads();
  for (int i = threadIdx.x; i < 1024 * 32; i += blockDim.x) {
    const int h = i >> 5, st = h >> 9, e = (h >> 1) & 255, half = h & 1;
    out[kColOff + i] = scratch[(2 * st + half) * 256 + e];
  }
  for (int i = threadIdx.x; i < kColFoldWords; i += blockDim.x) {
    const int lvl = i >> 7, j = (i >> 4) & 7, v = i & 15;
    out[kColFoldOff + i] = gf_mul((uint32_t)v << (4 * j), tp.col_fold[lvl]);
  }
}

// ---- K6 test tooling -------------------------------------------------------

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

__global__ void fill_kernel(uint8_t* p, uint64_t bytes, uint64_t key, int kind) {
  const uint64_t nwords = (bytes + 7) / 8;
  const bool al8 = (reinterpret_cast<uintptr_t>(p) & 7u) == 0;
  for (uint64_t w = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; w < nwords;
       w += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t word = mix64(key + (w + 1) * 0x9E3779B97F4A7C15ull);
    if (kind == 1) {
      const float lo = __uint2float_rn((uint32_t)word >> 8) * 5.9604644775390625e-08f;
      const float hi = __uint2float_rn((uint32_t)(word >> 32) >> 8) * 5.9604644775390625e-08f;
      word = (uint64_t)__float_as_uint(lo) | ((uint64_t)__float_as_uint(hi) << 32);
    } else if (kind == 2) {
      word = 0;
    }
    const uint64_t o = w * 8;
    if (al8 && o + 8 <= bytes) {
      *reinterpret_cast<uint64_t*>(p + o) = word;
    } else {
      for (uint64_t b = 0; b < 8 && o + b < bytes; ++b) p[o + b] = (uint8_t)(word >> (8 * b));
    }
  }
}

__global__ void compare_kernel(const uint8_t* a, const uint8_t* b, uint64_t bytes, unsigned long long* n_diff) {
  unsigned long long local = 0;
  const bool al = ((reinterpret_cast<uintptr_t>(a) | reinterpret_cast<uintptr_t>(b)) & 15u) == 0;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t tid = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  uint64_t done = 0;
  if (al) {
    const uint64_t nv = bytes / 16;
    for (uint64_t i = tid; i < nv; i += stride) {
      const uint4 x = reinterpret_cast<const uint4*>(a)[i], y = reinterpret_cast<const uint4*>(b)[i];
      const uint32_t d[4] = {x.x ^ y.x, x.y ^ y.y, x.z ^ y.z, x.w ^ y.w};
#pragma unroll
      for (int j = 0; j < 4; ++j)
        for (int k = 0; k < 4; ++k) local += ((d[j] >> (8 * k)) & 0xFFu) != 0;
    }
    done = nv * 16;
  }
  for (uint64_t i = done + tid; i < bytes; i += stride) local += a[i] != b[i];
  if (local) atomicAdd(n_diff, local);
}

// ---- plan expansion: buffer records -> flat chunk list (a2 / r2) -------------
// One thread per chunk: find the buffer (largest record index whose first_chunk
// <= c: zero-size records share first_chunk with the next record, so the search
// lands on the non-empty one), then emit {ptr + k*64K, off + k*64K, len, pad}.
// The pad of a buffer's last chunk runs to the next record's offset (or to
// payload_bytes): FORMAT.md "Chunk ownership of padding".
__global__ void expand_plan_kernel(const BufferRecord* __restrict__ recs, uint32_t n, uint64_t payload_bytes,
                                   uint64_t n_chunks, ChunkDesc* __restrict__ out, uint32_t* __restrict__ round_base,
                                   uint64_t total_rounds, unsigned long long* __restrict__ status) {
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    if (round_base) round_base[n_chunks] = (uint32_t)total_rounds;
    if (status) status[0] = ~0ull, status[1] = 0ull, status[2] = 0ull;  // the verify status of the launches that follow
  }
  for (uint64_t c = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; c < n_chunks;
       c += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t lo = 0, hi = n - 1;
    while (lo < hi) {
      const uint32_t mid = (lo + hi + 1) >> 1;
      if (recs[mid].first_chunk <= c) lo = mid; else hi = mid - 1;
    }
    const BufferRecord r = recs[lo];
    const uint64_t k = c - r.first_chunk, base = k * kChunkBytes;
    const uint64_t nch = (r.size + kChunkBytes - 1) / kChunkBytes;
    const uint32_t len = (uint32_t)(r.size - base < kChunkBytes ? r.size - base : kChunkBytes);
    uint32_t pad = 0;
    if (k + 1 == nch) pad = (uint32_t)((lo + 1 < n ? recs[lo + 1].off : payload_bytes) - (r.off + r.size));
    ChunkDesc d;
    d.ptr = r.ptr + base;
    d.img_off_256 = (uint32_t)((r.off + base) / kBufferAlign);
    d.len_pad = make_len_pad(len, pad);
    out[c] = d;
    if (round_base) round_base[c] = (uint32_t)(r.first_round + k * (kChunkBytes / kRoundBytes));
  }
}

// ---- incremental checkpoint: present set, compaction, stages (f1) -----------
// FORMAT.md "Incremental images": chunk k is present iff crc_now[k] != crc_base[k];
// the compacted payload is the concatenation of the present chunks' spans (chunk
// bytes + owned padding) in ascending k. One CTA walks the chunk list in tiles of
// 1024 (C4: 1 M chunks = 1024 tiles, tens of us next to a 17 ms CRC pass): a
// ballot writes 32 bitmap bits per warp, a block scan of (span, present) gives
// each present chunk its compacted offset and index, and the chunk's descriptor is
// re-emitted with the compacted offset (same ptr / len / pad).
// Exact dirty test (FORMAT.md dirty rule 1, reading 25). `shadow` holds the
// base state's payload in payload layout (chunk c at img_off_256 * 256). Unit u =
// (chunk u / 16, 4 KiB round u % 16), one warp per unit, grid-stride: the round's
// bytes in the registered buffer are compared with the shadow's; when they differ the
// round is copied into the shadow (which so becomes the current state) and the
// chunk's bit is set in dirty[c / 32] (zero before the launch). A pure stream: read S
// from the buffers + S from the shadow, write the changed rounds.
__global__ void __launch_bounds__(256) diff_kernel(const ChunkDesc* __restrict__ desc, uint64_t n,
                                                   uint8_t* __restrict__ shadow, uint32_t* __restrict__ dirty) {
  const int lane = threadIdx.x & 31;
  const unsigned full = 0xFFFFFFFFu;
  const uint64_t nwarps = (uint64_t)gridDim.x * (blockDim.x >> 5);
  for (uint64_t u = (uint64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); u < n * 16; u += nwarps) {
    const uint64_t c = u >> 4;
    const uint32_t r = (uint32_t)(u & 15u) * (uint32_t)kRoundBytes;
    const ChunkDesc d = desc[c];
    const uint32_t len = desc_len(d);
    if (r >= len) continue;
    const uint32_t nb = len - r < (uint32_t)kRoundBytes ? len - r : (uint32_t)kRoundBytes;
    const uint8_t* src = reinterpret_cast<const uint8_t*>(d.ptr) + r;
    uint8_t* sh = shadow + (uint64_t)d.img_off_256 * kBufferAlign + r;
    bool diff = false;
    if ((reinterpret_cast<uintptr_t>(src) & 15u) == 0) {
      // 16-byte granules (each warp instruction = 512 contiguous bytes), then the tail
      const uint32_t ng = nb >> 4;
      uint4 a[8], b[8];
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        const uint32_t g = (uint32_t)lane + 32u * k;
        if (g < ng) {
          a[k] = __ldg(reinterpret_cast<const uint4*>(src) + g);
          b[k] = *(reinterpret_cast<const uint4*>(sh) + g);
        }
      }
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        const uint32_t g = (uint32_t)lane + 32u * k;
        if (g < ng) diff |= a[k].x != b[k].x || a[k].y != b[k].y || a[k].z != b[k].z || a[k].w != b[k].w;
      }
      const uint32_t t = (ng << 4) + (uint32_t)lane;
      uint8_t tb = 0;
      if (t < nb) {
        tb = src[t];
        diff |= tb != sh[t];
      }
      if (__any_sync(full, diff)) {
#pragma unroll
        for (int k = 0; k < 8; ++k) {
          const uint32_t g = (uint32_t)lane + 32u * k;
          if (g < ng) *(reinterpret_cast<uint4*>(sh) + g) = a[k];
        }
        if (t < nb) sh[t] = tb;
        if (lane == 0) atomicOr(&dirty[c >> 5], 1u << (c & 31));
      }
    } else {  // a misaligned registration (a tensor view with a storage offset): bytes
      for (uint32_t i = (uint32_t)lane; i < nb; i += 32) diff |= src[i] != sh[i];
      if (__any_sync(full, diff)) {
        for (uint32_t i = (uint32_t)lane; i < nb; i += 32) sh[i] = src[i];
        if (lane == 0) atomicOr(&dirty[c >> 5], 1u << (c & 31));
      }
    }
  }
}

// a5 on the GPU for large device images: the meta CRC's register over the CRC table
// and the zero pad that follows it (FORMAT.md meta_crc), continuing from the host's
// register after header and manifest. By CRC linearity, R(T || Z, s) = s x^(8|T||Z|) +
// R(T, 0) x^(8|Z|), and R(T, 0) is unchanged by leading zeros, so T is viewed as
// `lead` zero words followed by the table, cut into G*256 pieces of `per` words:
// thread t CRCs piece t from zero (slicing-by-4, per-CTA shared tables) and shifts it
// by C^(Ttot-1-t), C = x^(32 per), one multiply by a constant per set bit (nibble
// tables of C^(2^j) built per CTA); the pieces are XORed per CTA and across CTAs
// (atomicXor), and the last CTA applies the pad shift and the host's state term.
struct MetaParams {
  const uint32_t* table;
  uint64_t words, per, lead;
  uint32_t cpow[16];   // C^(2^j), C = x^(8 * 4 * per)
  uint32_t pad_pow;    // x^(8 |Z|)
  uint32_t state_term; // host register after header + manifest, times x^(8 |T||Z|)
  unsigned long long* acc;  // [0] XOR of the CTAs' terms, [1] CTAs done (zero at rest)
  uint32_t* out;            // mapped host word: the final CRC (complemented)
};
__global__ void __launch_bounds__(256) meta_crc_kernel(const MetaParams mp) {
  __shared__ uint32_t T[4][256];
  __shared__ uint32_t nib[16][8][16];  // nib[j][i][v] = (v << 4i) * cpow[j]
  __shared__ uint32_t red[8];
  const int tid = threadIdx.x;
  {
    uint32_t r = (uint32_t)tid;
    for (int b = 0; b < 8; ++b) r = gf_mulx(r);
    T[0][tid] = r;
  }
  for (int e = tid; e < 16 * 8 * 16; e += blockDim.x) {
    const int j = e >> 7, i = (e >> 4) & 7, v = e & 15;
    nib[j][i][v] = gf_mul((uint32_t)v << (4 * i), mp.cpow[j]);
  }
  __syncthreads();
  {
    uint32_t r = T[0][tid];
    for (int k = 1; k < 4; ++k) {
      r = (r >> 8) ^ T[0][r & 0xFFu];
      T[k][tid] = r;
    }
  }
  __syncthreads();
  const uint64_t t = (uint64_t)blockIdx.x * blockDim.x + tid, ttot = (uint64_t)gridDim.x * blockDim.x;
  uint32_t r = 0;
  for (uint64_t v = t * mp.per; v < (t + 1) * mp.per; ++v) {
    if (v < mp.lead) continue;  // leading zero words leave a zero register unchanged
    r ^= mp.table[v - mp.lead];
    r = T[3][r & 0xFFu] ^ T[2][(r >> 8) & 0xFFu] ^ T[1][(r >> 16) & 0xFFu] ^ T[0][r >> 24];
  }
  uint64_t m = ttot - 1 - t;  // pieces after this one
  for (int j = 0; m && r; ++j, m >>= 1) {
    if (!(m & 1u)) continue;
    uint32_t q = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i) q ^= nib[j][i][(r >> (4 * i)) & 15u];
    r = q;
  }
  for (int o = 16; o; o >>= 1) r ^= __shfl_xor_sync(0xFFFFFFFFu, r, o);
  if ((tid & 31) == 0) red[tid >> 5] = r;
  __syncthreads();
  if (tid == 0) {
    uint32_t c = 0;
    for (int w = 0; w < (int)(blockDim.x >> 5); ++w) c ^= red[w];
    atomicXor(&mp.acc[0], (unsigned long long)c);
    __threadfence();
    if (atomicAdd(&mp.acc[1], 1ull) == gridDim.x - 1) {  // the last CTA
      const uint32_t all = (uint32_t)atomicExch(&mp.acc[0], 0ull);
      atomicExch(&mp.acc[1], 0ull);
      *reinterpret_cast<volatile uint32_t*>(mp.out) = ~(mp.state_term ^ gf_mul(all, mp.pad_pow));
    }
  }
}

// CRC table of an exact delta: entry cidx[k] of `table` (the base's table) takes the
// CRC computed for present chunk k (ccrc[k], from the gather launches), k < totals[0].
__global__ void crc_scatter_kernel(const uint32_t* __restrict__ ccrc, const uint32_t* __restrict__ cidx,
                                   const unsigned long long* __restrict__ totals, uint32_t* __restrict__ table) {
  const uint64_t np = totals[0];
  for (uint64_t k = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; k < np; k += (uint64_t)gridDim.x * blockDim.x)
    table[cidx[k]] = ccrc[k];
}

// Present set -> bitmap words, compacted chunk list (img_off = offset in the compacted
// payload), [n_present, compacted bytes], and optionally the global index of each
// present chunk (cidx). Present: dirty[c/32] bit set when `dirty` is given (bytes
// rule), else crc_now[c] != crc_base[c] (CRC rule). One CTA, chunks in order.
__global__ void __launch_bounds__(1024, 1) delta_scan_kernel(const ChunkDesc* __restrict__ desc,
                                                             const uint32_t* __restrict__ crc_now,
                                                             const uint32_t* __restrict__ crc_base,
                                                             const uint32_t* __restrict__ dirty, uint64_t n,
                                                             uint32_t* __restrict__ map_words,
                                                             ChunkDesc* __restrict__ cdesc, uint32_t* __restrict__ cidx,
                                                             unsigned long long* __restrict__ totals) {
  __shared__ unsigned long long w_bytes[32];
  __shared__ uint32_t w_cnt[32];
  __shared__ unsigned long long carry_bytes, carry_cnt;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) carry_bytes = carry_cnt = 0;
  __syncthreads();
  for (uint64_t base = 0; base < n; base += 1024) {
    const uint64_t i = base + threadIdx.x;
    const bool present = i < n && (dirty ? ((dirty[i >> 5] >> (i & 31)) & 1u) != 0 : crc_now[i] != crc_base[i]);
    ChunkDesc d{};
    if (present) d = desc[i];
    const unsigned long long span = present ? (unsigned long long)(desc_len(d) + desc_pad(d)) : 0ull;
    const uint32_t bits = __ballot_sync(0xFFFFFFFFu, present);
    if (lane == 0 && base + warp * 32 < n) map_words[(base >> 5) + warp] = bits;
    unsigned long long sb = span;
    uint32_t sc = present ? 1u : 0u;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned long long tb = __shfl_up_sync(0xFFFFFFFFu, sb, o);
      const uint32_t tc = __shfl_up_sync(0xFFFFFFFFu, sc, o);
      if (lane >= o) sb += tb, sc += tc;
    }
    if (lane == 31) w_bytes[warp] = sb, w_cnt[warp] = sc;
    __syncthreads();
    if (warp == 0) {
      unsigned long long xb = w_bytes[lane];
      uint32_t xc = w_cnt[lane];
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const unsigned long long tb = __shfl_up_sync(0xFFFFFFFFu, xb, o);
        const uint32_t tc = __shfl_up_sync(0xFFFFFFFFu, xc, o);
        if (lane >= o) xb += tb, xc += tc;
      }
      w_bytes[lane] = xb - w_bytes[lane];  // exclusive warp offsets
      w_cnt[lane] = xc - w_cnt[lane];
    }
    __syncthreads();
    const unsigned long long off = carry_bytes + w_bytes[warp] + sb - span;
    const unsigned long long idx = carry_cnt + w_cnt[warp] + sc - (present ? 1u : 0u);
    if (present) {
      ChunkDesc o;
      o.ptr = d.ptr;
      o.img_off_256 = (uint32_t)(off / kBufferAlign);
      o.len_pad = d.len_pad;
      cdesc[idx] = o;
      if (cidx) cidx[idx] = (uint32_t)i;
    }
    __syncthreads();
    if (threadIdx.x == 1023) carry_bytes = off + span, carry_cnt = idx + (present ? 1u : 0u);
    __syncthreads();
  }
  if (threadIdx.x == 0) totals[0] = carry_cnt, totals[1] = carry_bytes;
}

// Stage s of the compacted payload = the present chunks whose compacted start lies
// in [s*W, (s+1)*W); with W = slot - (64 KiB + 256) every stage fits one staging
// slot. first[s] = index of its first chunk (binary search over the ascending
// compacted offsets), lo[s] = that chunk's compacted start (total bytes if none).
__global__ void delta_stages_kernel(const ChunkDesc* __restrict__ cdesc, const unsigned long long* __restrict__ totals,
                                    uint64_t W, uint64_t n_stages, unsigned long long* __restrict__ first,
                                    unsigned long long* __restrict__ lo) {
  const uint64_t s = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  if (s > n_stages) return;
  const uint64_t np = totals[0], bytes = totals[1], want = s * W;
  uint64_t a = 0, b = np;  // first i with start(i) >= want
  while (a < b) {
    const uint64_t m = (a + b) >> 1;
    if ((uint64_t)cdesc[m].img_off_256 * kBufferAlign >= want) b = m; else a = m + 1;
  }
  first[s] = a;
  lo[s] = a < np ? (unsigned long long)cdesc[a].img_off_256 * kBufferAlign : bytes;
}

// ---- launchers (called from checl_engine.cpp) --------------------------------

cudaError_t launch_expand(const BufferRecord* recs, uint32_t n, uint64_t payload_bytes, uint64_t n_chunks,
                          ChunkDesc* out, uint32_t* round_base, uint64_t total_rounds, unsigned long long* status,
                          int n_sms, cudaStream_t s) {
  if (n_chunks == 0) return cudaSuccess;
  uint64_t blocks = (n_chunks + 255) / 256;
  if (blocks > (uint64_t)n_sms * 8) blocks = (uint64_t)n_sms * 8;
  expand_plan_kernel<<<(unsigned)blocks, 256, 0, s>>>(recs, n, payload_bytes, n_chunks, out, round_base, total_rounds,
                                                      status);
  return cudaGetLastError();
}

size_t snapshot_smem_bytes() { return kSmemBytes; }

template <int kOp>
static cudaError_t configure_op() {
  cudaError_t e = cudaFuncSetAttribute(snapshot_kernel<kOp>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmemBytes);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(sweep_kernel<kOp>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmemBytes);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(balanced_kernel<kOp>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kBalSmemBytes);
  if constexpr (kOp == kOpPack || kOp == kOpVerify || kOp == kOpCrc || kOp == kOpCheck)
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(tma_kernel<kOp, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kTmaSmemBytes);
#ifdef CHECL_EXPERIMENTS
  if constexpr (kOp == kOpPack || kOp == kOpVerify || kOp == kOpCrc || kOp == kOpCheck)
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(tma_kernel<kOp, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kTmaSmemBytes);
#endif
  return e;
}

// Kernel 4 as 2-CTA clusters with the multicast table prologue (experiments build
// only: measured no gain, profiles/r01o/table_mc_ab.txt): CHECL_TABLE_MC=1 asks for
// it; used only if every SM can hold a CTA of a co-resident cluster.
#ifdef CHECL_EXPERIMENTS
static bool g_table_mc = false;

static bool table_mc_possible() {
  int dev = 0, n_sms = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || cudaDeviceGetAttribute(&n_sms, cudaDevAttrMultiProcessorCount, dev))
    return false;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(n_sms & ~1));
  cfg.blockDim = dim3(kThreadsPerCta);
  cfg.dynamicSmemBytes = kTmaSmemBytes;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = 2;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  int n = 0;
  if (cudaOccupancyMaxActiveClusters(&n, tma_kernel<kOpPack, true>, &cfg) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return 2 * n >= (n_sms & ~1);
}
#else
constexpr bool g_table_mc = false;
#endif

cudaError_t snapshot_configure() {
  cudaError_t e = configure_op<kOpPack>();
  if (e == cudaSuccess) e = configure_op<kOpVerify>();
  if (e == cudaSuccess) e = configure_op<kOpCrc>();
  if (e == cudaSuccess) e = configure_op<kOpCheck>();
  if (e == cudaSuccess) e = configure_op<kOpCopy>();
  if (e == cudaSuccess) e = configure_op<kOpScatter>();
#ifdef CHECL_EXPERIMENTS
  if (e == cudaSuccess) {
    const char* m = std::getenv("CHECL_TABLE_MC");
    g_table_mc = m && std::atoi(m) != 0 && table_mc_possible();
  }
#endif
  return e;
}

cudaError_t launch_build_tables(const TableParams& tp, uint32_t* out, cudaStream_t s) {
  build_tables_kernel<<<1, 512, 0, s>>>(tp, out);
  return cudaGetLastError();
}

template <int kOp>
static void launch_op(const LaunchParams& p, unsigned ctas, cudaStream_t s, int kernel) {
  if constexpr (kOp == kOpPack || kOp == kOpVerify || kOp == kOpCrc || kOp == kOpCheck) {
    if (kernel == 4) {
      if (!g_table_mc) {
        tma_kernel<kOp, false><<<ctas, kThreadsPerCta, kTmaSmemBytes, s>>>(p);
        return;
      }
#ifdef CHECL_EXPERIMENTS
      cudaLaunchConfig_t cfg = {};
      cfg.gridDim = dim3(ctas);
      cfg.blockDim = dim3(kThreadsPerCta);
      cfg.dynamicSmemBytes = kTmaSmemBytes;
      cfg.stream = s;
      cudaLaunchAttribute at[1];
      at[0].id = cudaLaunchAttributeClusterDimension;
      at[0].val.clusterDim.x = 2;
      at[0].val.clusterDim.y = 1;
      at[0].val.clusterDim.z = 1;
      cfg.attrs = at;
      cfg.numAttrs = 1;
      cudaLaunchKernelEx(&cfg, tma_kernel<kOp, true>, p);
      return;
#endif
    }
  }
  if (kernel == 3 || kernel == 4)
    balanced_kernel<kOp><<<ctas, kThreadsPerCta, kBalSmemBytes, s>>>(p);
  else if (kernel == 2)
    sweep_kernel<kOp><<<ctas, kThreadsPerCta, kSmemBytes, s>>>(p);
  else
    snapshot_kernel<kOp><<<ctas, kThreadsPerCta, kSmemBytes, s>>>(p);
}

template <int kOp>
static const void* op_fn(int kernel, size_t* smem) {
  if constexpr (kOp == kOpPack || kOp == kOpVerify || kOp == kOpCrc || kOp == kOpCheck) {
    if (kernel == 4) {
      *smem = kTmaSmemBytes;
#ifdef CHECL_EXPERIMENTS
      if (g_table_mc) return reinterpret_cast<const void*>(tma_kernel<kOp, true>);
#endif
      return reinterpret_cast<const void*>(tma_kernel<kOp, false>);
    }
  }
  if (kernel == 3 || kernel == 4) {
    *smem = kBalSmemBytes;
    return reinterpret_cast<const void*>(balanced_kernel<kOp>);
  }
  *smem = kSmemBytes;
  return kernel == 2 ? reinterpret_cast<const void*>(sweep_kernel<kOp>)
                     : reinterpret_cast<const void*>(snapshot_kernel<kOp>);
}

static uint64_t snapshot_ctas(const LaunchParams& p, int n_sms, int kernel, uint64_t rounds) {
  const uint64_t chunks = p.c1 - p.c0;
  const uint64_t units = kernel >= 3 ? rounds : kernel == 2 ? chunks * 16 : chunks;
  uint64_t ctas = (units + kWarpsPerCta - 1) / kWarpsPerCta;
  ctas = ctas > (uint64_t)n_sms ? (uint64_t)n_sms : ctas;
  if (kernel == 4 && g_table_mc) ctas = ctas < 2 ? 2 : ctas & ~1ull;  // whole 2-CTA clusters
  return ctas;
}

// The kernel, grid and dynamic shared memory launch_snapshot would use (for a
// kernel node of a CUDA graph); *fn = nullptr when the launch has no chunks.
cudaError_t snapshot_launch_config(int op, const LaunchParams& p, int n_sms, int kernel, uint64_t rounds,
                                   const void** fn, unsigned* ctas, size_t* smem, unsigned* cluster) {
  *fn = nullptr;
  *cluster = kernel == 4 && g_table_mc && (op == kOpPack || op == kOpVerify || op == kOpCrc || op == kOpCheck) ? 2 : 1;
  if (p.c1 == p.c0) return cudaSuccess;
  *ctas = (unsigned)snapshot_ctas(p, n_sms, kernel, rounds);
  switch (op) {
    case kOpPack: *fn = op_fn<kOpPack>(kernel, smem); break;
    case kOpVerify: *fn = op_fn<kOpVerify>(kernel, smem); break;
    case kOpCrc: *fn = op_fn<kOpCrc>(kernel, smem); break;
    case kOpCheck: *fn = op_fn<kOpCheck>(kernel, smem); break;
    case kOpCopy: *fn = op_fn<kOpCopy>(kernel, smem); break;
    case kOpScatter: *fn = op_fn<kOpScatter>(kernel, smem); break;
    default: return cudaErrorInvalidValue;
  }
  return cudaSuccess;
}

// kernel 1 = warp per chunk (snapshot_kernel), 2 = 4 KiB units swept by the grid
// (sweep_kernel; p.unit_acc must be zero for the chunk range when the op CRCs —
// the kernel leaves it zero again)
// (3 = balanced_kernel: needs p.round_base; `rounds` = the launch's round count)
cudaError_t launch_snapshot(int op, const LaunchParams& p, int n_sms, cudaStream_t s, int kernel, uint64_t rounds) {
  if (p.c1 == p.c0) return cudaSuccess;
  const uint64_t ctas = snapshot_ctas(p, n_sms, kernel, rounds);
  switch (op) {
    case kOpPack: launch_op<kOpPack>(p, (unsigned)ctas, s, kernel); break;
    case kOpVerify: launch_op<kOpVerify>(p, (unsigned)ctas, s, kernel); break;
    case kOpCrc: launch_op<kOpCrc>(p, (unsigned)ctas, s, kernel); break;
    case kOpCheck: launch_op<kOpCheck>(p, (unsigned)ctas, s, kernel); break;
    case kOpCopy: launch_op<kOpCopy>(p, (unsigned)ctas, s, kernel); break;
    case kOpScatter: launch_op<kOpScatter>(p, (unsigned)ctas, s, kernel); break;
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

cudaError_t launch_delta_scan(const ChunkDesc* desc, const uint32_t* crc_now, const uint32_t* crc_base,
                              const uint32_t* dirty, uint64_t n, uint32_t* map_words, ChunkDesc* cdesc, uint32_t* cidx,
                              unsigned long long* totals, cudaStream_t s) {
  delta_scan_kernel<<<1, 1024, 0, s>>>(desc, crc_now, crc_base, dirty, n, map_words, cdesc, cidx, totals);
  return cudaGetLastError();
}

cudaError_t launch_meta_crc(const uint32_t* table, uint64_t table_bytes, uint64_t total_bytes, uint32_t state,
                            unsigned long long* acc, uint32_t* out, int n_sms, cudaStream_t s) {
  MetaParams mp{};
  mp.table = table;
  mp.words = table_bytes / 4;
  uint64_t grid = (mp.words + 255) / 256;  // at least one word per thread
  grid = grid < 1 ? 1 : grid > (uint64_t)n_sms ? (uint64_t)n_sms : grid;
  const uint64_t ttot = grid * 256;
  mp.per = (mp.words + ttot - 1) / ttot;
  mp.lead = mp.per * ttot - mp.words;
  uint32_t c = gf_x8n(4 * mp.per);
  for (int j = 0; j < 16; ++j, c = gf_mul(c, c)) mp.cpow[j] = c;
  mp.pad_pow = gf_x8n(total_bytes - table_bytes);
  mp.state_term = gf_mul(state, gf_x8n(total_bytes));
  mp.acc = acc;
  mp.out = out;
  meta_crc_kernel<<<(unsigned)grid, 256, 0, s>>>(mp);
  return cudaGetLastError();
}

cudaError_t launch_diff(const ChunkDesc* desc, uint64_t n, uint8_t* shadow, uint32_t* dirty, int n_sms,
                        cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  uint64_t blocks = (n * 16 + 7) / 8;  // 8 warps per CTA, one unit each per pass
  if (blocks > (uint64_t)n_sms * 8) blocks = (uint64_t)n_sms * 8;
  diff_kernel<<<(unsigned)blocks, 256, 0, s>>>(desc, n, shadow, dirty);
  return cudaGetLastError();
}

cudaError_t launch_crc_scatter(const uint32_t* ccrc, const uint32_t* cidx, const unsigned long long* totals,
                               uint64_t n_max, uint32_t* table, int n_sms, cudaStream_t s) {
  if (n_max == 0) return cudaSuccess;
  uint64_t blocks = (n_max + 255) / 256;
  if (blocks > (uint64_t)n_sms * 4) blocks = (uint64_t)n_sms * 4;
  crc_scatter_kernel<<<(unsigned)blocks, 256, 0, s>>>(ccrc, cidx, totals, table);
  return cudaGetLastError();
}

cudaError_t launch_delta_stages(const ChunkDesc* cdesc, const unsigned long long* totals, uint64_t W, uint64_t n_stages,
                                unsigned long long* first, unsigned long long* lo, cudaStream_t s) {
  const uint64_t n = n_stages + 1;
  delta_stages_kernel<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(cdesc, totals, W, n_stages, first, lo);
  return cudaGetLastError();
}

cudaError_t launch_fill(uint8_t* ptr, uint64_t bytes, uint64_t key, int kind, int n_sms, cudaStream_t s) {
  if (bytes == 0) return cudaSuccess;
  uint64_t blocks = ((bytes + 7) / 8 + 255) / 256;
  if (blocks > (uint64_t)n_sms * 8) blocks = (uint64_t)n_sms * 8;
  fill_kernel<<<(unsigned)blocks, 256, 0, s>>>(ptr, bytes, key, kind);
  return cudaGetLastError();
}

cudaError_t launch_compare(const uint8_t* a, const uint8_t* b, uint64_t bytes, unsigned long long* n_diff, int n_sms,
                           cudaStream_t s) {
  if (bytes == 0) return cudaSuccess;
  uint64_t blocks = (bytes / 16 + 255) / 256 + 1;
  if (blocks > (uint64_t)n_sms * 8) blocks = (uint64_t)n_sms * 8;
  compare_kernel<<<(unsigned)blocks, 256, 0, s>>>(a, b, bytes, n_diff);
  return cudaGetLastError();
}

}  // namespace checl
