// checl_kernels.cu — sm_100a kernels of the CheCL snapshot hot path.
//
//  K1 pack_gather_crc  (checkpoint step 2, §III-C; north_star "gather
//     ... into one contiguous checkpoint image carrying a per-64 KiB CRC32C")
//  K2 verify_scatter   (restart step 3, L16 §III-C; north_star "every chunk is
//     CRC-verified, and its bytes are scattered into freshly re-created buffers")
//  K6 debug fill / compare (test tooling: synth/ generator on the device)
//
// Both K1 and K2 are one template (snapshot_kernel<kVerify>): a persistent grid,
// one warp per 64 KiB chunk of a flat chunk list. The chunk is cut into 32
// contiguous 2 KiB stripes, one per lane; each lane runs a slicing-by-4 CRC over
// its stripe with lane-private lookup tables in shared memory (entry e of table k
// for lane l sits at word (k*256 + e)*32 + l, so every lane always reads its own
// bank: conflict-free lookups on random data). Data moves in rounds of 32 x 128 B:
// coalesced 16-byte global loads (each warp instruction covers four full 128-byte
// lines), a coalesced 16-byte store of the same registers to the destination, and
// a transposition through a padded 32 x 144 B shared-memory tile so that each lane
// then reads its own stripe segment with conflict-free 16-byte shared loads.
// The 32 stripe registers are folded with a 5-level warp-shuffle tree (multiply by
// x^(8*2048*2^k) mod P through nibble tables); a short chunk (the last chunk of a
// buffer) is corrected with one multiply by x^(-8z), z = 65536 - len.
// DESIGN.md §5 derives the resource budget.
#include <cuda_runtime.h>

#include "checl_internal.h"

namespace checl {

constexpr int kTabWords = 4 * 256 * 32;          // 128 KiB, lane-private slicing-by-4
constexpr int kFoldWords = kFoldLevels * 8 * 16; // 2.5 KiB nibble tables
constexpr int kStageBytes = 32 * kRowPitch;      // per warp
constexpr size_t kSmemBytes = (size_t)(kTabWords + kFoldWords) * 4 + (size_t)kWarpsPerCta * kStageBytes;

__device__ __forceinline__ uint4 ld_stream_v4(const void* p) {
  uint4 r;
  asm("ld.global.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
      : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
      : "l"(p));
  return r;
}

__device__ __forceinline__ uint32_t ld_stream_u32(const void* p) {
  uint32_t r;
  asm("ld.global.L1::no_allocate.u32 %0, [%1];" : "=r"(r) : "l"(p));
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

// One slicing-by-4 step over the little-endian word w (tl = this lane's column).
__device__ __forceinline__ uint32_t crc_step4(uint32_t crc, uint32_t w, const uint32_t* tl) {
  const uint32_t x = crc ^ w;
  return tl[(768u + (x & 0xFFu)) << 5] ^ tl[(512u + ((x >> 8) & 0xFFu)) << 5] ^
         tl[(256u + ((x >> 16) & 0xFFu)) << 5] ^ tl[(x >> 24) << 5];
}

__device__ __forceinline__ uint32_t crc_step1(uint32_t crc, uint32_t b, const uint32_t* tl) {
  return (crc >> 8) ^ tl[((crc ^ b) & 0xFFu) << 5];
}

__device__ __forceinline__ uint32_t crc_step16(uint32_t crc, uint4 q, const uint32_t* tl) {
  crc = crc_step4(crc, q.x, tl);
  crc = crc_step4(crc, q.y, tl);
  crc = crc_step4(crc, q.z, tl);
  return crc_step4(crc, q.w, tl);
}

// f * x^(8*2048*2^level) mod P via 8 nibble lookups.
__device__ __forceinline__ uint32_t fold_mul(uint32_t f, const uint32_t* ft) {
  uint32_t r = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) r ^= ft[j * 16 + ((f >> (4 * j)) & 15u)];
  return r;
}

template <bool kVerify>
__global__ void __launch_bounds__(kThreadsPerCta, 1) snapshot_kernel(const LaunchParams p) {
  extern __shared__ __align__(16) uint32_t smem[];
  uint32_t* tab = smem;
  uint32_t* ftab = smem + kTabWords;
  uint8_t* stage_all = reinterpret_cast<uint8_t*>(smem + kTabWords + kFoldWords);

  // Tables: T_k[e] = CRC register of byte e followed by k zero bytes (zero init),
  // replicated once per lane; fold nibble tables N_l[j][v] = (v << 4j) * C_l.
  for (int i = threadIdx.x; i < 1024; i += blockDim.x) {
    const int k = i >> 8;
    uint32_t r = (uint32_t)(i & 255);
    for (int b = 0; b < 8 * (k + 1); ++b) r = gf_mulx(r);
    uint4* dstv = reinterpret_cast<uint4*>(tab + (i << 5));
    const uint4 rv = make_uint4(r, r, r, r);
#pragma unroll
    for (int j = 0; j < 8; ++j) dstv[j] = rv;
  }
  for (int i = threadIdx.x; i < kFoldWords; i += blockDim.x) {
    const int lvl = i >> 7, j = (i >> 4) & 7, v = i & 15;
    // select, not p.fold[lvl]: a dynamic index into kernel parameters spills them to the stack
    const uint32_t cl = lvl == 0 ? p.fold[0] : lvl == 1 ? p.fold[1] : lvl == 2 ? p.fold[2] : lvl == 3 ? p.fold[3] : p.fold[4];
    ftab[i] = gf_mul((uint32_t)v << (4 * j), cl);
  }
  __syncthreads();

  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint8_t* stage = stage_all + warp * kStageBytes;
  const uint32_t* tl = tab + lane;
  const uint64_t nwarps = (uint64_t)gridDim.x * kWarpsPerCta;
  const unsigned full = 0xFFFFFFFFu;
  // this lane's slot for the transposition stores / its own row for the CRC
  const int g_lane = lane & 7, s_lane = lane >> 3;

  for (uint64_t c = p.c0 + (uint64_t)blockIdx.x * kWarpsPerCta + warp; c < p.c1; c += nwarps) {
    const ChunkDesc d = p.desc[c];
    const uint32_t len = desc_len(d), pad = desc_pad(d);
    uint8_t* img = p.image + ((uint64_t)d.img_off_256 * kBufferAlign - p.image_base);
    const uint8_t* src = kVerify ? img : reinterpret_cast<const uint8_t*>(d.ptr);
    uint8_t* dst = kVerify ? reinterpret_cast<uint8_t*>(d.ptr) : img;
    const int mode = kVerify ? 0 : ((d.ptr & 15u) == 0 ? 0 : ((d.ptr & 3u) == 0 ? 1 : 2));

    const int my_len = min(max((int)len - lane * kStripeBytes, 0), kStripeBytes);
    uint32_t crc = lane == 0 ? 0xFFFFFFFFu : 0u;
    const uint32_t longest = len < (uint32_t)kStripeBytes ? len : (uint32_t)kStripeBytes;
    const int nrounds = (int)((longest + kSegBytes - 1) / kSegBytes);

    for (int r = 0; r < nrounds; ++r) {
      uint4 v[8];
      uint32_t off[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        off[i] = (uint32_t)(4 * i + s_lane) * kStripeBytes + (uint32_t)r * kSegBytes + (uint32_t)g_lane * 16;
        if (off[i] + 16 <= len)
          v[i] = ld_granule(src + off[i], mode);
        else if (off[i] < len)
          v[i] = ld_partial(src + off[i], len - off[i]);
        else
          v[i] = make_uint4(0u, 0u, 0u, 0u);
      }
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        if (off[i] < len) {
          if (!kVerify || off[i] + 16 <= len)
            *reinterpret_cast<uint4*>(dst + off[i]) = v[i];  // pack: zeros past len are owned padding
          else
            st_partial(dst + off[i], v[i], len - off[i]);
        }
        *reinterpret_cast<uint4*>(stage + (4 * i + s_lane) * kRowPitch + g_lane * 16) = v[i];
      }
      __syncwarp();
      const int vb = min(max(my_len - r * kSegBytes, 0), kSegBytes);
      const uint4* row = reinterpret_cast<const uint4*>(stage + lane * kRowPitch);
      if (vb == kSegBytes) {
#pragma unroll
        for (int g = 0; g < 8; ++g) crc = crc_step16(crc, row[g], tl);
      } else if (vb > 0) {
        const int nw = vb >> 2;
        const uint32_t* roww = reinterpret_cast<const uint32_t*>(row);
        for (int w = 0; w < nw; ++w) crc = crc_step4(crc, roww[w], tl);
        if (vb & 3) {
          const uint32_t w = roww[nw];
          for (int b = 0; b < (vb & 3); ++b) crc = crc_step1(crc, (w >> (8 * b)) & 0xFFu, tl);
        }
      }
      __syncwarp();
    }

    uint32_t pad_bad = 0;
    if (pad) {
      if (!kVerify) {
        const uint32_t start = (len + 15u) & ~15u, end = len + pad;
        for (uint32_t o = start + lane * 16u; o < end; o += 512u)
          *reinterpret_cast<uint4*>(dst + o) = make_uint4(0u, 0u, 0u, 0u);
      } else {
        for (uint32_t o = len + lane; o < len + pad; o += 32u) pad_bad |= src[o];
      }
    }
    if (kVerify) pad_bad = __any_sync(full, pad_bad != 0);

    // Fold the full stripes: at level k lane l (l % 2^(k+1) == 0) combines its
    // group with the one 2^k stripes to the right: shift left group by 2048*2^k B.
    const uint32_t q = len / kStripeBytes;
    uint32_t f = ((uint32_t)lane < q) ? crc : 0u;
#pragma unroll
    for (int k = 0; k < kFoldLevels; ++k) {
      const uint32_t o = __shfl_down_sync(full, f, 1 << k);
      if ((lane & ((2 << k) - 1)) == 0) f = fold_mul(f, ftab + k * 128) ^ o;
    }
    const uint32_t rq = __shfl_sync(full, crc, (int)(q & 31u));
    if (lane == 0) {
      uint32_t t = f;
      if (len < kChunkBytes) t = gf_mul(t, p.inv_z[kChunkBytes - len]) ^ rq;
      const uint32_t out = ~t;
      if (!kVerify) {
        p.crc[c] = out;
      } else if (out != p.crc[c] || pad_bad) {
        atomicMin(&p.status[0], (unsigned long long)c);
        atomicAdd(&p.status[1], 1ull);
      }
    }
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

// ---- launchers (called from checl_engine.cpp) --------------------------------

size_t snapshot_smem_bytes() { return kSmemBytes; }

cudaError_t snapshot_configure() {
  cudaError_t e = cudaFuncSetAttribute(snapshot_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmemBytes);
  if (e != cudaSuccess) return e;
  return cudaFuncSetAttribute(snapshot_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmemBytes);
}

cudaError_t launch_snapshot(bool verify, const LaunchParams& p, int n_sms, cudaStream_t s) {
  const uint64_t chunks = p.c1 - p.c0;
  if (chunks == 0) return cudaSuccess;
  uint64_t ctas = (chunks + kWarpsPerCta - 1) / kWarpsPerCta;
  if (ctas > (uint64_t)n_sms) ctas = (uint64_t)n_sms;
  if (verify)
    snapshot_kernel<true><<<(unsigned)ctas, kThreadsPerCta, kSmemBytes, s>>>(p);
  else
    snapshot_kernel<false><<<(unsigned)ctas, kThreadsPerCta, kSmemBytes, s>>>(p);
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
