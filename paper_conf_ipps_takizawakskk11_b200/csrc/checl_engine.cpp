// checl_engine.cpp — libchecl host engine and C ABI (include/checl.h).
//
// Object database + handle table (§III-B, L19 §III-C), checkpoint
// (L16 §III-C steps 1, 2, 4), restart (L16 restart steps 2-3, restore order
// L19-L20 reduced to device -> buffers -> rebind), migration (L40 §IV-C), over the
// image layout of FORMAT.md. The data path runs in checl_kernels.cu; this file
// plans it (flat chunk list, stages), drives the staging pipeline on two streams
// (copy engine D2H/H2D overlapped with the pack / verify kernels), and commits.
//
// State kept across calls:
//   Plan         per device: the registry's chunk list, stages, header + manifest and
//                their meta-CRC register, cached per registry version;
//   LayoutCache  per device: the last full-image restore's layout (restore fast path);
//   Binding      per commit: where its records live (segment + offset) and the
//                segments themselves (re-created buffers, reading 18);
//   spares       per device: the segments the last commit released (next restore);
//   shadow       per device: the exact incremental rule's copy of the last delta's
//                state (reading 25).
#include <cuda_runtime.h>
#include <fcntl.h>
#include <signal.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <unistd.h>

#include <algorithm>
#include <unordered_map>
#include <unordered_set>
#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>
#include <new>
#include <string>
#include <thread>
#include <vector>

#include "../../include/checl.h"
#include "checl_internal.h"

namespace checl {
size_t snapshot_smem_bytes();
cudaError_t snapshot_configure();
cudaError_t launch_snapshot(int op, const LaunchParams& p, int n_sms, cudaStream_t s, int kernel, uint64_t rounds);
cudaError_t snapshot_launch_config(int op, const LaunchParams& p, int n_sms, int kernel, uint64_t rounds,
                                   const void** fn, unsigned* ctas, size_t* smem, unsigned* cluster);
cudaError_t launch_build_tables(const TableParams& tp, uint32_t* out, cudaStream_t s);
cudaError_t launch_fill(uint8_t* ptr, uint64_t bytes, uint64_t key, int kind, int n_sms, cudaStream_t s);
cudaError_t launch_compare(const uint8_t* a, const uint8_t* b, uint64_t bytes, unsigned long long* n_diff, int n_sms,
                           cudaStream_t s);
cudaError_t launch_delta_scan(const ChunkDesc* desc, const uint32_t* crc_now, const uint32_t* crc_base,
                              const uint32_t* dirty, uint64_t n, uint32_t* map_words, ChunkDesc* cdesc, uint32_t* cidx,
                              unsigned long long* totals, cudaStream_t s);
cudaError_t launch_diff(const ChunkDesc* desc, uint64_t n, uint8_t* shadow, uint32_t* dirty, int n_sms, cudaStream_t s);
cudaError_t launch_meta_crc(const uint32_t* table, uint64_t table_bytes, uint64_t total_bytes, uint32_t state,
                            unsigned long long* acc, uint32_t* out, int n_sms, cudaStream_t s);
cudaError_t launch_crc_scatter(const uint32_t* ccrc, const uint32_t* cidx, const unsigned long long* totals,
                               uint64_t n_max, uint32_t* table, int n_sms, cudaStream_t s);
cudaError_t launch_delta_stages(const ChunkDesc* cdesc, const unsigned long long* totals, uint64_t W, uint64_t n_stages,
                                unsigned long long* first, unsigned long long* lo, cudaStream_t s);
cudaError_t launch_expand(const BufferRecord* recs, uint32_t n, uint64_t payload_bytes, uint64_t n_chunks,
                          ChunkDesc* out, uint32_t* round_base, uint64_t total_rounds, unsigned long long* status,
                          int n_sms, cudaStream_t s);
uint32_t host_crc32c_update(uint32_t crc, const void* data, size_t n);
uint32_t host_crc32c(const void* data, size_t n);
}  // namespace checl

using namespace checl;

namespace {

constexpr int kMaxDevices = 64;
constexpr uint32_t kMaxSlots = 8;
constexpr size_t kSlotSlack = 256;  // pack writes whole 16-B granules past a last buffer's end
constexpr size_t kDefaultSlotBytes = 64ull << 20;
constexpr uint64_t kMetaKernelMinBytes = 128u << 10;  // CRC tables at least this large: meta CRC on the GPU

thread_local std::string t_last_cuda_error;

// signal number -> context of checl_install_signal (delayed checkpointing mode)
constexpr int kMaxSignal = 65;
std::atomic<checl_ctx*> g_signal_ctx[kMaxSignal];

// Pinned host memory for images. cudaHostAlloc pins at ~2.4-2.8 GB/s on the B200
// boxes (page by page, one thread); a large buffer is instead taken 2 MiB-aligned with
// transparent huge pages requested, faulted in by several threads at once and
// registered with one cudaHostRegister: 26-30 GB/s for 4-8 GiB, copies at the same
// PCIe rate (tools/microbench/pin_rate.cu, profiles/r02/pin_rate.txt). Buffers under
// 8 MiB keep cudaHostAlloc. pin_free knows which is which.
constexpr size_t kFastPinMin = 8ull << 20;
// buffers of pin_alloc's registered path (never destroyed: images may be freed while
// the process exits, after static destructors ran)
struct Registered {
  std::mutex mu;
  std::unordered_set<void*> set;
};
Registered& registered() {
  static Registered* r = new Registered();
  return *r;
}

void* pin_alloc(size_t n) {
  if (n >= kFastPinMin) {
    void* p = nullptr;
    if (posix_memalign(&p, 2u << 20, n) == 0) {
      madvise(p, n, MADV_HUGEPAGE);  // (advice only: 4 KiB pages still work)
      // one thread per 32 MiB, at most 16 (and the machine's count)
      const unsigned hw = std::thread::hardware_concurrency();
      const size_t T = std::max<size_t>(1, std::min<size_t>({16, hw ? hw : 4, n >> 25}));
      const size_t piece = (n / T + (2u << 20) - 1) & ~(size_t)((2u << 20) - 1);
      auto touch = [=](size_t t) {
        volatile uint8_t* q = static_cast<uint8_t*>(p) + t * piece;
        const size_t m = std::min(piece, n - t * piece);
        for (size_t o = 0; o < m; o += 4096) q[o] = 0;
      };
      std::vector<std::thread> th;
      for (size_t t = 1; t < T && t * piece < n; ++t) th.emplace_back(touch, t);
      touch(0);
      for (auto& x : th) x.join();
      if (cudaHostRegister(p, n, cudaHostRegisterPortable | cudaHostRegisterMapped) == cudaSuccess) {
        std::lock_guard<std::mutex> lk(registered().mu);
        registered().set.insert(p);
        return p;
      }
      cudaGetLastError();
      std::free(p);
    }
  }
  void* p = nullptr;
  if (cudaHostAlloc(&p, n, cudaHostAllocPortable | cudaHostAllocMapped) != cudaSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  return p;
}

void pin_free(void* p) {
  if (!p) return;
  bool reg = false;
  {
    std::lock_guard<std::mutex> lk(registered().mu);
    reg = registered().set.erase(p) != 0;
  }
  if (reg) {
    cudaHostUnregister(p);
    std::free(p);
  } else {
    cudaFreeHost(p);
  }
}

// Pinned host buffers of freed library-owned images, kept for the next image
// (cudaHostAlloc pins ~2.4 GB/s on the B200 boxes: an incremental checkpoint loop, or
// a file restore loop, would otherwise pin a new image every step). Bounded by
// CHECL_PINNED_POOL_BYTES (default min(16 GiB, 1/8 of the host's RAM): a 4 GiB cap
// re-pinned every C3-sized image, 1.8 s per 4 GiB, profiles/r02/cost_model_*); the
// least recently returned buffers are released first; checl_trim empties it. Pinned sizes are rounded up to size classes (<= 12.5% slack) so
// that images of similar size reuse each other's buffers.
size_t pinned_class(size_t n) {
  if (n <= (2u << 20)) return (n + 4095) & ~(size_t)4095;
  size_t p2 = 1;
  while (p2 * 2 <= n) p2 *= 2;
  const size_t step = std::max<size_t>(p2 / 8, 2u << 20);
  return (n + step - 1) / step * step;
}

struct PinnedPool {
  std::mutex mu;
  std::vector<std::pair<size_t, void*>> free_;  // oldest first
  size_t bytes = 0, limit = 0;
  PinnedPool() {
    const char* e = std::getenv("CHECL_PINNED_POOL_BYTES");
    const long pages = sysconf(_SC_PHYS_PAGES), psz = sysconf(_SC_PAGESIZE);
    const size_t ram = pages > 0 && psz > 0 ? (size_t)pages * (size_t)psz : (32ull << 30);
    limit = e ? (size_t)std::strtoull(e, nullptr, 10) : std::min<size_t>(16ull << 30, ram / 8);
  }
  // the smallest pooled buffer with n <= capacity <= 2n + 64 MiB, or nullptr
  void* take(size_t n, size_t* cap) {
    std::lock_guard<std::mutex> lk(mu);
    size_t best = free_.size();
    for (size_t i = 0; i < free_.size(); ++i)
      if (free_[i].first >= n && free_[i].first <= 2 * n + (64ull << 20) &&
          (best == free_.size() || free_[i].first < free_[best].first))
        best = i;
    if (best == free_.size()) return nullptr;
    void* p = free_[best].second;
    *cap = free_[best].first;
    bytes -= *cap;
    free_.erase(free_.begin() + (long)best);
    return p;
  }
  void trim() {
    std::vector<std::pair<size_t, void*>> all;
    {
      std::lock_guard<std::mutex> lk(mu);
      all.swap(free_);
      bytes = 0;
    }
    for (auto& e : all) pin_free(e.second);
  }
  void give(void* p, size_t cap) {
    std::vector<void*> drop;
    {
      std::lock_guard<std::mutex> lk(mu);
      if (cap > limit) {
        drop.push_back(p);
      } else {
        free_.emplace_back(cap, p);
        bytes += cap;
        while (bytes > limit) {  // evict the oldest
          drop.push_back(free_.front().second);
          bytes -= free_.front().first;
          free_.erase(free_.begin());
        }
      }
    }
    for (void* d : drop) pin_free(d);
  }
};
PinnedPool& pinned_pool() {
  static PinnedPool* pool = new PinnedPool();  // never destroyed: may outlive the CUDA runtime
  return *pool;
}

double now_ms() {
  return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

// CHECL_TRACE=1: host timestamps of an op's phases on stderr (diagnostics only).
struct Trace {
  bool on;
  double t0, last;
  std::string line;
  explicit Trace(const char* op) : on(std::getenv("CHECL_TRACE") != nullptr), t0(now_ms()), last(t0) {
    if (on) line = op;
  }
  void operator()(const char* what) {
    if (!on) return;
    const double t = now_ms();
    char buf[64];
    std::snprintf(buf, sizeof buf, " %s=%.1f", what, (t - last) * 1e3);
    line += buf;
    last = t;
  }
  ~Trace() {
    if (on) std::fprintf(stderr, "[checl] %s total=%.1f us\n", line.c_str(), (now_ms() - t0) * 1e3);
  }
};

uint64_t align_up(uint64_t x, uint64_t a) { return (x + a - 1) / a * a; }
uint64_t chunks_of(uint64_t size) { return (size + kChunkBytes - 1) / kChunkBytes; }

void put_u32(uint8_t* p, uint32_t v) { std::memcpy(p, &v, 4); }
void put_u64(uint8_t* p, uint64_t v) { std::memcpy(p, &v, 8); }
uint32_t get_u32(const uint8_t* p) {
  uint32_t v;
  std::memcpy(&v, p, 4);
  return v;
}
uint64_t get_u64(const uint8_t* p) {
  uint64_t v;
  std::memcpy(&v, p, 8);
  return v;
}

struct CudaFail {
  cudaError_t e;
};

// Throws on a CUDA error; the C ABI converts it into CHECL_ERR_CUDA.
void ck(cudaError_t e) {
  if (e != cudaSuccess) {
    t_last_cuda_error = cudaGetErrorName(e);
    cudaGetLastError();
    throw CudaFail{e};
  }
}

int fake_devices() {
  static const int n = [] {
    const char* s = std::getenv("CHECL_FAKE_DEVICES");
    return s ? std::atoi(s) : 0;
  }();
  return n;
}

int device_count() {
  static const int n = [] {
    int c = 0;
    if (cudaGetDeviceCount(&c) != cudaSuccess) {
      cudaGetLastError();
      c = 0;
    }
    return c;
  }();
  return n > 0 ? n : fake_devices();
}

bool valid_device(int d) { return d >= 0 && d < device_count() && d < kMaxDevices; }

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int d) {
    ck(cudaGetDevice(&prev));
    if (prev != d) ck(cudaSetDevice(d));
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

// x^(-8z) mod P for z in [0, 4096): the zero-padding correction of the kernels.
const std::vector<uint32_t>& inv_z_table() {
  static const std::vector<uint32_t> t = [] {
    std::vector<uint32_t> v(kRoundBytes);
    uint32_t r = kOne;
    for (uint32_t z = 0; z < (uint32_t)kRoundBytes; ++z) {
      v[z] = r;
      for (int b = 0; b < 8; ++b) r = gf_divx(r);
    }
    return v;
  }();
  return t;
}

TableParams table_params() {
  TableParams tp{};
  for (int k = 0; k < kFoldLevels; ++k) tp.fold[k] = gf_x_pow2k(10 + k);  // x^(8*128*2^k)
  tp.horner = gf_x8n(kRoundBytes - kSegBytes);
  for (int l = 0; l < 32; ++l) tp.lanepow[l] = gf_x8n((uint64_t)kSegBytes * (31 - l));
  for (int k = 0; k < 16; ++k) tp.unitpow[k] = gf_x8n((uint64_t)kRoundBytes * k);
  tp.col_shift = gf_x8n((uint64_t)kSegBytes * kColChains);
  for (int k = 0; k < kColFoldLevels; ++k) {
    uint32_t r = kOne;
    for (int i = 0; i < 32 << k; ++i) r = gf_divx(r);  // x^(-32 * 2^k)
    tp.col_fold[k] = r;
  }
  return tp;
}

// ---- per-device resources ---------------------------------------------------

// One instantiated CUDA graph [event record a -> snapshot kernel -> event record b]
// per (kernel function, grid): a timed launch updates the kernel node's parameters
// and the two events and launches the graph, so the GPU receives the three together
// (the host's launch latency is no longer inside the kernel's event span) and the
// host spends one graph launch instead of record + launch + record
// (profiles/r01k/launch_graph.txt). CHECL_GRAPH=0 uses plain stream launches.
struct LaunchGraph {
  const void* fn = nullptr;
  unsigned ctas = 0;
  cudaGraph_t graph = nullptr;  // kept: the exec updates name its nodes by these handles
  cudaGraphExec_t exec = nullptr;
  cudaGraphNode_t ev_a = nullptr, kern = nullptr, ev_b = nullptr;
};

// Two halves used by alternate calls on a device: the event spans of a call stay
// readable during the next call, which reads them while its own kernel runs
// (deferred timing, see PendingTiming).
struct EventPool {
  std::vector<cudaEvent_t> ev[2];
  size_t used = 0;
  int active = 0;
  cudaEvent_t get() {
    std::vector<cudaEvent_t>& v = ev[active];
    if (used == v.size()) {
      cudaEvent_t e;
      ck(cudaEventCreate(&e));
      v.push_back(e);
    }
    return v[used++];
  }
  void reset() {
    active ^= 1;
    used = 0;
  }
  void destroy_all() {
    for (auto& v : ev) {
      for (auto e : v) cudaEventDestroy(e);
      v.clear();
    }
  }
  ~EventPool() { destroy_all(); }
};

template <typename T>
struct DevBuf {  // grow-only device scratch (cudaMalloc)
  T* p = nullptr;
  size_t cap = 0;
  void ensure(size_t n) {
    if (n <= cap) return;
    if (p) cudaFree(p);
    p = nullptr;
    cap = 0;
    ck(cudaMalloc(&p, std::max<size_t>(n, 1) * sizeof(T)));
    cap = n;
  }
  void release() {
    if (p) cudaFree(p);
    p = nullptr;
    cap = 0;
  }
};

template <typename T>
struct PinnedBuf {  // grow-only pinned host scratch
  T* p = nullptr;
  size_t cap = 0;
  void ensure(size_t n, unsigned flags = cudaHostAllocDefault) {
    if (n <= cap) return;
    if (p) cudaFreeHost(p);
    p = nullptr;
    cap = 0;
    ck(cudaHostAlloc(reinterpret_cast<void**>(&p), std::max<size_t>(n, 1) * sizeof(T), flags));
    cap = n;
  }
  void release() {
    if (p) cudaFreeHost(p);
    p = nullptr;
    cap = 0;
  }
};

struct Stage {
  uint64_t c0, c1, img_lo, img_hi;
};

struct BufRec {
  uint64_t handle, size, off, first_chunk;
  uint32_t flags;
  uint8_t* ptr;
};

// Everything a checkpoint of one device needs that depends only on the registry
// (cached until the registry of that device changes).
struct Plan {
  uint64_t version = ~0ull;
  size_t slot_bytes = 0;
  std::vector<BufRec> bufs;
  uint64_t n_chunks = 0, payload_bytes = 0, crc_off = 0, payload_off = 0, image_bytes = 0;
  std::vector<BufferRecord> recs;
  std::vector<Stage> stages;
  std::vector<uint8_t> meta;  // header (meta_crc = 0, epoch = 0) + manifest
  // the CRC32C register after meta's header bytes [0, 124) and manifest [128, crc_off)
  // (epoch 0), and x^(8 (crc_off - 100)): the shift of the epoch bytes to the end of
  // the manifest (finalize adds the epoch by linearity instead of re-reading the
  // manifest); meta_gen changes whenever meta is rebuilt
  uint32_t meta_state0 = 0, epoch_shift = 0;
  uint64_t meta_gen = 0;
  // the restore layout (LayoutCache::gen) the plan's buffers were re-created with, and
  // the segments its chunk list addresses (0 / empty: built from the registry)
  uint64_t layout_gen = 0;
  std::vector<void*> list_bases;
  DevBuf<ChunkDesc> d_desc;
  DevBuf<uint32_t> d_round;  // round_base of the balanced kernel (n_chunks + 1)
  DevBuf<BufferRecord> d_recs;
};

struct DevState {
  int dev = -1, n_sms = 0;
  cudaStream_t compute = nullptr, copy = nullptr;
  DevBuf<uint8_t> slots;
  size_t slot_bytes = 0;
  uint32_t n_slots = 0;
  DevBuf<uint32_t> inv_z, crc_scratch, tables;
  DevBuf<ChunkDesc> desc_scratch;
  DevBuf<uint32_t> round_scratch;
  DevBuf<BufferRecord> recs_scratch;
  // what desc_scratch / round_scratch hold: the chunk list of layout scratch_gen over
  // the segments at scratch_bases (0: nothing known); a restore with the same key
  // skips its expansion
  uint64_t scratch_gen = 0;
  std::vector<void*> scratch_bases;
  // verify status {first bad, n bad, CTAs done}; between restores it rests at
  // {~0, 0, 0} (reset by the publishing launch) unless status_clean is false
  DevBuf<unsigned long long> status;
  bool status_clean = false;
  unsigned long long* status_host_dev = nullptr;  // device address of h_status (mapped), or nullptr
  DevBuf<unsigned long long> unit_acc;
  DevBuf<unsigned long long> warp_trace;  // CHECL_WARP_TRACE diagnostics
  DevBuf<unsigned long long> work;        // dynamic-block counter + finished CTAs (zero at rest)
  // incremental checkpoint (f1): base CRC table, bitmap words, compacted chunk
  // list, [n_present, bytes], stage table
  DevBuf<uint32_t> base_crc, map_words;
  DevBuf<ChunkDesc> cdesc;
  DevBuf<unsigned long long> dtotals, stage_first, stage_lo;
  PinnedBuf<unsigned long long> h_dtab;
  // exact incremental checkpoint (dirty rule 1, reading 25): the shadow holds
  // the payload of the state a checkpoint last described (payload layout), identified by
  // that image's epoch, CRC-table CRC and manifest CRC; dirty bits, the compacted
  // chunks' CRCs and global indices
  DevBuf<uint8_t> shadow;
  bool shadow_ok = false;
  uint64_t shadow_epoch = 0, shadow_payload = 0;
  uint32_t shadow_table_crc = 0, shadow_meta_crc = 0;
  DevBuf<uint32_t> dirty, ccrc, cidx;
  // 1 = warp per chunk (throughput), 2 = 4 KiB units swept by the grid (latency of
  // small launches), 3 = balanced stretches of rounds, 4 = balanced stretches with
  // bulk (TMA) copies and the column CRC; 0 = by plan; env
  // CHECL_KERNEL=1..4 forces one
  int kernel = 0;
  uint64_t aux_launches = 0;  // plan expansion / delta scan kernels (checl_timing.n_kernels)
  PinnedBuf<unsigned long long> h_status;
  PinnedBuf<BufferRecord> h_recs;
  // the meta CRC a meta_crc_kernel computed (mapped pinned word) and its device address
  PinnedBuf<uint32_t> h_meta;
  uint32_t* meta_dev = nullptr;
  DevBuf<unsigned long long> meta_acc;  // meta_crc_kernel's accumulator + CTA count (zero at rest)
  EventPool events;
  std::vector<LaunchGraph> graphs;
  Plan plan;

  void init(int d) {
    dev = d;
    DeviceGuard g(d);
    ck(cudaDeviceGetAttribute(&n_sms, cudaDevAttrMultiProcessorCount, d));
    ck(cudaStreamCreateWithFlags(&compute, cudaStreamNonBlocking));
    ck(cudaStreamCreateWithFlags(&copy, cudaStreamNonBlocking));
    ck(snapshot_configure());
    inv_z.ensure(kRoundBytes);
    ck(cudaMemcpy(inv_z.p, inv_z_table().data(), kRoundBytes * 4, cudaMemcpyHostToDevice));
    work.ensure(2);
    ck(cudaMemset(work.p, 0, 2 * sizeof(unsigned long long)));
    status.ensure(3);
    h_status.ensure(2, cudaHostAllocMapped);
    {
      void* dp = nullptr;
      if (cudaHostGetDevicePointer(&dp, h_status.p, 0) == cudaSuccess)
        status_host_dev = static_cast<unsigned long long*>(dp);
      else
        cudaGetLastError();
      const unsigned long long init[3] = {~0ull, 0ull, 0ull};
      ck(cudaMemcpy(status.p, init, sizeof(init), cudaMemcpyHostToDevice));
      status_clean = true;
    }
    h_meta.ensure(1, cudaHostAllocMapped);
    meta_acc.ensure(2);
    ck(cudaMemset(meta_acc.p, 0, 2 * sizeof(unsigned long long)));
    {
      void* dp = nullptr;
      if (cudaHostGetDevicePointer(&dp, h_meta.p, 0) == cudaSuccess)
        meta_dev = static_cast<uint32_t*>(dp);
      else
        cudaGetLastError();
    }
    tables.ensure(kTableWords);
    ck(launch_build_tables(table_params(), tables.p, compute));
    ck(cudaStreamSynchronize(compute));
    if (const char* k = std::getenv("CHECL_KERNEL")) kernel = std::atoi(k) >= 1 && std::atoi(k) <= 4 ? std::atoi(k) : 0;
  }
  void ensure_slots(size_t bytes, uint32_t n) {
    if (slot_bytes == bytes && n_slots == n && slots.p) return;
    slots.release();
    slots.ensure(n * (bytes + kSlotSlack));
    slot_bytes = bytes;
    n_slots = n;
  }
  uint8_t* slot(uint32_t i) { return slots.p + (size_t)i * (slot_bytes + kSlotSlack); }
  void destroy() {
    if (dev < 0) return;
    int prev = -1;
    cudaGetDevice(&prev);
    cudaSetDevice(dev);
    cudaDeviceSynchronize();
    slots.release();
    inv_z.release();
    crc_scratch.release();
    desc_scratch.release();
    recs_scratch.release();
    round_scratch.release();
    plan.d_round.release();
    plan.d_recs.release();
    status.release();
    unit_acc.release();
    warp_trace.release();
    work.release();
    tables.release();
    base_crc.release();
    map_words.release();
    cdesc.release();
    dtotals.release();
    shadow.release();
    dirty.release();
    ccrc.release();
    cidx.release();
    stage_first.release();
    stage_lo.release();
    h_dtab.release();
    plan.d_desc.release();
    h_status.release();
    h_recs.release();
    h_meta.release();
    meta_acc.release();
    for (auto& g : graphs) {
      cudaGraphExecDestroy(g.exec);
      cudaGraphDestroy(g.graph);
    }
    graphs.clear();
    events.destroy_all();
    if (compute) cudaStreamDestroy(compute);
    if (copy) cudaStreamDestroy(copy);
    if (prev >= 0) cudaSetDevice(prev);
    dev = -1;
  }
};

// ---- library-owned memory (buffers re-created by restore / migrate) ----------

// One allocation of re-created buffers: a *segment* of a restore, i.e. a run of
// consecutive manifest records laid out like their part of the payload (buffer b
// at base + off_b - lo). Freed when its last handle is released or rebound.
struct Arena {
  checl_allocator alloc;
  int device;
  void* stream;
  void* base = nullptr;
  uint64_t bytes = 0;
  uint64_t n_handles = 0;  // entries bound into it (under the context lock)
  ~Arena() {
    if (!base) return;
    if (alloc.free)
      alloc.free(base, device, stream, alloc.user);
    else {
      int prev = -1;
      cudaGetDevice(&prev);
      cudaSetDevice(device);
      cudaFree(base);
      if (prev >= 0) cudaSetDevice(prev);
    }
  }
};

struct LayoutCache;

// The bindings of one commit (restore / migrate): record i lives in segment seg[i] at
// offset rel[i] (seg = ~0: a zero-size buffer), and each segment's arena (owned here)
// and address are kept once. The entries it bound point at their record (Entry::bind, idx)
// instead of holding an address, so a commit that rebinds the same handles to the
// same layout in new segments rewrites one pointer per segment (80 for C3's 10 000
// buffers), not one map node per handle.
struct Binding {
  std::vector<uint32_t> seg;
  std::vector<uint64_t> rel;
  std::vector<uint8_t*> seg_base;
  // the segments themselves: the binding owns them (a segment whose last handle is
  // released is moved out and freed; null from then on)
  std::vector<std::shared_ptr<Arena>> seg_arena;
  uint64_t refs = 0;  // entries bound through it
};

struct Entry {
  int device;
  uint8_t* ptr;  // user-registered buffers (bind == nullptr)
  uint64_t bytes;
  uint32_t flags;
  bool owned;
  Binding* bind;  // owned (re-created) buffers: their slot, bind->ptr[idx] / bind->arena[idx]
  uint32_t idx;
};

uint8_t* entry_ptr(const Entry& e) {
  if (!e.bind) return e.ptr;
  const uint32_t k = e.bind->seg[e.idx];
  return k == ~0u ? nullptr : e.bind->seg_base[k] + e.bind->rel[e.idx];
}


// Phase-time events for checl_timing.
struct KernelTimer {  // the event pair around every timed launch of a call
  std::vector<std::pair<cudaEvent_t, cudaEvent_t>> spans;
};

}  // namespace

// ---- opaque types -------------------------------------------------------------

struct checl_image {
  int location = CHECL_IMAGE_HOST;
  // device payload / CRC table from this allocator when set (the migration image
  // comes from the context's allocator, so freeing it returns the memory to the
  // caller's pool); cudaMalloc / cudaFree otherwise
  checl_allocator dalloc{nullptr, nullptr, nullptr};
  void* dstream = nullptr;
  int device = -1;  // device image: where payload and CRC table live
  bool owned = true;
  bool pinned = false;
  const uint8_t* host = nullptr;  // host: full image; device: mirror of [0, payload_off)
  uint8_t* host_mut = nullptr;    // same pointer when library-owned
  size_t host_cap = 0;
  uint64_t image_bytes = 0, payload_off = 0;
  uint8_t* d_payload = nullptr;
  size_t d_payload_cap = 0;
  uint32_t* d_crc = nullptr;
  size_t d_crc_cap = 0;
  // device address of host_mut (mapped pinned memory), cached: nullptr = not known yet
  const uint8_t* mapped_for = nullptr;
  uint8_t* mapped_dev = nullptr;
  // host_mut[128, crc_off) holds the manifest of plan generation meta_gen
  bool meta_valid = false;
  uint64_t meta_gen = 0;

  void* dev_alloc(size_t n) {  // on the current device (= `device`); nullptr on failure
    if (dalloc.alloc) return dalloc.alloc(n, device, dstream, dalloc.user);
    void* p = nullptr;
    if (cudaMalloc(&p, n) != cudaSuccess) {
      cudaGetLastError();
      return nullptr;
    }
    return p;
  }
  void dev_free(void* p) {
    if (!p) return;
    if (dalloc.free)
      dalloc.free(p, device, dstream, dalloc.user);
    else
      cudaFree(p);
  }
  void free_device() {
    if (device >= 0 && (d_payload || d_crc)) {
      int prev = -1;
      cudaGetDevice(&prev);
      cudaSetDevice(device);
      dev_free(d_payload);
      dev_free(d_crc);
      if (prev >= 0) cudaSetDevice(prev);
    }
    d_payload = nullptr;
    d_crc = nullptr;
    d_payload_cap = d_crc_cap = 0;
  }
  void free_host() {
    if (owned && host_mut) {
      if (pinned) {
        pinned_pool().give(host_mut, host_cap);
      } else {
        std::free(host_mut);
      }
    }
    host = host_mut = nullptr;
    host_cap = 0;
    meta_valid = false;
  }
  void ensure_host(size_t n, bool want_pinned) {
    if (owned && host_mut && host_cap >= n && pinned == want_pinned) return;
    free_host();
    owned = true;
    void* p = nullptr;
    size_t cap = std::max<size_t>(n, 1);
    if (want_pinned) {
      cap = pinned_class(cap);
      p = pinned_pool().take(cap, &cap);
      if (!p) p = pin_alloc(cap);
      if (!p) ck(cudaErrorMemoryAllocation);
    } else {
      p = std::malloc(std::max<size_t>(n, 1));
      if (!p) throw std::bad_alloc();
    }
    host = host_mut = static_cast<uint8_t*>(p);
    host_cap = cap;
    pinned = want_pinned;
    meta_valid = false;
  }
};

struct checl_ctx {
  mutable std::mutex mu;
  checl_allocator alloc{nullptr, nullptr, nullptr};
  std::map<uint64_t, Entry> entries;                  // ascending handle = database order (L19)
  uint64_t n_live[kMaxDevices] = {};                  // entries per device
  // live address ranges of user registrations per device (overlap checks; the
  // library's own segments are checked through the bindings that own them)
  struct Range {
    uint64_t bytes, handle;
  };
  std::map<uintptr_t, Range> by_addr[kMaxDevices];
  uint64_t version[kMaxDevices] = {};
  uint64_t next_id = 1;
  std::atomic<bool> busy{false};
  // delayed checkpointing mode (L16 §III-C): set by checl_request_checkpoint (or
  // the installed signal handler), consumed by checl_sync_point
  std::atomic<uint32_t> requested{0};
  DevState* devs[kMaxDevices] = {};
  size_t slot_bytes = kDefaultSlotBytes;
  uint32_t n_slots = 2;
  // timing of the last call; its CUDA-event spans are read lazily (PendingTiming)
  mutable checl_timing last{};
  // The last call's kernel / copy spans, not read yet: cudaEventElapsedTime costs
  // ~3 us of host time per call on this pool (profiles/r01o/launch_cost_events.txt),
  // so a call leaves its spans here and the next call reads them while its own kernel
  // runs; checl_last_timing / checl_stats_get read them on demand.
  struct PendingTiming {
    bool on = false;
    int kind = 0;
    const EventPool* pool = nullptr;
    int half = 0;
    std::vector<std::pair<cudaEvent_t, cudaEvent_t>> spans;
    cudaEvent_t c_begin = nullptr, c_end = nullptr;
  };
  mutable PendingTiming pend;
  mutable checl_stats stats[CHECL_STATS_KINDS] = {};
  mutable std::mutex tmu;
  // the segments the last commit on each device released (bounded by
  // CHECL_SPARE_BYTES, default 8 GiB), kept for the next restore of (nearly) the same
  // layout: a checkpoint/restore loop re-creates same-sized segments every time and
  // skips one allocator round trip per segment; checl_trim frees them
  std::vector<std::shared_ptr<Arena>> spares[kMaxDevices];
  // arenas whose last handle was released while a checkpoint / restore / migrate ran
  // (its plan may still read them): freed when that call ends (BusyGuard)
  std::vector<std::shared_ptr<Arena>> deferred;
  // per device: the layout of its last full-image restore (restore fast path)
  std::unique_ptr<LayoutCache> layout[kMaxDevices];
  // the bindings of the last commit: its entries in manifest order (map nodes are
  // stable) and the segments they point into; a commit of the same layout onto the
  // same device with the registry unchanged since (version) rebinds them in place
  struct BindCache {
    int device = -1;
    uint64_t gen = 0, version = 0;
    Binding* binding = nullptr;  // bound exactly the entries of that commit (nullptr: none)
  } bind;
  std::unordered_set<Binding*> bindings;  // with refs > 0

  DevState& dev(int d) {
    if (!devs[d]) {
      auto* s = new DevState();
      try {
        s->init(d);
      } catch (...) {
        s->destroy();
        delete s;
        throw;
      }
      devs[d] = s;
    }
    return *devs[d];
  }
};

namespace {

// Frees arenas once their devices are idle (no kernel of any stream can still read
// or write them).
void free_arenas(std::vector<std::shared_ptr<Arena>>& v) {
  bool synced[kMaxDevices] = {};
  int prev = -1;
  for (auto& a : v) {
    if (a && a.use_count() == 1 && a->base && !synced[a->device]) {  // one wait per device
      if (prev < 0) cudaGetDevice(&prev);
      cudaSetDevice(a->device);
      cudaDeviceSynchronize();
      synced[a->device] = true;
    }
  }
  if (prev >= 0) cudaSetDevice(prev);
  v.clear();  // (the arenas free their allocations)
}

struct BusyGuard {
  checl_ctx* ctx;
  bool ok;
  explicit BusyGuard(checl_ctx* c) : ctx(c) {
    bool expected = false;
    ok = ctx->busy.compare_exchange_strong(expected, true);
  }
  ~BusyGuard() {
    if (!ok) return;
    std::vector<std::shared_ptr<Arena>> d;
    {
      // (under the lock checl_release decides between freeing and deferring)
      std::lock_guard<std::mutex> lk(ctx->mu);
      ctx->busy.store(false);
      d.swap(ctx->deferred);
    }
    free_arenas(d);
  }
};

template <typename F>
checl_status guarded(F&& f) {
  try {
    return f();
  } catch (const CudaFail&) {
    return CHECL_ERR_CUDA;
  } catch (const std::bad_alloc&) {
    return CHECL_ERR_OUT_OF_HOST_MEMORY;
  } catch (...) {
    return CHECL_ERR_INVALID_VALUE;
  }
}

// -- layout (FORMAT.md), independent of the oracle ------------------------------

struct Layout {
  uint64_t n_chunks = 0, payload_bytes = 0, crc_off = 0, payload_off = 0, image_bytes = 0;
};

// Fills off / first_chunk of each record (ascending handle) and the region offsets.
Layout layout_records(std::vector<BufRec>& bufs) {
  Layout L;
  uint64_t end = 0;
  for (size_t b = 0; b < bufs.size(); ++b) {
    bufs[b].off = b == 0 ? 0 : align_up(end, kBufferAlign);
    bufs[b].first_chunk = L.n_chunks;
    end = bufs[b].off + bufs[b].size;
    L.n_chunks += chunks_of(bufs[b].size);
  }
  L.payload_bytes = bufs.empty() ? 0 : end;
  L.crc_off = kHeaderBytes + (uint64_t)kRecordBytes * bufs.size();
  L.payload_off = align_up(L.crc_off + 4 * L.n_chunks, kPayloadAlign);
  L.image_bytes = L.payload_off + L.payload_bytes;
  return L;
}

// Per-buffer records for the GPU chunk-list expansion (expand_plan_kernel);
// ptr(b) is the device address of record b (pack: source; restore: destination).
// Returns the total number of 4 KiB rounds (a chunk of len bytes has ceil(len/4096)).
template <typename PtrOf>
uint64_t build_records(const std::vector<BufRec>& bufs, PtrOf ptr_of, BufferRecord* out) {
  uint64_t rounds = 0;
  for (size_t b = 0; b < bufs.size(); ++b) {
    out[b] = BufferRecord{reinterpret_cast<uint64_t>(ptr_of(b)), bufs[b].size, bufs[b].off, bufs[b].first_chunk,
                          rounds, 0};
    const uint64_t nch = chunks_of(bufs[b].size);
    if (nch)
      rounds += (nch - 1) * (kChunkBytes / kRoundBytes) +
                (bufs[b].size - (nch - 1) * kChunkBytes + kRoundBytes - 1) / kRoundBytes;
  }
  return rounds;
}

// Stages = maximal runs of consecutive chunks whose image span (chunk bytes plus
// owned padding) fits in one staging slot; a stage always takes at least one
// chunk. Computed per buffer in O(#buffers + #stages): inside a buffer, chunk j
// (not the last) ends at off + (j+1)*64K, the last one at the next buffer's offset.
std::vector<Stage> build_stages(const std::vector<BufRec>& bufs, uint64_t payload_bytes, size_t slot) {
  std::vector<Stage> st;
  bool open = false;
  Stage cur{0, 0, 0, 0};
  for (size_t b = 0; b < bufs.size(); ++b) {
    const uint64_t nch = chunks_of(bufs[b].size);
    if (!nch) continue;
    const uint64_t off = bufs[b].off, first = bufs[b].first_chunk;
    const uint64_t end_last = b + 1 < bufs.size() ? bufs[b + 1].off : payload_bytes;
    uint64_t j = 0;
    while (j < nch) {
      if (!open) {
        cur = Stage{first + j, first + j, off + j * kChunkBytes, off + j * kChunkBytes};
        open = true;
      }
      if (end_last - cur.img_lo <= slot) {  // the rest of the buffer fits
        cur.c1 = first + nch;
        cur.img_hi = end_last;
        j = nch;
        continue;
      }
      // non-last chunks jj < fit end inside the slot: off + fit*64K <= img_lo + slot
      uint64_t fit = cur.img_lo + slot >= off ? (cur.img_lo + slot - off) / kChunkBytes : 0;
      fit = std::min(fit, nch - 1);
      if (fit > j) {
        cur.c1 = first + fit;
        cur.img_hi = off + fit * kChunkBytes;
        j = fit;
      } else if (cur.c1 == cur.c0) {  // empty stage: take one chunk regardless
        cur.c1 = first + j + 1;
        cur.img_hi = j + 1 < nch ? off + (j + 1) * kChunkBytes : end_last;
        ++j;
      }
      st.push_back(cur);
      open = false;
    }
  }
  if (open) st.push_back(cur);
  return st;
}

void write_header(uint8_t* h, const Layout& L, uint64_t n_buffers, int device, uint64_t epoch) {
  std::memset(h, 0, kHeaderBytes);
  std::memcpy(h, "CHECLIM1", 8);
  put_u32(h + 8, 1);
  put_u32(h + 12, kHeaderBytes);
  put_u32(h + 16, kChunkBytes);
  put_u32(h + 20, kBufferAlign);
  put_u64(h + 24, n_buffers);
  put_u64(h + 32, L.n_chunks);
  put_u64(h + 40, kHeaderBytes);
  put_u64(h + 48, L.crc_off);
  put_u64(h + 56, L.payload_off);
  put_u64(h + 64, L.payload_bytes);
  put_u64(h + 72, L.image_bytes);
  put_u32(h + 80, (uint32_t)device);
  put_u32(h + 84, 0);
  put_u64(h + 88, epoch);
}

void write_manifest(uint8_t* m, const std::vector<BufRec>& bufs, int device) {
  for (size_t b = 0; b < bufs.size(); ++b) {
    uint8_t* r = m + (size_t)kRecordBytes * b;
    put_u64(r, bufs[b].handle);
    put_u64(r + 8, bufs[b].size);
    put_u64(r + 16, bufs[b].off);
    put_u64(r + 24, bufs[b].first_chunk);
    put_u32(r + 32, bufs[b].flags);
    put_u32(r + 36, (uint32_t)device);
    put_u64(r + 40, 0);
  }
}

uint32_t meta_crc(const uint8_t* img, uint64_t payload_off) {
  uint32_t c = host_crc32c_update(0xFFFFFFFFu, img, 124);
  c = host_crc32c_update(c, img + kHeaderBytes, payload_off - kHeaderBytes);
  return ~c;
}

// -- validation (FORMAT.md "Validation order" step 1) -----------------------------

bool add_ok(uint64_t a, uint64_t b, uint64_t* out) {
  if (a > ~0ull - b) return false;
  *out = a + b;
  return true;
}

struct Parsed {
  int source_device = 0;
  Layout L;  // L.payload_bytes = the header field (the compacted payload of a delta)
  std::vector<BufRec> bufs;
  uint32_t flags = 0;          // 0 full, 1 incremental (FORMAT.md "Incremental images")
  uint64_t epoch = 0, full_payload = 0, map_off = 0, map_bytes = 0, n_present = 0;
  uint64_t base_epoch = 0;
  uint32_t base_table_crc = 0;
};

// Full-payload span [start, stop) of chunk j of buffer b: its bytes plus, for the
// buffer's last chunk, the padding it owns (FORMAT.md "Span of a chunk").
void chunk_span(const std::vector<BufRec>& bufs, size_t b, uint64_t j, uint64_t full_payload, uint64_t* start,
                uint64_t* stop) {
  *start = bufs[b].off + (uint64_t)kChunkBytes * j;
  if (j + 1 < chunks_of(bufs[b].size))
    *stop = *start + kChunkBytes;
  else
    *stop = b + 1 < bufs.size() ? bufs[b + 1].off : full_payload;
}

bool bit_set(const uint8_t* map, uint64_t k) { return (map[k >> 3] >> (k & 7)) & 1u; }

checl_status parse_image(const uint8_t* img, size_t len, bool meta_only, Parsed* out, bool check_meta_crc = true) {
  // meta_only: `len` covers [0, payload_off) only (device image mirror)
  // check_meta_crc = false: the caller checks the meta CRC itself (do_restore, while
  // its kernel runs); every structural check is made here
  if (!img || len < kHeaderBytes) return CHECL_ERR_BAD_IMAGE;
  if (std::memcmp(img, "CHECLIM1", 8) != 0) return CHECL_ERR_BAD_IMAGE;
  const uint32_t flags = get_u32(img + 84);
  if (get_u32(img + 8) != 1 || get_u32(img + 12) != kHeaderBytes || get_u32(img + 16) != kChunkBytes ||
      get_u32(img + 20) != kBufferAlign || get_u64(img + 40) != kHeaderBytes || flags > 1)
    return CHECL_ERR_BAD_IMAGE;
  if (flags == 0) {
    for (int i = 96; i < 124; ++i)
      if (img[i]) return CHECL_ERR_BAD_IMAGE;
  } else if (get_u32(img + 108) > 1 || get_u32(img + 120) != 0) {  // dirty_rule 0 (CRC) or 1 (bytes)
    return CHECL_ERR_BAD_IMAGE;
  }
  const uint64_t n = get_u64(img + 24), nch = get_u64(img + 32);
  Layout L;
  L.n_chunks = nch;
  L.crc_off = get_u64(img + 48);
  L.payload_off = get_u64(img + 56);
  L.payload_bytes = get_u64(img + 64);
  L.image_bytes = get_u64(img + 72);
  if (n > (~0ull - kHeaderBytes) / kRecordBytes || L.crc_off != kHeaderBytes + kRecordBytes * n)
    return CHECL_ERR_BAD_IMAGE;
  if (nch > (~0ull - L.crc_off - kPayloadAlign) / 5) return CHECL_ERR_BAD_IMAGE;
  const uint64_t map_bytes = flags ? (nch + 7) / 8 : 0;
  if (L.payload_off != align_up(L.crc_off + 4 * nch + map_bytes, kPayloadAlign)) return CHECL_ERR_BAD_IMAGE;
  uint64_t want;
  if (!add_ok(L.payload_off, L.payload_bytes, &want) || want != L.image_bytes) return CHECL_ERR_BAD_IMAGE;
  if ((uint64_t)len < (meta_only ? L.payload_off : L.image_bytes)) return CHECL_ERR_BAD_IMAGE;
  if (check_meta_crc && get_u32(img + 124) != meta_crc(img, L.payload_off)) return CHECL_ERR_BAD_IMAGE;
  for (uint64_t i = L.crc_off + 4 * nch + map_bytes; i < L.payload_off; ++i)
    if (img[i]) return CHECL_ERR_BAD_IMAGE;
  const int device = (int32_t)get_u32(img + 80);
  std::vector<BufRec> bufs(n);
  uint64_t off = 0, end = 0, chunk = 0, prev = 0;
  for (uint64_t b = 0; b < n; ++b) {
    const uint8_t* r = img + kHeaderBytes + kRecordBytes * b;
    const uint64_t h = get_u64(r), size = get_u64(r + 8);
    if (h == 0 || (b > 0 && h <= prev)) return CHECL_ERR_BAD_IMAGE;
    if (b > 0) {
      if (!add_ok(end, kBufferAlign - 1, &off)) return CHECL_ERR_BAD_IMAGE;
      off = off / kBufferAlign * kBufferAlign;
    }
    if (get_u64(r + 16) != off || get_u64(r + 24) != chunk) return CHECL_ERR_BAD_IMAGE;
    if ((int32_t)get_u32(r + 36) != device || get_u64(r + 40) != 0) return CHECL_ERR_BAD_IMAGE;
    if (!add_ok(off, size, &end)) return CHECL_ERR_BAD_IMAGE;
    chunk += chunks_of(size);
    bufs[b] = BufRec{h, size, off, get_u64(r + 24), get_u32(r + 32), nullptr};
    prev = h;
  }
  const uint64_t full_payload = n ? end : 0;
  if (chunk != nch || (flags == 0 && L.payload_bytes != full_payload)) return CHECL_ERR_BAD_IMAGE;
  // the kernels address chunk offsets as u32 multiples of 256 (1 TiB payload)
  if (full_payload > (1ull << 40)) return CHECL_ERR_BAD_IMAGE;
  if (flags == 1) {  // present bitmap: unused bits zero, popcount, spans
    const uint8_t* map = img + L.crc_off + 4 * nch;
    for (uint64_t k = nch; k < map_bytes * 8; ++k)
      if (bit_set(map, k)) return CHECL_ERR_BAD_IMAGE;
    uint64_t np = 0, sum = 0;
    for (size_t b = 0; b < bufs.size(); ++b) {
      const uint64_t nb = chunks_of(bufs[b].size);
      for (uint64_t j = 0; j < nb; ++j) {
        if (!bit_set(map, bufs[b].first_chunk + j)) continue;
        uint64_t a, z;
        chunk_span(bufs, b, j, full_payload, &a, &z);
        ++np;
        sum += z - a;
      }
    }
    if (np != get_u64(img + 112) || sum != L.payload_bytes) return CHECL_ERR_BAD_IMAGE;
    out->n_present = np;
    out->base_epoch = get_u64(img + 96);
    out->base_table_crc = get_u32(img + 104);
  }
  out->flags = flags;
  out->epoch = get_u64(img + 88);
  out->full_payload = full_payload;
  out->map_off = L.crc_off + 4 * nch;
  out->map_bytes = map_bytes;
  out->source_device = device;
  out->L = L;
  out->bufs = std::move(bufs);
  return CHECL_SUCCESS;
}

// -- checkpoint -------------------------------------------------------------------

std::atomic<uint64_t> g_meta_gen{0};  // process-wide: a generation names one manifest

void plan_meta_state(Plan& P) {
  P.meta_state0 = host_crc32c_update(0xFFFFFFFFu, P.meta.data(), 124);
  P.meta_state0 = host_crc32c_update(P.meta_state0, P.meta.data() + kHeaderBytes, P.crc_off - kHeaderBytes);
  P.epoch_shift = gf_x8n(P.crc_off - 100);  // bytes after the epoch's last one: header 96..123 + manifest
  P.meta_gen = ++g_meta_gen;
}

// Builds (or reuses) the plan of `device` under the context lock.
Plan& get_plan(checl_ctx* ctx, DevState& ds, int device) {
  std::lock_guard<std::mutex> lk(ctx->mu);
  Plan& P = ds.plan;
  if (P.version == ctx->version[device] && P.slot_bytes == ctx->slot_bytes) return P;
  P.bufs.clear();
  for (auto& kv : ctx->entries)
    if (kv.second.device == device)
      P.bufs.push_back(BufRec{kv.first, kv.second.bytes, 0, 0, kv.second.flags, entry_ptr(kv.second)});
  Layout L = layout_records(P.bufs);
  if (L.payload_bytes > (1ull << 40)) throw std::bad_alloc();
  P.n_chunks = L.n_chunks;
  P.payload_bytes = L.payload_bytes;
  P.crc_off = L.crc_off;
  P.payload_off = L.payload_off;
  P.image_bytes = L.image_bytes;
  P.recs.resize(P.bufs.size());
  const uint64_t rounds = build_records(P.bufs, [&](size_t b) { return P.bufs[b].ptr; }, P.recs.data());
  if (rounds >= (1ull << 32)) throw std::bad_alloc();  // round_base is u32 (16 TiB of payload)
  P.stages = build_stages(P.bufs, L.payload_bytes, ctx->slot_bytes);
  P.meta.assign(L.crc_off, 0);
  write_header(P.meta.data(), L, P.bufs.size(), device, 0);
  write_manifest(P.meta.data() + kHeaderBytes, P.bufs, device);
  plan_meta_state(P);
  P.d_desc.ensure(std::max<uint64_t>(L.n_chunks, 1));
  P.d_round.ensure(L.n_chunks + 1);
  P.d_recs.ensure(std::max<size_t>(P.recs.size(), 1));
  if (L.n_chunks) {  // chunk list expanded on the GPU from one record per buffer
    ck(cudaMemcpyAsync(P.d_recs.p, P.recs.data(), P.recs.size() * sizeof(BufferRecord), cudaMemcpyHostToDevice,
                       ds.compute));
    ++ds.aux_launches;
    ck(launch_expand(P.d_recs.p, (uint32_t)P.recs.size(), L.payload_bytes, L.n_chunks, P.d_desc.p, P.d_round.p,
                     rounds, nullptr, ds.n_sms, ds.compute));
    // no sync: a pageable-source cudaMemcpyAsync returns once P.recs has been staged
  }
  P.version = ctx->version[device];
  P.slot_bytes = ctx->slot_bytes;
  P.layout_gen = 0;
  P.list_bases.clear();
  return P;
}

LaunchParams base_params(DevState& ds) {
  LaunchParams p{};
  p.inv_z = ds.inv_z.p;
  p.status = ds.status.p;
  p.tables = ds.tables.p;
  return p;
}

// Drain copy of one stage into the pinned image. Stage spans start at 256-B aligned
// image offsets (odd buffer sizes), so consecutive copies start at drifting offsets
// within a 4 KiB host page; such copies measured 2.5-4 % slower than the same bytes
// split into a head up to the next 4 KiB boundary, a page-aligned middle and a tail
// (tools/microbench/pinned_d2h.cu; profiles/r01m/pinned_d2h5.txt).
void d2h_page_aligned(uint8_t* dst, const uint8_t* src, uint64_t n, cudaStream_t s) {
  const uintptr_t d0 = reinterpret_cast<uintptr_t>(dst), d1 = d0 + n;
  const uintptr_t a0 = (d0 + 4095) & ~static_cast<uintptr_t>(4095), a1 = d1 & ~static_cast<uintptr_t>(4095);
#ifdef CHECL_EXPERIMENTS
  static const bool split = [] {  // CHECL_D2H_SPLIT=0: one copy per stage (A/B, experiments build)
    const char* e = std::getenv("CHECL_D2H_SPLIT");
    return !e || std::atoi(e) != 0;
  }();
#else
  constexpr bool split = true;
#endif
  if (!split || n < 4 * 4096 || (a0 == d0 && a1 == d1)) {
    ck(cudaMemcpyAsync(dst, src, n, cudaMemcpyDeviceToHost, s));
    return;
  }
  if (a0 > d0) ck(cudaMemcpyAsync(dst, src, a0 - d0, cudaMemcpyDeviceToHost, s));
  ck(cudaMemcpyAsync(dst + (a0 - d0), src + (a0 - d0), a1 - a0, cudaMemcpyDeviceToHost, s));
  if (d1 > a1) ck(cudaMemcpyAsync(dst + (a1 - d0), src + (a1 - d0), d1 - a1, cudaMemcpyDeviceToHost, s));
}

void gck(const char* what, cudaError_t e) {
  if (e != cudaSuccess && std::getenv("CHECL_TRACE")) std::fprintf(stderr, "[checl] %s: %s\n", what, cudaGetErrorName(e));
  ck(e);
}

void timed_launch(DevState& ds, KernelTimer& kt, int op, const LaunchParams& p0, cudaStream_t s) {
  LaunchParams p = p0;
#ifdef CHECL_EXPERIMENTS
  // experiments build only (libchecl_exp.so, tools/exp_run.py): CHECL_EXP_PACK_OP=2|4
  // replaces the pack launches by the CRC-only / copy-only op over the same plan (no
  // valid image); the product library does not read it
  static const int exp_pack_op = [] {
    const char* e = std::getenv("CHECL_EXP_PACK_OP");
    return e ? std::atoi(e) : -1;
  }();
  if (op == kOpPack && (exp_pack_op == kOpCrc || exp_pack_op == kOpCopy)) op = exp_pack_op;
#endif
  const uint64_t chunks = p.c1 - p.c0;
  // kernel 4 (bulk copies, column CRC; scheduled stretches of rounds) whenever the
  // chunk list has a round_base (kernel 3 for the ops kernel 4 does not implement);
  // otherwise a warp needs ~55 us per 64 KiB chunk in kernel 1, and when chunks are
  // fewer than half the warps the 4 KiB-unit sweep finishes sooner
  int kernel = ds.kernel;
  if (kernel == 4 && op != kOpPack && op != kOpVerify && op != kOpCrc && op != kOpCheck) kernel = 3;
  if (kernel >= 3 && !p.round_base) kernel = 0;
  const bool small = chunks * 2 <= (uint64_t)ds.n_sms * kWarpsPerCta;
  // (below 16 MiB of rounds the bulk-copy path measured no better, and with a dirty
  // L2 worse: C1 pack 16.5 -> 21 us)
  const bool tma_op = op == kOpPack || op == kOpVerify || op == kOpCrc || op == kOpCheck;
  // launches of at most 128 chunks (<= 8 MiB) take the 4 KiB-unit sweep even with a
  // round_base: no stretch search and a smaller table prologue; measured C1 (3 x 1 MiB,
  // 48 chunks, `profiles/r01r/c1_kernels.txt`) pack 15.9 -> 14.6 us, verify 15.7 -> 12.8 us
  if (!kernel)
    kernel = p.round_base ? (chunks <= 128 ? 2 : tma_op && chunks * (kChunkBytes / kRoundBytes) >= 4096 ? 4 : 3)
                          : (small ? 2 : 1);
  if (kernel < 3) p.round_base = nullptr;
  // balanced / TMA launches large enough to have a tail: static stretches for the
  // first part of the rounds, dynamic blocks for the rest (DESIGN.md §5 "Work split");
  // the experiments build reads CHECL_STATIC_PERMILLE / CHECL_DYN_BLOCK /
  // CHECL_DYN_MIN_ROUNDS overrides (sweeps, and the kernel-shape tests that force the
  // tail on at small sizes)
#ifdef CHECL_EXPERIMENTS
  static const int env_pm = [] {
    const char* e = std::getenv("CHECL_STATIC_PERMILLE");
    return e ? std::min(1000, std::max(0, std::atoi(e))) : -1;
  }();
  static const int env_blk = [] {
    const char* e = std::getenv("CHECL_DYN_BLOCK");
    return e ? std::max(1, std::atoi(e)) : -1;
  }();
  static const uint64_t dyn_min = [] {
    const char* e = std::getenv("CHECL_DYN_MIN_ROUNDS");
    return e ? (uint64_t)std::strtoull(e, nullptr, 10) : ~0ull;
  }();
#else
  constexpr int env_pm = -1, env_blk = -1;
  constexpr uint64_t dyn_min = ~0ull;
#endif
  // The split by rounds per warp (rpw; chunks x 16 bounds the rounds), from the sweeps
  // in profiles/r02/split_sweep (pack / verify us, static permille : block rounds):
  //   rpw < 16 (64 MiB: 11)   static only   (37 us; 500:4 40, 640:2 42)
  //   rpw < 64 (128-256 MiB)  500 : 4       (128 MiB 59 vs 64 static; 256 MiB 99 vs 112)
  //   rpw < 256 (C2: 76)      500 : 8       (C2 159.5 vs 166 with 750 : 8)
  //   otherwise (C3, 4 GiB)   750 : 8       (C3 1626; 850 : 8 1640, 950 : 8 1775;
  //                                          4 GiB 1295; 900 : 8 1380)
  // A larger static share loses to the SMs' position-dependent bulk-copy rate (the
  // slowest stretch sets the end), a smaller one or smaller blocks to the per-block
  // fetch, chunk search and split-chunk accounting.
  // (kernel 3 keeps static stretches only: measured slower with the dynamic tail)
  const uint64_t rounds_ub = chunks * (kChunkBytes / kRoundBytes);
  const uint64_t rpw = rounds_ub / ((uint64_t)ds.n_sms * kWarpsPerCta);
  const uint64_t min_rounds = dyn_min != ~0ull ? dyn_min : (uint64_t)ds.n_sms * kWarpsPerCta * 16;
  uint32_t static_pm = rpw < 256 ? 500u : 750u, dyn_block = rpw < 64 ? 4u : 8u;
  if (env_pm >= 0) static_pm = (uint32_t)env_pm;
  if (env_blk >= 0) dyn_block = (uint32_t)env_blk;
  if (kernel == 4 && static_pm < 1000 && rounds_ub >= min_rounds) {
    p.work = ds.work.p;
    p.static_permille = static_pm;
    p.dyn_block = dyn_block;
  }
  if (kernel >= 2) {
    if (ds.unit_acc.cap < chunks) {  // zeroed once; every sweep launch leaves it zero
      ds.unit_acc.ensure(chunks);
      ck(cudaMemsetAsync(ds.unit_acc.p, 0, ds.unit_acc.cap * 8, s));
    }
    p.unit_acc = ds.unit_acc.p;
  }
  // diagnostics (experiments build): CHECL_WARP_TRACE=1 prints the warps' start /
  // tables-ready / end times of every balanced or TMA launch (relative to the earliest
  // start, us)
#ifdef CHECL_EXPERIMENTS
  static const bool warp_tr = std::getenv("CHECL_WARP_TRACE") != nullptr;
#else
  constexpr bool warp_tr = false;
#endif
  const uint64_t n_tr = (uint64_t)ds.n_sms * kWarpsPerCta * 4;
  if (warp_tr && kernel >= 3) {
    ds.warp_trace.ensure(n_tr);
    ck(cudaMemsetAsync(ds.warp_trace.p, 0, n_tr * 8, s));
    p.warp_trace = ds.warp_trace.p;
  }
  static const bool host_tr = std::getenv("CHECL_TRACE") != nullptr;
  const double h0 = host_tr ? now_ms() : 0;
  cudaEvent_t a = ds.events.get(), b = ds.events.get();
  static const bool use_graph = [] {
    const char* e = std::getenv("CHECL_GRAPH");
    return !e || std::atoi(e) != 0;
  }();
  const void* fn = nullptr;
  unsigned ctas = 0, cluster = 1;
  size_t smem = 0;
  if (use_graph)
    ck(snapshot_launch_config(op, p, ds.n_sms, kernel, chunks * (kChunkBytes / kRoundBytes), &fn, &ctas, &smem,
                              &cluster));
  double h1 = 0, h2 = 0;
  LaunchGraph* g = nullptr;
  if (fn) {
    for (auto& x : ds.graphs)
      if (x.fn == fn && x.ctas == ctas) g = &x;
    // (a bounded cache: grids of every size from a stream of odd-sized launches fall
    // back to stream launches past 256 instantiated graphs)
    if (!g && ds.graphs.size() >= 256) fn = nullptr;
  }
  if (fn) {
    void* args[] = {&p};
    cudaKernelNodeParams kp = {};
    kp.func = const_cast<void*>(fn);
    kp.gridDim = dim3(ctas);
    kp.blockDim = dim3(kThreadsPerCta);
    kp.sharedMemBytes = (unsigned)smem;
    kp.kernelParams = args;
    if (!g) {
      LaunchGraph n;
      n.fn = fn;
      n.ctas = ctas;
      gck("cudaGraphCreate", cudaGraphCreate(&n.graph, 0));
      cudaGraph_t gr = n.graph;
      try {
        gck("cudaGraphAddEventRecordNode", cudaGraphAddEventRecordNode(&n.ev_a, gr, nullptr, 0, a));
        gck("cudaGraphAddKernelNode", cudaGraphAddKernelNode(&n.kern, gr, &n.ev_a, 1, &kp));
        if (cluster > 1) {  // kernel 4 as 2-CTA clusters (multicast table prologue)
          cudaKernelNodeAttrValue v = {};
          v.clusterDim.x = cluster;
          v.clusterDim.y = 1;
          v.clusterDim.z = 1;
          gck("cudaGraphKernelNodeSetAttribute",
              cudaGraphKernelNodeSetAttribute(n.kern, cudaLaunchAttributeClusterDimension, &v));
        }
        gck("cudaGraphAddEventRecordNode", cudaGraphAddEventRecordNode(&n.ev_b, gr, &n.kern, 1, b));
        gck("cudaGraphInstantiate", cudaGraphInstantiate(&n.exec, gr, 0));
      } catch (...) {
        cudaGraphDestroy(gr);
        throw;
      }
      ds.graphs.push_back(n);
      g = &ds.graphs.back();
    } else {
      gck("cudaGraphExecKernelNodeSetParams", cudaGraphExecKernelNodeSetParams(g->exec, g->kern, &kp));
      gck("cudaGraphExecEventRecordNodeSetEvent", cudaGraphExecEventRecordNodeSetEvent(g->exec, g->ev_a, a));
      gck("cudaGraphExecEventRecordNodeSetEvent", cudaGraphExecEventRecordNodeSetEvent(g->exec, g->ev_b, b));
    }
    h1 = host_tr ? now_ms() : 0;
    gck("cudaGraphLaunch", cudaGraphLaunch(g->exec, s));
    h2 = host_tr ? now_ms() : 0;
  } else {
    ck(cudaEventRecord(a, s));
    h1 = host_tr ? now_ms() : 0;
    ck(launch_snapshot(op, p, ds.n_sms, s, kernel, chunks * (kChunkBytes / kRoundBytes)));
    h2 = host_tr ? now_ms() : 0;
    ck(cudaEventRecord(b, s));
  }
  kt.spans.push_back({a, b});
  if (host_tr)
    std::fprintf(stderr, "[checl] timed_launch op %d kernel %d%s: record/update %.1f launch %.1f record %.1f us\n", op,
                 kernel, fn ? " (graph)" : "",
                 (h1 - h0) * 1e3, (h2 - h1) * 1e3, (now_ms() - h2) * 1e3);
#ifdef CHECL_EXPERIMENTS
  if (p.warp_trace) {
    std::vector<unsigned long long> h(n_tr);
    ck(cudaMemcpyAsync(h.data(), p.warp_trace, n_tr * 8, cudaMemcpyDeviceToHost, s));
    ck(cudaStreamSynchronize(s));
    std::vector<double> st, tb, en;
    unsigned long long t0 = ~0ull;
    for (uint64_t w = 0; w < n_tr / 4; ++w)
      if (h[4 * w]) t0 = std::min(t0, h[4 * w]);
    for (uint64_t w = 0; w < n_tr / 4; ++w) {
      if (!h[4 * w]) continue;
      st.push_back((h[4 * w] - t0) * 1e-3);
      if (h[4 * w + 1]) tb.push_back((h[4 * w + 1] - t0) * 1e-3);
      en.push_back((h[4 * w + 2] - t0) * 1e-3);
    }
    auto q = [](std::vector<double>& v, double f) {
      if (v.empty()) return 0.0;
      std::sort(v.begin(), v.end());
      return v[(size_t)(f * (v.size() - 1))];
    };
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    std::fprintf(stderr,
                 "[checl] op %d kernel %d warps %zu event %.1f us | start p50 %.1f max %.1f | tables p50 %.1f max %.1f | "
                 "end min %.1f p10 %.1f p50 %.1f p90 %.1f max %.1f us\n",
                 op, kernel, st.size(), ms * 1e3, q(st, 0.5), q(st, 1.0), q(tb, 0.5), q(tb, 1.0), q(en, 0.0), q(en, 0.1),
                 q(en, 0.5), q(en, 0.9), q(en, 1.0));
    const char* wt = std::getenv("CHECL_WARP_TRACE");
    if (wt && std::atoi(wt) == 3) {  // raw, one line per warp: cta warp slot3 start slot1 slot2 (us)
      for (uint64_t w = 0; w < n_tr / 4; ++w) {
        if (!h[4 * w]) continue;
        std::fprintf(stderr, "[checl] w %llu %llu %llu %llu %.2f %.2f %.2f\n", (unsigned long long)(w / kWarpsPerCta),
                     (unsigned long long)(w % kWarpsPerCta), h[4 * w + 3] & 0xFFFFFFFFull, h[4 * w + 3] >> 32,
                     (h[4 * w] - t0) * 1e-3, h[4 * w + 1] ? (h[4 * w + 1] - t0) * 1e-3 : -1.0, (h[4 * w + 2] - t0) * 1e-3);
      }
    }
    if (wt && std::atoi(wt) == 2) {  // raw end times, one line per CTA
      for (int c = 0; c < ds.n_sms; ++c) {
        std::string line = "[checl] cta " + std::to_string(c) + " sm " + std::to_string(h[4 * (uint64_t)c * kWarpsPerCta + 3]);
        for (int w = 0; w < kWarpsPerCta; ++w) {
          const uint64_t i = (uint64_t)c * kWarpsPerCta + w;
          char buf[32];
          std::snprintf(buf, sizeof buf, " %.1f", h[4 * i] ? (h[4 * i + 2] - t0) * 1e-3 : -1.0);
          line += buf;
        }
        std::fprintf(stderr, "%s\n", line.c_str());
      }
    }
  }
#endif
}

// a5, first half (while K1 runs): header and manifest into the image's host bytes (the
// manifest only when the image does not hold this plan's already), the zero pad after
// the CRC table, and the meta CRC register after header + manifest: the plan's
// epoch-0 register plus the epoch bytes' term, R(e, 0) * x^(8 (crc_off - 100)) (CRC
// linearity; DESIGN.md §5 "Finalize"). Nothing DMAs into [0, crc_off) or the pad.
uint32_t prefinalize(checl_image* img, const Plan& P, uint64_t epoch) {
  uint8_t* host = img->host_mut;
  if (!img->meta_valid || img->meta_gen != P.meta_gen) {
    std::memcpy(host + kHeaderBytes, P.meta.data() + kHeaderBytes, P.crc_off - kHeaderBytes);
    img->meta_valid = true;
    img->meta_gen = P.meta_gen;
  }
  std::memcpy(host, P.meta.data(), kHeaderBytes);
  put_u64(host + 88, epoch);
  std::memset(host + P.crc_off + 4 * P.n_chunks, 0, P.payload_off - P.crc_off - 4 * P.n_chunks);
  uint8_t e[8];
  put_u64(e, epoch);
  return P.meta_state0 ^ gf_mul(host_crc32c_update(0u, e, 8), P.epoch_shift);
}

// a5, second half (the CRC table has landed): the meta CRC over the table and the pad.
void finalize_meta(uint8_t* host, const Plan& P, uint32_t state) {
  put_u32(host + 124, ~host_crc32c_update(state, host + P.crc_off, P.payload_off - P.crc_off));
}

// -- deferred timing (checl_ctx::PendingTiming) -----------------------------------

// Reads the pending spans of the last call into ctx->last and its statistics slot.
void settle(const checl_ctx* ctx) {
  std::lock_guard<std::mutex> lk(ctx->tmu);
  auto& q = ctx->pend;
  if (!q.on) return;
  double k = 0;
  for (auto& sp : q.spans) {
    float ms = 0;
    if (cudaEventElapsedTime(&ms, sp.first, sp.second) == cudaSuccess) k += ms;
  }
  float c = 0;
  if (q.c_begin && cudaEventElapsedTime(&c, q.c_begin, q.c_end) != cudaSuccess) c = 0;
  cudaGetLastError();
  ctx->last.kernel_ms = k;
  ctx->last.copy_ms = c;
  ctx->stats[q.kind].kernel_ms += k;
  ctx->stats[q.kind].copy_ms += c;
  q.on = false;
}

// End of a call: its host-clock timing now, its event spans when next needed.
void defer_timing(checl_ctx* ctx, const DevState& ds, const checl_timing& tm, const KernelTimer& kt,
                  cudaEvent_t c_begin, cudaEvent_t c_end, int kind) {
  settle(ctx);  // (normally done already, during this call's kernel)
  std::lock_guard<std::mutex> lk(ctx->tmu);
  ctx->last = tm;
  ctx->last.kernel_ms = ctx->last.copy_ms = 0;
  checl_stats& st = ctx->stats[kind];
  st.n_calls++;
  st.total_ms += tm.total_ms;
  st.n_kernels += tm.n_kernels;
  auto& q = ctx->pend;
  q.on = true;
  q.kind = kind;
  q.pool = &ds.events;
  q.half = ds.events.active;
  q.spans = kt.spans;
  q.c_begin = c_begin;
  q.c_end = c_end;
}

// Start of a call on ds: switch its event pool to the other half, reading first the
// pending spans if they live in that half.
void begin_events(checl_ctx* ctx, DevState& ds) {
  bool need = false;
  {
    std::lock_guard<std::mutex> lk(ctx->tmu);
    need = ctx->pend.on && ctx->pend.pool == &ds.events && ctx->pend.half != ds.events.active;
  }
  if (need) settle(ctx);
  ds.events.reset();
}

// The caller's stream, if it belongs to `device` (the allocator hands out memory that
// is safe to use in the order of that stream); nullptr (the legacy default stream of
// the current device) otherwise.
void* stream_on(void* stream, int device) {
  if (!stream) return nullptr;
  int d = -1;
  if (cudaStreamGetDevice(static_cast<cudaStream_t>(stream), &d) != cudaSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  return d == device ? stream : nullptr;
}

// New allocations are written by the library's own streams, but the allocator (the
// PyTorch caching allocator) hands out blocks that are safe only in the order of the
// stream they were requested on: a block the application freed while its kernels
// were still pending could otherwise be overwritten by those kernels after K2. The
// library's streams wait for everything queued on that stream so far.
void order_after(DevState& ds, void* stream) {
  // nothing queued on it is still pending: nothing to order after (the common case:
  // no cross-stream wait in front of K2's graph launch)
  if (cudaStreamQuery(static_cast<cudaStream_t>(stream)) == cudaSuccess) return;
  cudaGetLastError();  // (cudaErrorNotReady)
  cudaEvent_t ev = ds.events.get();
  ck(cudaEventRecord(ev, static_cast<cudaStream_t>(stream)));
  ck(cudaStreamWaitEvent(ds.compute, ev, 0));
  ck(cudaStreamWaitEvent(ds.copy, ev, 0));
}

checl_status do_checkpoint(checl_ctx* ctx, int device, void* stream, uint64_t epoch, checl_image* img,
                           bool to_device) {
  (void)stream;
  const double t0 = now_ms();
  Trace tr("checkpoint");
  DeviceGuard g(device);
  DevState& ds = ctx->dev(device);
  const uint64_t aux0 = ds.aux_launches;
  begin_events(ctx, ds);
  KernelTimer kt;
  checl_timing tm{};
  tr("setup");

  // a1: synchronise the host and every queue of the device (L16 step 1)
  const double ts = now_ms();
  ck(cudaDeviceSynchronize());
  tm.sync_ms = now_ms() - ts;
  tr("sync");

  // a2: database walk -> manifest + chunk list (L19), cached per registry version
  const double tp = now_ms();
  Plan& P = get_plan(ctx, ds, device);
  tr("plan");
  LaunchParams lp = base_params(ds);
  lp.desc = P.d_desc.p;
  lp.round_base = P.d_round.p;
  tm.plan_ms = now_ms() - tp;

  cudaEvent_t c_begin = ds.events.get(), c_end = ds.events.get();
  uint32_t meta_state = 0;
  bool meta_on_gpu = false;
  if (to_device) {
    // device-resident image: payload and CRC table in HBM, meta mirrored on host
    if (img->location != CHECL_IMAGE_DEVICE || img->device != device) {
      img->free_device();
      img->free_host();
    }
    img->location = CHECL_IMAGE_DEVICE;
    img->device = device;
    if (img->d_payload_cap < P.payload_bytes + kSlotSlack) {
      img->dev_free(img->d_payload);
      img->d_payload = nullptr;
      img->d_payload_cap = 0;
      img->d_payload = static_cast<uint8_t*>(img->dev_alloc(P.payload_bytes + kSlotSlack));
      if (!img->d_payload) return CHECL_ERR_OUT_OF_DEVICE_MEMORY;
      img->d_payload_cap = P.payload_bytes + kSlotSlack;
    }
    if (img->d_crc_cap < std::max<uint64_t>(P.n_chunks, 1)) {
      img->dev_free(img->d_crc);
      img->d_crc = nullptr;
      img->d_crc_cap = 0;
      img->d_crc = static_cast<uint32_t*>(img->dev_alloc(std::max<uint64_t>(P.n_chunks, 1) * 4));
      if (!img->d_crc) return CHECL_ERR_OUT_OF_DEVICE_MEMORY;
      img->d_crc_cap = std::max<uint64_t>(P.n_chunks, 1);
    }
    if (img->dalloc.alloc) order_after(ds, img->dstream);
    img->ensure_host(P.payload_off, true);
    lp.c0 = 0;
    lp.c1 = P.n_chunks;
    lp.image = img->d_payload;
    lp.image_base = 0;
    lp.crc = img->d_crc;
    // the host mirror's CRC table is written by the kernel itself through the
    // mapped pinned mirror (no D2H copy after the kernel); plain copy if unmapped
    if (img->mapped_for != img->host_mut) {
      void* dp = nullptr;
      if (cudaHostGetDevicePointer(&dp, img->host_mut, 0) != cudaSuccess) {
        cudaGetLastError();
        dp = nullptr;
      }
      img->mapped_for = img->host_mut;
      img->mapped_dev = static_cast<uint8_t*>(dp);
    }
    void* mirror = img->mapped_dev ? img->mapped_dev + P.crc_off : nullptr;
    lp.crc_mirror = static_cast<uint32_t*>(mirror);
    tr("mirror");
    if (P.n_chunks) timed_launch(ds, kt, kOpPack, lp, ds.compute);
    tr("launch");
    meta_state = prefinalize(img, P, epoch);  // (while K1 runs)
    // a large CRC table (C3: 346 KB, C4: 4 MiB) is CRC'd on the GPU, where K1 left it in
    // L2, instead of by the host from pinned memory the GPU just wrote (~40 us for C3)
    if (ds.meta_dev && 4 * P.n_chunks >= kMetaKernelMinBytes) {
      ++ds.aux_launches;
      ck(launch_meta_crc(img->d_crc, 4 * P.n_chunks, P.payload_off - P.crc_off, meta_state, ds.meta_acc.p, ds.meta_dev,
                         ds.n_sms, ds.compute));
      meta_on_gpu = true;
    }
    if (P.n_chunks && !mirror) {
      ck(cudaEventRecord(c_begin, ds.compute));
      ck(cudaMemcpyAsync(img->host_mut + P.crc_off, img->d_crc, 4 * P.n_chunks, cudaMemcpyDeviceToHost, ds.compute));
      ck(cudaEventRecord(c_end, ds.compute));
    } else {
      c_begin = c_end = nullptr;  // nothing copied
    }
    tm.n_stages = 1;
    settle(ctx);  // the previous call's spans, read while K1 runs
    ck(cudaStreamSynchronize(ds.compute));
    tr("wait");
  } else {
    // a3 + a4: pack stage s into slot s % n_slots on the compute stream while the
    // copy engine drains the previous slot to the pinned image
    if (img->location != CHECL_IMAGE_HOST) {
      img->free_device();
      img->free_host();
      img->location = CHECL_IMAGE_HOST;
      img->device = -1;
    }
    img->ensure_host(P.image_bytes + kSlotSlack, true);
    ds.ensure_slots(ctx->slot_bytes, ctx->n_slots);
    ds.crc_scratch.ensure(std::max<uint64_t>(P.n_chunks, 1));
    lp.crc = ds.crc_scratch.p;
    // small images (<= 128 chunks, i.e. the sweep kernel with its register stores and
    // exact tails; payload <= CHECL_ZERO_COPY_MAX, default 8 MiB): K1 stores the payload and
    // the CRC table straight into the mapped pinned image over PCIe, so there is no
    // staging slot and no D2H copy; the drain span is K1's own
    static const uint64_t zc_max = [] {
      const char* e = std::getenv("CHECL_ZERO_COPY_MAX");
      return e ? (uint64_t)std::strtoull(e, nullptr, 10) : (8ull << 20);
    }();
    uint8_t* mapped = nullptr;
    // (not under a forced kernel 4: its bulk stores are for device memory)
    if (P.n_chunks && P.n_chunks <= 128 && P.stages.size() == 1 && P.payload_bytes <= zc_max && ds.kernel != 4) {
      void* dp = nullptr;
      if (cudaHostGetDevicePointer(&dp, img->host_mut, 0) == cudaSuccess)
        mapped = static_cast<uint8_t*>(dp);
      else
        cudaGetLastError();
    }
    if (mapped) {
      lp.c0 = 0;
      lp.c1 = P.n_chunks;
      lp.image = mapped + P.payload_off;
      lp.image_base = 0;
      lp.crc_mirror = reinterpret_cast<uint32_t*>(mapped + P.crc_off);
      ck(cudaEventRecord(c_begin, ds.compute));
      timed_launch(ds, kt, kOpPack, lp, ds.compute);
      ck(cudaEventRecord(c_end, ds.compute));
      tm.n_stages = 1;
      meta_state = prefinalize(img, P, epoch);
      settle(ctx);  // the previous call's spans, read while K1 runs
      ck(cudaStreamSynchronize(ds.compute));
    } else {
    std::vector<cudaEvent_t> packed(ds.n_slots), drained(ds.n_slots);
    for (uint32_t i = 0; i < ds.n_slots; ++i) {
      packed[i] = ds.events.get();
      drained[i] = ds.events.get();
    }
    // diagnostics (experiments build): CHECL_STAGE_TRACE=1 times every stage's D2H
#ifdef CHECL_EXPERIMENTS
    static const bool stage_tr = std::getenv("CHECL_STAGE_TRACE") != nullptr;
#else
    constexpr bool stage_tr = false;
#endif
    std::vector<std::pair<cudaEvent_t, cudaEvent_t>> d2h;
    ck(cudaEventRecord(c_begin, ds.copy));
    for (size_t s = 0; s < P.stages.size(); ++s) {
      const Stage& S = P.stages[s];
      const uint32_t k = (uint32_t)(s % ds.n_slots);
      if (s >= ds.n_slots) ck(cudaStreamWaitEvent(ds.compute, drained[k], 0));
      lp.c0 = S.c0;
      lp.c1 = S.c1;
      lp.image = ds.slot(k);
      lp.image_base = S.img_lo;
      timed_launch(ds, kt, kOpPack, lp, ds.compute);
      ck(cudaEventRecord(packed[k], ds.compute));
      ck(cudaStreamWaitEvent(ds.copy, packed[k], 0));
      if (stage_tr) {
        d2h.push_back({ds.events.get(), ds.events.get()});
        ck(cudaEventRecord(d2h.back().first, ds.copy));
      }
      d2h_page_aligned(img->host_mut + P.payload_off + S.img_lo, ds.slot(k), S.img_hi - S.img_lo, ds.copy);
      if (stage_tr) ck(cudaEventRecord(d2h.back().second, ds.copy));
      ck(cudaEventRecord(drained[k], ds.copy));
    }
    if (stage_tr && !d2h.empty()) {
      ck(cudaStreamSynchronize(ds.copy));
      double busy = 0, gap = 0, gap_max = 0, pk_to_start = 0;
      for (size_t s = 0; s < d2h.size(); ++s) {
        float a = 0, b = 0, k_end = 0;
        cudaEventElapsedTime(&a, c_begin, d2h[s].first);
        cudaEventElapsedTime(&b, c_begin, d2h[s].second);
        cudaEventElapsedTime(&k_end, c_begin, kt.spans[s].second);
        busy += b - a;
        pk_to_start += a - k_end;
        if (s) {
          float pb = 0;
          cudaEventElapsedTime(&pb, c_begin, d2h[s - 1].second);
          gap += a - pb;
          gap_max = std::max(gap_max, (double)(a - pb));
        }
      }
      float tot = 0;
      cudaEventElapsedTime(&tot, c_begin, d2h.back().second);
      std::fprintf(stderr,
                   "[checl] stages %zu: span %.3f ms, D2H busy %.3f ms (%.1f us each), gaps %.1f us total (max %.1f), "
                   "first D2H starts %.1f us after begin, D2H start - pack end mean %.1f us\n",
                   d2h.size(), tot, busy, busy / d2h.size() * 1e3, gap * 1e3, gap_max * 1e3,
                   [&] { float a = 0; cudaEventElapsedTime(&a, c_begin, d2h[0].first); return a * 1e3; }(),
                   pk_to_start / d2h.size() * 1e3);
    }
    if (P.n_chunks)
      ck(cudaMemcpyAsync(img->host_mut + P.crc_off, ds.crc_scratch.p, 4 * P.n_chunks, cudaMemcpyDeviceToHost, ds.copy));
    ck(cudaEventRecord(c_end, ds.copy));
    tm.n_stages = P.stages.size();
    meta_state = prefinalize(img, P, epoch);
    settle(ctx);  // the previous call's spans, read while the pipeline runs
    ck(cudaStreamSynchronize(ds.copy));
    }
  }
  // a5: the meta CRC over the CRC table, which has landed (header and manifest were
  // written while K1 ran)
  const double tf = now_ms();
  if (meta_on_gpu)
    put_u32(img->host_mut + 124, *reinterpret_cast<volatile uint32_t*>(ds.h_meta.p));
  else
    finalize_meta(img->host_mut, P, meta_state);
  tm.commit_ms = now_ms() - tf;
  tr("finalize");
  img->image_bytes = P.image_bytes;
  img->payload_off = P.payload_off;
  tm.n_kernels = kt.spans.size() + (ds.aux_launches - aux0);
  tm.total_ms = now_ms() - t0;
  defer_timing(ctx, ds, tm, kt, c_begin, c_end, CHECL_STATS_CHECKPOINT);
  return CHECL_SUCCESS;
}

// -- restore ----------------------------------------------------------------------

void set_report(checl_report* rep, const Parsed& P, uint64_t n_bad, uint64_t first_bad) {
  if (!rep) return;
  rep->n_buffers = P.bufs.size();
  rep->payload_bytes = P.full_payload;
  rep->n_chunks = P.L.n_chunks;
  rep->n_bad_chunks = n_bad;
  rep->first_bad_chunk = n_bad ? first_bad : ~0ull;
  rep->first_bad_handle = 0;
  if (n_bad) {
    for (auto& b : P.bufs)
      if (first_bad >= b.first_chunk && first_bad < b.first_chunk + chunks_of(b.size)) rep->first_bad_handle = b.handle;
  }
}

bool ensure_peer(int dev, int peer) {
  // CHECL_FORCE_NO_PEER=1 (tests): report no peer access, so the one-GPU test box runs
  // the migration fallback (cudaMemcpyPeerAsync into a local copy, then K2 on it)
  static const bool force_no_peer = std::getenv("CHECL_FORCE_NO_PEER") != nullptr;
  if (force_no_peer) return false;
  if (dev == peer) return true;
  int can = 0;
  if (cudaDeviceCanAccessPeer(&can, dev, peer) != cudaSuccess || !can) {
    cudaGetLastError();
    return false;
  }
  cudaError_t e = cudaDeviceEnablePeerAccess(peer, 0);  // current device = dev
  if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) {
    cudaGetLastError();
    return false;
  }
  cudaGetLastError();
  return true;
}

// Bytes of segments kept as spares per device (CHECL_SPARE_BYTES, default 8 GiB):
// larger re-creations amortise their allocator calls anyway, and a spare holds HBM idle
// (checl_trim releases it).
uint64_t spare_limit() {
  static const uint64_t v = [] {
    const char* e = std::getenv("CHECL_SPARE_BYTES");
    return e ? (uint64_t)std::strtoull(e, nullptr, 10) : (8ull << 30);
  }();
  return v;
}

// Target size of one allocation of re-created buffers (CHECL_SEGMENT_BYTES, default
// 64 MiB; 0 = one allocation per restore). Restore re-creates the objects of an image
// as a few segments instead of one object at a time (10 000 allocator calls for C3)
// or one block for all (which could not be returned until every handle is released).
uint64_t segment_bytes() {
  static const uint64_t v = [] {
    const char* e = std::getenv("CHECL_SEGMENT_BYTES");
    return e ? (uint64_t)std::strtoull(e, nullptr, 10) : (64ull << 20);
  }();
  return v;
}

// A segment: records [b0, b1), payload span [lo, hi) = from buffer b0's offset to the
// next segment's first offset (or payload_bytes), so the padding a chunk owns lies
// inside its segment.
struct Segment {
  size_t b0, b1;
  uint64_t lo, hi;
};

// The layout of the last full-image restore on a device: its header and manifest bytes
// (epoch and meta CRC zeroed), parse, segment plan and round count. A restore whose
// image header matches reuses it without parsing the manifest again; the manifest
// bytes are compared while K2 runs (a mismatch redoes the restore the long way).
// `gen` names the layout process-wide in chunk-list keys.
struct LayoutCache {
  uint64_t gen = 0;
  std::vector<uint8_t> meta;
  Parsed P;
  std::vector<Segment> segs;
  uint64_t rounds = 0;
};
std::atomic<uint64_t> g_layout_gen{0};

// The header fields a layout is made of: everything but the epoch (88) and meta CRC (124).
bool header_same(const uint8_t* h, const std::vector<uint8_t>& meta) {
  return meta.size() >= kHeaderBytes && std::memcmp(h, meta.data(), 88) == 0 &&
         std::memcmp(h + 96, meta.data() + 96, 28) == 0;
}

// Consecutive records in manifest order; a segment is closed before a record that
// would take it past segment_bytes(), so a buffer at least that large is alone.
std::vector<Segment> plan_segments(const std::vector<BufRec>& bufs, uint64_t payload_bytes) {
  std::vector<Segment> out;
  if (bufs.empty()) return out;
  const uint64_t T = segment_bytes();
  size_t b0 = 0;
  for (size_t b = 1; b < bufs.size(); ++b) {
    if (T && bufs[b].off + bufs[b].size - bufs[b0].off > T) {
      out.push_back(Segment{b0, b, bufs[b0].off, bufs[b].off});
      b0 = b;
    }
  }
  out.push_back(Segment{b0, bufs.size(), bufs[b0].off, payload_bytes});
  return out;
}

// The re-created buffers of one restore (r2).
struct RestoreAlloc {
  std::vector<Segment> segs;
  std::vector<std::shared_ptr<Arena>> arenas;  // one per segment (base nullptr when empty)
  std::vector<uint32_t> seg_of;                // per record
  // device address of record b (nullptr for a zero-size buffer)
  uint8_t* buf(const std::vector<BufRec>& bufs, size_t b) const {
    if (!bufs[b].size) return nullptr;
    const uint32_t k = seg_of[b];
    return static_cast<uint8_t*>(arenas[k]->base) + (bufs[b].off - segs[k].lo);
  }
  // device address of full-payload offset o (inside some segment's span)
  uint8_t* at(uint64_t o) const {
    size_t lo = 0, hi = segs.size();
    while (hi - lo > 1) {
      const size_t mid = (lo + hi) / 2;
      (segs[mid].lo <= o ? lo : hi) = mid;
    }
    return static_cast<uint8_t*>(arenas[lo]->base) + (o - segs[lo].lo);
  }
};

std::shared_ptr<Arena> alloc_arena(checl_ctx* ctx, int device, void* stream, uint64_t bytes) {
  auto arena = std::make_shared<Arena>();
  arena->alloc = ctx->alloc;
  arena->device = device;
  arena->stream = stream;
  arena->bytes = bytes;
  if (bytes) {
    if (ctx->alloc.alloc)
      arena->base = ctx->alloc.alloc(bytes, device, stream, ctx->alloc.user);
    else if (cudaMalloc(&arena->base, bytes) != cudaSuccess) {
      cudaGetLastError();
      arena->base = nullptr;
    }
    if (!arena->base) return nullptr;
  }
  return arena;
}

// r2: the segments of `bufs` on `device`, each from the spares the last commit on
// this device released (best fit, at most 1/8 larger) or through the context's
// allocator. false when the allocator fails (whatever was taken is freed).
bool new_alloc(checl_ctx* ctx, int device, void* stream, const std::vector<BufRec>& bufs, uint64_t payload_bytes,
               RestoreAlloc* out, const std::vector<Segment>* segs = nullptr) {
  out->segs = segs ? *segs : plan_segments(bufs, payload_bytes);
  out->arenas.assign(out->segs.size(), nullptr);
  out->seg_of.assign(bufs.size(), ~0u);
  std::vector<size_t> need;  // segments the spares did not cover
  {
    std::lock_guard<std::mutex> lk(ctx->mu);
    auto& sp = ctx->spares[device];
    // the spares of the previous restore of the same layout are in segment order:
    // taken in place when every size matches exactly (a checkpoint/restore loop)
    bool in_order = sp.size() == out->segs.size();
    for (size_t k = 0; in_order && k < sp.size(); ++k) in_order = sp[k]->bytes == out->segs[k].hi - out->segs[k].lo;
    if (in_order) {
      for (size_t k = 0; k < sp.size(); ++k) out->arenas[k] = std::move(sp[k]);
      sp.clear();
    }
    for (size_t k = 0; !in_order && k < out->segs.size(); ++k) {
      const uint64_t n = out->segs[k].hi - out->segs[k].lo;
      size_t best = sp.size();
      for (size_t i = 0; n && i < sp.size(); ++i)
        if (sp[i] && sp[i]->bytes >= n && sp[i]->bytes - n <= n / 8 &&
            (best == sp.size() || sp[i]->bytes < sp[best]->bytes))
          best = i;
      if (best != sp.size()) {
        out->arenas[k] = std::move(sp[best]);
        sp.erase(sp.begin() + (long)best);
      } else {
        need.push_back(k);
      }
    }
  }
  for (size_t k : need) {
    out->arenas[k] = alloc_arena(ctx, device, stream, out->segs[k].hi - out->segs[k].lo);
    if (!out->arenas[k]) {
      out->arenas.clear();
      return false;
    }
  }
  for (size_t k = 0; k < out->segs.size(); ++k)
    for (size_t b = out->segs[k].b0; b < out->segs[k].b1; ++b) out->seg_of[b] = (uint32_t)k;
  return true;
}

std::vector<void*> bases_of(const RestoreAlloc& A) {
  std::vector<void*> v(A.arenas.size());
  for (size_t k = 0; k < v.size(); ++k) v[k] = A.arenas[k]->base;
  return v;
}

// Swaps every handle of the image to its new buffer (L15); frees library-owned
// buffers previously bound to those handles (after their devices are idle). `gen` is
// the image's layout (LayoutCache::gen, 0 = none).
// An entry leaves its binding (released or rebound); the binding goes with its last
// entry. Under the context lock.
void unbind(checl_ctx* ctx, Entry& e);

// An owned entry gives up its buffer: its segment loses a handle, and a segment left
// without handles moves to `dropped` (freed by the caller outside the lock). Under the
// context lock.
void release_slot(checl_ctx* ctx, Entry& e, std::vector<std::shared_ptr<Arena>>& dropped) {
  if (e.bind) {
    const uint32_t k = e.bind->seg[e.idx];
    if (k != ~0u) {
      std::shared_ptr<Arena>& slot = e.bind->seg_arena[k];
      if (slot && --slot->n_handles == 0) dropped.push_back(std::move(slot));
    }
  }
  unbind(ctx, e);
}

void unbind(checl_ctx* ctx, Entry& e) {
  Binding* b = e.bind;
  if (!b) return;
  e.bind = nullptr;
  if (--b->refs == 0) {
    if (ctx->bind.binding == b) ctx->bind.binding = nullptr;
    ctx->bindings.erase(b);
    delete b;
  }
}

void commit(checl_ctx* ctx, const Parsed& P, int device, RestoreAlloc& A, uint64_t gen) {
  std::vector<std::shared_ptr<Arena>> dropped;  // segments that lost their last handle
  auto& bc = ctx->bind;
  Trace tr("commit");
  bool fast_bind = false;
  {
    std::lock_guard<std::mutex> lk(ctx->mu);
    const size_t n = P.bufs.size();
    for (auto& a : A.arenas) a->n_handles = 0;  // (a reused spare may carry its old count)
    Binding* B = bc.binding;
    const size_t nseg = A.arenas.size();
    if (gen && B && bc.gen == gen && bc.device == device && bc.version == ctx->version[device] && B->refs == n &&
        B->seg.size() == n && B->seg_base.size() == nseg) {
      // The same layout onto the same device, registry untouched since the last commit:
      // these handles are exactly that commit's entries, bound through B to its
      // segments and to nothing else, in the same segment plan. B takes the new
      // segments (each with its predecessor's handle count); the old ones lose all
      // their handles.
      fast_bind = true;
      for (size_t k = 0; k < nseg; ++k) {
        std::shared_ptr<Arena>& slot = B->seg_arena[k];
        A.arenas[k]->n_handles = slot ? slot->n_handles : 0;
        if (slot) dropped.push_back(std::move(slot));
        slot = A.arenas[k];
        B->seg_base[k] = static_cast<uint8_t*>(slot->base) - A.segs[k].lo;
      }
    } else {
      B = new Binding();
      B->seg.assign(n, ~0u);
      B->rel.assign(n, 0);
      B->seg_base.resize(nseg);
      B->seg_arena = A.arenas;
      for (size_t k = 0; k < nseg; ++k)
        B->seg_base[k] = static_cast<uint8_t*>(A.arenas[k]->base) - A.segs[k].lo;
      ctx->bindings.insert(B);
      uint64_t max_h = 0;
      // P.bufs ascend by handle, like the map: walk both in order (O(n), sequential)
      // instead of one O(log n) search per handle (C3: 10 000 handles)
      auto it = P.bufs.empty() ? ctx->entries.end() : ctx->entries.lower_bound(P.bufs.front().handle);
      for (size_t bi = 0; bi < n; ++bi) {
        const BufRec& b = P.bufs[bi];
        while (it != ctx->entries.end() && it->first < b.handle) ++it;
        const bool fresh = it == ctx->entries.end() || it->first != b.handle;
        if (fresh) it = ctx->entries.emplace_hint(it, b.handle, Entry{});
        Entry& e = it->second;
        if (!fresh) {  // rebind an existing handle in place
          if (!e.owned && e.bytes) ctx->by_addr[e.device].erase(reinterpret_cast<uintptr_t>(e.ptr));
          ctx->version[e.device]++;
          ctx->n_live[e.device]--;
          release_slot(ctx, e, dropped);
        }
        ctx->n_live[device]++;
        e.device = device;
        e.ptr = nullptr;
        e.bytes = b.size;
        e.flags = b.flags;
        e.owned = true;
        e.bind = B;
        e.idx = (uint32_t)bi;
        if (b.size) {
          const uint32_t k = A.seg_of[bi];
          B->seg[bi] = k;
          B->rel[bi] = b.off;
          A.arenas[k]->n_handles++;
        }
        max_h = std::max(max_h, b.handle);
      }
      B->refs = n;
      if (!n) {
        ctx->bindings.erase(B);
        delete B;
        B = nullptr;
      }
      ctx->next_id = std::max(ctx->next_id, max_h + 1);
    }
    tr(fast_bind ? "rebind_in_place" : "rebind_walk");
    ctx->version[device]++;
    bc.device = device;
    bc.gen = gen;
    bc.version = ctx->version[device];
    bc.binding = B;
  }
  // segments whose last handle moved away are freed here, outside the lock, once their
  // device is idle (the restore synchronised `device` after K2; another device is
  // synchronised here); on this device they become the spares of the next restore
  // (the previous spares are freed)
  std::vector<std::shared_ptr<Arena>> keep, old;
  uint64_t kept = 0;
  for (auto& a : dropped) {
    if (a->device != device) continue;
    if (a.use_count() == 1 && a->base && kept + a->bytes <= spare_limit()) {
      kept += a->bytes;
      keep.push_back(std::move(a));
    }
  }
  if (!keep.empty()) {
    std::lock_guard<std::mutex> lk(ctx->mu);
    old.swap(ctx->spares[device]);
    ctx->spares[device] = std::move(keep);
  }
  tr("spares");
  free_arenas(old);
  free_arenas(dropped);
  tr("free");
}

// After a successful restore onto `device`, the chunk list it expanded for the new
// allocation (ds.desc_scratch / round_scratch) is exactly the plan the next
// checkpoint of `device` needs when the device's live buffers are the image's: it
// becomes that plan (buffers swapped, no re-expansion), so a checkpoint right
// after a restore or migration skips the plan rebuild.
void adopt_plan(checl_ctx* ctx, DevState& ds, int device, const Parsed& P, const RestoreAlloc& A, uint64_t gen) {
  std::lock_guard<std::mutex> lk(ctx->mu);
  if (ctx->n_live[device] != P.bufs.size() || !P.L.n_chunks) return;
  Plan& Q = ds.plan;
  // the plan's current chunk list moves to the scratch buffers, its key with it; the
  // restore's list (key: gen over A's segments) becomes the plan's
  auto swap_lists = [&] {
    std::swap(Q.d_desc.p, ds.desc_scratch.p);
    std::swap(Q.d_desc.cap, ds.desc_scratch.cap);
    std::swap(Q.d_round.p, ds.round_scratch.p);
    std::swap(Q.d_round.cap, ds.round_scratch.cap);
    ds.scratch_gen = Q.layout_gen;
    ds.scratch_bases.swap(Q.list_bases);
    Q.layout_gen = gen;
    Q.list_bases = bases_of(A);
  };
  // the same layout as the current plan (every restore of a checkpoint/restore loop):
  // only the buffer addresses change; stages, header and manifest stay. (The plan's
  // BufRec pointers are not used after the plan is built: its chunk list is.)
  bool same = Q.version != ~0ull && gen && Q.layout_gen == gen && Q.slot_bytes == ctx->slot_bytes;
  if (!same) {
    same = Q.version != ~0ull && Q.bufs.size() == P.bufs.size() && Q.n_chunks == P.L.n_chunks &&
           Q.payload_bytes == P.full_payload && Q.crc_off == P.L.crc_off && Q.slot_bytes == ctx->slot_bytes;
    for (size_t i = 0; same && i < Q.bufs.size(); ++i) {
      const BufRec &q = Q.bufs[i], &b = P.bufs[i];
      same = q.handle == b.handle && q.size == b.size && q.off == b.off && q.first_chunk == b.first_chunk &&
             q.flags == b.flags;
    }
  }
  if (same) {
    swap_lists();
    Q.version = ctx->version[device];
    return;
  }
  Q.bufs = P.bufs;
  for (size_t i = 0; i < Q.bufs.size(); ++i) Q.bufs[i].ptr = A.buf(Q.bufs, i);
  Q.n_chunks = P.L.n_chunks;
  Q.payload_bytes = P.full_payload;
  Q.crc_off = P.L.crc_off;
  Q.payload_off = align_up(P.L.crc_off + 4 * P.L.n_chunks, kPayloadAlign);
  Q.image_bytes = Q.payload_off + Q.payload_bytes;
  Q.recs.resize(Q.bufs.size());
  build_records(Q.bufs, [&](size_t b) { return Q.bufs[b].ptr; }, Q.recs.data());
  Q.stages = build_stages(Q.bufs, Q.payload_bytes, ctx->slot_bytes);
  Layout L;
  L.n_chunks = Q.n_chunks;
  L.payload_bytes = Q.payload_bytes;
  L.crc_off = Q.crc_off;
  L.payload_off = Q.payload_off;
  L.image_bytes = Q.image_bytes;
  Q.meta.assign(Q.crc_off, 0);
  write_header(Q.meta.data(), L, Q.bufs.size(), device, 0);
  write_manifest(Q.meta.data() + kHeaderBytes, Q.bufs, device);
  plan_meta_state(Q);
  swap_lists();
  Q.version = ctx->version[device];
  Q.slot_bytes = ctx->slot_bytes;
}

checl_status do_restore(checl_ctx* ctx, const checl_image* img, int device, void* stream, checl_report* rep,
                        bool in_migrate, bool long_way = false) {
  const double t0 = now_ms();
  Trace tr("restore");
  DeviceGuard g(device);
  DevState& ds = ctx->dev(device);
  const uint64_t aux0 = ds.aux_launches;
  begin_events(ctx, ds);
  KernelTimer kt;
  checl_timing tm{};
  if (rep) std::memset(rep, 0, sizeof(*rep)), rep->first_bad_chunk = ~0ull;

  // (the target is quiesced before anything is rebound — its old buffers may be
  // freed at commit — by the device-wide wait for K2 below; nothing before it touches
  // memory the application may still be using: tm.sync_ms stays 0)

  // r1: validate header + manifest here; the meta CRC (over header, manifest and CRC
  // table) is checked while K2 runs, and decides before anything is rebound: every
  // structural check has passed, so K2 only reads inside the image and writes inside
  // the new allocation, which an invalid image leaves unbound and frees
  const double tp = now_ms();
  const bool dev_img = img->location == CHECL_IMAGE_DEVICE;
  const size_t len = dev_img ? img->payload_off : img->image_bytes;
  // Fast path: the image's header names the layout of this device's last full-image
  // restore (every restore of a checkpoint/restore loop): its parse, segments and
  // chunk list are reused, and the manifest bytes are compared with it while K2 runs.
  // K2 with that layout stays inside the image (the header fixes its sizes) and inside
  // the new segments, so a mismatching manifest only costs a second, long-way restore.
  LayoutCache* lc = ctx->layout[device].get();
  const bool fast = !long_way && lc && lc->gen && img->host && len >= kHeaderBytes && header_same(img->host, lc->meta) &&
                    len >= (dev_img ? lc->P.L.payload_off : lc->P.L.image_bytes);
  Parsed parsed;
  if (!fast) {
    checl_status st = parse_image(img->host, len, dev_img, &parsed, false);
    if (st) return st;
    if (parsed.flags != 0) return CHECL_ERR_BAD_IMAGE;  // a delta restores only as part of a chain
  }
  const Parsed& P = fast ? lc->P : parsed;
  if (rep) set_report(rep, P, 0, 0);
  tr("parse");

  // r2: re-create the buffers: a few allocations (segments) laid out like the payload
  const double ta = now_ms();
  stream = stream_on(stream, device);
  RestoreAlloc A;
  if (!new_alloc(ctx, device, stream, P.bufs, P.L.payload_bytes, &A, fast ? &lc->segs : nullptr))
    // (an invalid image still reports BAD_IMAGE first)
    return get_u32(img->host + 124) == meta_crc(img->host, P.L.payload_off) ? CHECL_ERR_OUT_OF_DEVICE_MEMORY
                                                                           : CHECL_ERR_BAD_IMAGE;
  order_after(ds, stream);  // nothing below touches the new memory before the caller's queued work
  tm.alloc_ms = now_ms() - ta;
  tr("alloc");
  const uint64_t nch = P.L.n_chunks;
  std::vector<void*> bases = bases_of(A);
  ds.desc_scratch.ensure(std::max<uint64_t>(nch, 1));
  ds.round_scratch.ensure(nch + 1);
  ds.recs_scratch.ensure(std::max<size_t>(P.bufs.size(), 1));
  LaunchParams lp = base_params(ds);
  lp.desc = ds.desc_scratch.p;
  lp.round_base = ds.round_scratch.p;
  tm.plan_ms = now_ms() - tp;

  cudaEvent_t c_begin = ds.events.get(), c_end = ds.events.get();
  // the verify status is at rest unless an earlier restore stopped midway; the
  // publishing launch below leaves it at rest again (status_clean set after the sync)
  const bool was_clean = ds.status_clean, status_clean = was_clean && ds.status_host_dev;
  ds.status_clean = false;
  // the chunk list of the new segments: already in the scratch buffers when its key
  // (layout, segment addresses) is that of an earlier restore (segments alternate
  // between the two sets of consecutive restores: see adopt_plan), else expanded on
  // the GPU from one record per buffer (compute stream, ahead of the verify launches);
  // the expansion also initialises the verify status
  const bool have_list = status_clean && fast && ds.scratch_gen == lc->gen && ds.scratch_bases == bases;
  if (nch && !have_list) {
    ds.scratch_gen = 0;
    ds.h_recs.ensure(std::max<size_t>(P.bufs.size(), 1));
    // (zero-size buffers get a null pointer)
    const uint64_t rounds = build_records(P.bufs, [&](size_t b) { return A.buf(P.bufs, b); }, ds.h_recs.p);
    ck(cudaMemcpyAsync(ds.recs_scratch.p, ds.h_recs.p, P.bufs.size() * sizeof(BufferRecord), cudaMemcpyHostToDevice,
                       ds.compute));
    ++ds.aux_launches;
    ck(launch_expand(ds.recs_scratch.p, (uint32_t)P.bufs.size(), P.L.payload_bytes, nch, ds.desc_scratch.p,
                     ds.round_scratch.p, rounds, ds.status.p, ds.n_sms, ds.compute));
    if (fast) {  // the key of the list just expanded (a long-way restore sets it on success)
      ds.scratch_gen = lc->gen;
      ds.scratch_bases = bases;
    }
  }
  lp.status_host = ds.status_host_dev;  // the last verify launch publishes (below)
  tr("expand");
  DevBuf<uint8_t> tmp_payload;  // only when the source device is not peer-reachable
  DevBuf<uint32_t> tmp_crc;
  if (dev_img) {
    // device image (same GPU, or a peer GPU read over NVLink by the kernel)
    const uint8_t* src = img->d_payload;
    const uint32_t* crc = img->d_crc;
    if (!ensure_peer(device, img->device)) {
      ck(cudaEventRecord(c_begin, ds.copy));
      tmp_payload.ensure(P.L.payload_bytes + kSlotSlack);
      tmp_crc.ensure(std::max<uint64_t>(nch, 1));
      if (P.L.payload_bytes)
        ck(cudaMemcpyPeerAsync(tmp_payload.p, device, img->d_payload, img->device, P.L.payload_bytes, ds.copy));
      if (nch) ck(cudaMemcpyPeerAsync(tmp_crc.p, device, img->d_crc, img->device, 4 * nch, ds.copy));
      src = tmp_payload.p;
      crc = tmp_crc.p;
      ck(cudaEventRecord(c_end, ds.copy));
      ck(cudaStreamWaitEvent(ds.compute, c_end, 0));
    } else {  // nothing to copy: the kernel reads the image where it is
      c_begin = c_end = nullptr;
      // CHECL_FORCE_IMAGE_REMOTE=1 (tests): treat a same-device image as a peer GPU's,
      // so the one-GPU test box runs K2's peer-read path (register loads for every round)
      static const bool force_remote = std::getenv("CHECL_FORCE_IMAGE_REMOTE") != nullptr;
      lp.image_remote = img->device != device || force_remote;
#ifdef CHECL_EXPERIMENTS
      static const bool peer_bulk = std::getenv("CHECL_PEER_BULK") != nullptr;
      lp.remote_bulk = peer_bulk;
#endif
    }
    lp.c0 = 0;
    lp.c1 = nch;
    lp.image = const_cast<uint8_t*>(src);
    lp.image_base = 0;
    lp.crc = const_cast<uint32_t*>(crc);
    if (nch) timed_launch(ds, kt, kOpVerify, lp, ds.compute);
    tm.n_stages = 1;
    tr("launch");
  } else {
    // small pinned images (<= 128 chunks, payload <= CHECL_ZERO_COPY_MAX): K2 reads the
    // payload and the CRC table straight from the mapped pinned image over PCIe (exact
    // register loads), so there is no staging slot and no H2D copy
    static const uint64_t zc_max = [] {
      const char* e = std::getenv("CHECL_ZERO_COPY_MAX");
      return e ? (uint64_t)std::strtoull(e, nullptr, 10) : (8ull << 20);
    }();
    const uint8_t* mapped = nullptr;
    if (nch && nch <= 128 && img->pinned && img->host_cap >= P.L.image_bytes && P.L.payload_bytes <= zc_max &&
        P.L.payload_bytes <= ctx->slot_bytes) {
      void* dp = nullptr;
      if (cudaHostGetDevicePointer(&dp, const_cast<uint8_t*>(img->host), 0) == cudaSuccess)
        mapped = static_cast<const uint8_t*>(dp);
      else
        cudaGetLastError();
    }
    if (mapped) {
      ck(cudaEventRecord(c_begin, ds.compute));
      lp.c0 = 0;
      lp.c1 = nch;
      lp.image = const_cast<uint8_t*>(mapped + P.L.payload_off);
      lp.image_base = 0;
      lp.image_remote = 2;  // mapped pinned host memory: register loads only
      lp.crc = reinterpret_cast<uint32_t*>(const_cast<uint8_t*>(mapped + P.L.crc_off));
      timed_launch(ds, kt, kOpVerify, lp, ds.compute);
      ck(cudaEventRecord(c_end, ds.compute));
      tm.n_stages = 1;
    } else {
    // r3 + r4: fill slot s % n_slots over PCIe while the previous slot is verified
    ck(cudaEventRecord(c_begin, ds.copy));
    ds.ensure_slots(ctx->slot_bytes, ctx->n_slots);
    ds.crc_scratch.ensure(std::max<uint64_t>(nch, 1));
    if (nch) ck(cudaMemcpyAsync(ds.crc_scratch.p, img->host + P.L.crc_off, 4 * nch, cudaMemcpyHostToDevice, ds.copy));
    lp.crc = ds.crc_scratch.p;
    std::vector<Stage> stages = build_stages(P.bufs, P.L.payload_bytes, ctx->slot_bytes);
    std::vector<cudaEvent_t> filled(ds.n_slots), verified(ds.n_slots);
    for (uint32_t i = 0; i < ds.n_slots; ++i) {
      filled[i] = ds.events.get();
      verified[i] = ds.events.get();
    }
    for (size_t s = 0; s < stages.size(); ++s) {
      const Stage& S = stages[s];
      const uint32_t k = (uint32_t)(s % ds.n_slots);
      if (s >= ds.n_slots) ck(cudaStreamWaitEvent(ds.copy, verified[k], 0));
      ck(cudaMemcpyAsync(ds.slot(k), img->host + P.L.payload_off + S.img_lo, S.img_hi - S.img_lo,
                         cudaMemcpyHostToDevice, ds.copy));
      ck(cudaEventRecord(filled[k], ds.copy));
      ck(cudaStreamWaitEvent(ds.compute, filled[k], 0));
      lp.c0 = S.c0;
      lp.c1 = S.c1;
      lp.image = ds.slot(k);
      lp.image_base = S.img_lo;
      LaunchParams ls = lp;
      if (s + 1 != stages.size()) ls.status_host = nullptr;  // only the last launch publishes
      timed_launch(ds, kt, kOpVerify, ls, ds.compute);
      ck(cudaEventRecord(verified[k], ds.compute));
    }
    ck(cudaEventRecord(c_end, ds.copy));
    if (stages.empty()) ck(cudaStreamWaitEvent(ds.compute, c_end, 0));
    tm.n_stages = stages.size();
    }
  }
  if (nch && !lp.status_host) {
    ck(cudaMemcpyAsync(ds.h_status.p, ds.status.p, 16, cudaMemcpyDeviceToHost, ds.compute));
  } else if (!nch) {
    ds.h_status.p[0] = ~0ull;
    ds.h_status.p[1] = 0;
  }
  // r1, under K2: the meta CRC; on the fast path also the manifest the parse was skipped for
  const bool layout_ok =
      !fast || std::memcmp(img->host + kHeaderBytes, lc->meta.data() + kHeaderBytes, P.L.crc_off - kHeaderBytes) == 0;
  const bool meta_ok = layout_ok && get_u32(img->host + 124) == meta_crc(img->host, P.L.payload_off);
  settle(ctx);  // the previous call's spans, read while K2 runs
  ck(cudaDeviceSynchronize());  // K2, the copies, and every queue of the target (quiesce, L16)
  tr("wait");
  if (!layout_ok) {  // another manifest behind the same header: the long way
    ds.status_clean = nch ? lp.status_host != nullptr : was_clean;
    tmp_payload.release();
    tmp_crc.release();
    A = RestoreAlloc{};
    return do_restore(ctx, img, device, stream, rep, in_migrate, true);
  }
  ds.status_clean = nch ? lp.status_host != nullptr : was_clean;
  const uint64_t first_bad = ds.h_status.p[0], n_bad = ds.h_status.p[1];
  tm.n_kernels = kt.spans.size() + (ds.aux_launches - aux0);
  tmp_payload.release();
  tmp_crc.release();
  if (!meta_ok) {  // as if validation had failed first: no report, nothing rebound
    if (rep) std::memset(rep, 0, sizeof(*rep)), rep->first_bad_chunk = ~0ull;
    tm.total_ms = now_ms() - t0;
    defer_timing(ctx, ds, tm, kt, c_begin, c_end, CHECL_STATS_RESTORE);
    return CHECL_ERR_BAD_IMAGE;
  }
  if (rep) set_report(rep, P, n_bad, first_bad);
  if (n_bad) {
    tm.total_ms = now_ms() - t0;
    defer_timing(ctx, ds, tm, kt, c_begin, c_end, CHECL_STATS_RESTORE);
    return CHECL_ERR_CRC_MISMATCH;  // segments freed by their destructors; nothing rebound
  }
  // r5: rebind every handle (all-or-nothing)
  (void)in_migrate;
  const double tc = now_ms();
  tr("events");
  if (!fast) {  // this layout becomes the device's cached one
    auto nl = std::make_unique<LayoutCache>();
    nl->gen = ++g_layout_gen;
    nl->meta.assign(img->host, img->host + P.L.crc_off);
    std::memset(nl->meta.data() + 88, 0, 8);
    std::memset(nl->meta.data() + 124, 0, 4);
    nl->P = std::move(parsed);
    nl->segs = A.segs;
    ctx->layout[device] = std::move(nl);
    lc = ctx->layout[device].get();
    if (nch) {  // the list just expanded is this layout's over these segments
      ds.scratch_gen = lc->gen;
      ds.scratch_bases = bases;
    }
  }
  commit(ctx, lc->P, device, A, lc->gen);
  tr("commit");
  adopt_plan(ctx, ds, device, lc->P, A, lc->gen);
  tr("adopt");
  tm.commit_ms = now_ms() - tc;
  tm.total_ms = now_ms() - t0;
  defer_timing(ctx, ds, tm, kt, c_begin, c_end, CHECL_STATS_RESTORE);
  return CHECL_SUCCESS;
}

// -- incremental checkpoint (f1; §IV-D; FORMAT.md "Incremental images") --

// True when `base` describes the same registry layout as plan P (identical manifest
// bytes, chunk count and device): only then is a delta written.
bool same_layout(const uint8_t* base, const Parsed& B, const Plan& P, int device) {
  return B.L.n_chunks == P.n_chunks && B.L.crc_off == P.crc_off && B.source_device == device &&
         std::memcmp(base + kHeaderBytes, P.meta.data() + kHeaderBytes, P.crc_off - kHeaderBytes) == 0;
}

// The shadow of `device` now holds the payload of the full state `host_payload` (a full
// host image's payload) / `dev_payload` (a device image's); identified like the image.
void seed_shadow(DevState& ds, const Plan& P, const uint8_t* host_payload, const checl_image* dimg, uint64_t epoch,
                 uint32_t table_crc, uint32_t meta_crc_v) {
  ds.shadow_ok = false;
  ds.shadow.ensure(std::max<uint64_t>(P.payload_bytes, 1));
  if (P.payload_bytes) {
    if (host_payload)
      ck(cudaMemcpyAsync(ds.shadow.p, host_payload, P.payload_bytes, cudaMemcpyHostToDevice, ds.compute));
    else if (dimg->device == ds.dev)
      ck(cudaMemcpyAsync(ds.shadow.p, dimg->d_payload, P.payload_bytes, cudaMemcpyDeviceToDevice, ds.compute));
    else
      ck(cudaMemcpyPeerAsync(ds.shadow.p, ds.dev, dimg->d_payload, dimg->device, P.payload_bytes, ds.compute));
  }
  ds.shadow_epoch = epoch;
  ds.shadow_table_crc = table_crc;
  ds.shadow_meta_crc = meta_crc_v;
  ds.shadow_payload = P.payload_bytes;
  ds.shadow_ok = true;
}

checl_status do_checkpoint_incremental(checl_ctx* ctx, int device, void* stream, uint64_t epoch,
                                       const checl_image* base, checl_image* img, uint32_t rule) {
  // r1-style validation of the base's metadata (header, manifest, CRC table, bitmap)
  Parsed B;
  checl_status st = parse_image(base->host, base->location == CHECL_IMAGE_DEVICE ? base->payload_off : base->image_bytes,
                                true, &B);
  if (st) return st;
  const double t0 = now_ms();
  DeviceGuard g(device);
  DevState& ds = ctx->dev(device);
  const uint64_t aux0 = ds.aux_launches;
  const bool exact = rule == CHECL_DIRTY_BYTES;
  uint32_t mcrc = 0, tcrc = 0;
  {
    // the plan (and so the layout test) needs the registry as of this call
    Plan& P0 = get_plan(ctx, ds, device);
    const bool same = same_layout(base->host, B, P0, device);
    if (exact) {
      mcrc = host_crc32c(P0.meta.data() + kHeaderBytes, P0.crc_off - kHeaderBytes);
      tcrc = host_crc32c(base->host + B.L.crc_off, 4 * B.L.n_chunks);
    }
    const bool have_state = ds.shadow_ok && ds.shadow_epoch == B.epoch && ds.shadow_table_crc == tcrc &&
                            ds.shadow_meta_crc == mcrc && ds.shadow_payload == P0.payload_bytes;
    if (!same || (exact && !have_state && B.flags != 0)) {
      // a layout change, or (bytes rule) a delta base whose state the device does not
      // hold: the full image, which is a valid result of any incremental checkpoint
      st = do_checkpoint(ctx, device, stream, epoch, img, false);
      if (st == CHECL_SUCCESS && exact) {  // its state becomes the shadow (next delta: exact)
        Plan& P1 = get_plan(ctx, ds, device);
        seed_shadow(ds, P1, img->host + P1.payload_off, nullptr, epoch, host_crc32c(img->host + P1.crc_off, 4 * P1.n_chunks),
                    host_crc32c(P1.meta.data() + kHeaderBytes, P1.crc_off - kHeaderBytes));
        ck(cudaStreamSynchronize(ds.compute));
      }
      return st;
    }
    if (exact && !have_state) {  // a full base: its payload becomes the shadow
      if (base->location == CHECL_IMAGE_DEVICE)
        seed_shadow(ds, P0, nullptr, base, B.epoch, tcrc, mcrc);
      else
        seed_shadow(ds, P0, base->host + B.L.payload_off, nullptr, B.epoch, tcrc, mcrc);
    }
  }
  begin_events(ctx, ds);
  KernelTimer kt;
  checl_timing tm{};

  // a1: quiesce (L16 step 1)
  const double ts = now_ms();
  ck(cudaDeviceSynchronize());
  tm.sync_ms = now_ms() - ts;
  const double tp = now_ms();
  Plan& P = get_plan(ctx, ds, device);
  const uint64_t n = P.n_chunks;
  const uint64_t map_bytes = (n + 7) / 8;
  const uint64_t W = ctx->slot_bytes - (kChunkBytes + kBufferAlign);  // stage window (a span fits the slack)
  const uint64_t max_stages = (P.payload_bytes + W - 1) / W + 1;
  ds.crc_scratch.ensure(std::max<uint64_t>(n, 1));
  ds.base_crc.ensure(std::max<uint64_t>(n, 1));
  ds.map_words.ensure(std::max<uint64_t>((n + 31) / 32, 1));
  ds.cdesc.ensure(std::max<uint64_t>(n, 1));
  ds.dtotals.ensure(2);
  ds.stage_first.ensure(max_stages + 1);
  ds.stage_lo.ensure(max_stages + 1);
  ds.h_dtab.ensure(2 + 2 * (max_stages + 1));
  if (exact) {
    ds.dirty.ensure(std::max<uint64_t>((n + 31) / 32, 1));
    ds.ccrc.ensure(std::max<uint64_t>(n, 1));
    ds.cidx.ensure(std::max<uint64_t>(n, 1));
  }
  tm.plan_ms = now_ms() - tp;

  // The present set:
  //  CRC rule: CRC of every chunk as it is now (kOpCrc: read-only pass) vs base's table;
  //  bytes rule: every chunk compared with the shadow (diff_kernel, which also brings
  //  the shadow up to date); then the compacted chunk list and the stage table
  //  (delta_scan / delta_stages)
  LaunchParams lp = base_params(ds);
  lp.desc = P.d_desc.p;
  lp.round_base = P.d_round.p;
  lp.crc = ds.crc_scratch.p;
  lp.c0 = 0;
  lp.c1 = n;
  if (n)
    ck(cudaMemcpyAsync(exact ? ds.crc_scratch.p : ds.base_crc.p, base->host + B.L.crc_off, 4 * n, cudaMemcpyHostToDevice,
                       ds.compute));
  cudaEvent_t sa = ds.events.get(), sb = ds.events.get();
  if (exact) {
    ds.shadow_ok = false;  // (advanced in place below; valid again once the delta is written)
    ck(cudaEventRecord(sa, ds.compute));
    ck(cudaMemsetAsync(ds.dirty.p, 0, 4 * ((n + 31) / 32), ds.compute));
    ds.aux_launches += 3;
    ck(launch_diff(P.d_desc.p, n, ds.shadow.p, ds.dirty.p, ds.n_sms, ds.compute));
    ck(launch_delta_scan(P.d_desc.p, nullptr, nullptr, ds.dirty.p, n, ds.map_words.p, ds.cdesc.p, ds.cidx.p, ds.dtotals.p,
                         ds.compute));
  } else {
    if (n) timed_launch(ds, kt, kOpCrc, lp, ds.compute);
    ck(cudaEventRecord(sa, ds.compute));
    ds.aux_launches += 2;
    ck(launch_delta_scan(P.d_desc.p, ds.crc_scratch.p, ds.base_crc.p, nullptr, n, ds.map_words.p, ds.cdesc.p, nullptr,
                         ds.dtotals.p, ds.compute));
  }
  ck(launch_delta_stages(ds.cdesc.p, ds.dtotals.p, W, max_stages, ds.stage_first.p, ds.stage_lo.p, ds.compute));
  ck(cudaEventRecord(sb, ds.compute));
  kt.spans.push_back({sa, sb});
  unsigned long long* h = ds.h_dtab.p;
  ck(cudaMemcpyAsync(h, ds.dtotals.p, 16, cudaMemcpyDeviceToHost, ds.compute));
  ck(cudaMemcpyAsync(h + 2, ds.stage_first.p, 8 * (max_stages + 1), cudaMemcpyDeviceToHost, ds.compute));
  ck(cudaMemcpyAsync(h + 3 + max_stages, ds.stage_lo.p, 8 * (max_stages + 1), cudaMemcpyDeviceToHost, ds.compute));
  ck(cudaStreamSynchronize(ds.compute));
  const uint64_t n_present = h[0], dbytes = h[1];
  const unsigned long long* first = h + 2;
  const unsigned long long* lo = h + 3 + max_stages;

  // delta layout (FORMAT.md): bitmap after the CRC table, compacted payload
  const uint64_t payload_off = align_up(P.crc_off + 4 * n + map_bytes, kPayloadAlign);
  const uint64_t image_bytes = payload_off + dbytes;
  if (img->location != CHECL_IMAGE_HOST) {
    img->free_device();
    img->free_host();
    img->location = CHECL_IMAGE_HOST;
    img->device = -1;
  }
  img->ensure_host(image_bytes, true);

  // a3 + a4 over the present chunks only: gather into slot s % n_slots while the copy
  // engine drains the previous slot (CRC rule: kOpCopy, the CRCs are known; bytes rule:
  // kOpPack, the CRC of each present chunk into ccrc, scattered into the table after)
  ds.ensure_slots(ctx->slot_bytes, ctx->n_slots);
  std::vector<cudaEvent_t> packed(ds.n_slots), drained(ds.n_slots);
  for (uint32_t i = 0; i < ds.n_slots; ++i) {
    packed[i] = ds.events.get();
    drained[i] = ds.events.get();
  }
  cudaEvent_t c_begin = ds.events.get(), c_end = ds.events.get();
  ck(cudaEventRecord(c_begin, ds.copy));
  lp.desc = ds.cdesc.p;
  lp.round_base = nullptr;  // compacted list: grid-stride kernels
  if (exact) lp.crc = ds.ccrc.p;
  size_t used = 0;
  for (uint64_t s = 0; s < max_stages; ++s) {
    if (first[s] == first[s + 1]) continue;
    const uint32_t k = (uint32_t)(used % ds.n_slots);
    if (used >= ds.n_slots) ck(cudaStreamWaitEvent(ds.compute, drained[k], 0));
    lp.c0 = first[s];
    lp.c1 = first[s + 1];
    lp.image = ds.slot(k);
    lp.image_base = lo[s];
    timed_launch(ds, kt, exact ? kOpPack : kOpCopy, lp, ds.compute);
    ck(cudaEventRecord(packed[k], ds.compute));
    ck(cudaStreamWaitEvent(ds.copy, packed[k], 0));
    d2h_page_aligned(img->host_mut + payload_off + lo[s], ds.slot(k), lo[s + 1] - lo[s], ds.copy);
    ck(cudaEventRecord(drained[k], ds.copy));
    ++used;
  }
  if (n) {
    if (exact) {  // the base's table with the present chunks' new CRCs
      ++ds.aux_launches;
      ck(launch_crc_scatter(ds.ccrc.p, ds.cidx.p, ds.dtotals.p, n_present, ds.crc_scratch.p, ds.n_sms, ds.compute));
      cudaEvent_t tab = ds.events.get();
      ck(cudaEventRecord(tab, ds.compute));
      ck(cudaStreamWaitEvent(ds.copy, tab, 0));
    }
    ck(cudaMemcpyAsync(img->host_mut + P.crc_off, ds.crc_scratch.p, 4 * n, cudaMemcpyDeviceToHost, ds.copy));
    ck(cudaMemcpyAsync(img->host_mut + P.crc_off + 4 * n, ds.map_words.p, map_bytes, cudaMemcpyDeviceToHost, ds.copy));
  }
  ck(cudaEventRecord(c_end, ds.copy));
  tm.n_stages = used;
  ck(cudaStreamSynchronize(ds.copy));

  // a5: header (the full image's, then the incremental fields), manifest, meta CRC
  const double tf = now_ms();
  uint8_t* o = img->host_mut;
  std::memcpy(o, P.meta.data(), P.crc_off);
  put_u64(o + 56, payload_off);
  put_u64(o + 64, dbytes);
  put_u64(o + 72, image_bytes);
  put_u32(o + 84, 1);
  put_u64(o + 88, epoch);
  put_u64(o + 96, B.epoch);
  put_u32(o + 104, exact ? tcrc : host_crc32c(base->host + B.L.crc_off, 4 * n));
  put_u32(o + 108, rule);
  put_u64(o + 112, n_present);
  put_u32(o + 120, 0);
  std::memset(o + P.crc_off + 4 * n + map_bytes, 0, payload_off - P.crc_off - 4 * n - map_bytes);
  put_u32(o + 124, meta_crc(o, payload_off));
  if (exact) {  // the shadow now holds this image's state
    ds.shadow_epoch = epoch;
    ds.shadow_table_crc = host_crc32c(o + P.crc_off, 4 * n);
    ds.shadow_ok = true;
  }
  tm.commit_ms = now_ms() - tf;
  img->image_bytes = image_bytes;
  img->payload_off = payload_off;
  tm.n_kernels = kt.spans.size() + (ds.aux_launches - aux0);
  tm.total_ms = now_ms() - t0;
  defer_timing(ctx, ds, tm, kt, c_begin, c_end, CHECL_STATS_INCREMENTAL);
  return CHECL_SUCCESS;
}

// Link of a delta D to the previous image E of a chain (FORMAT.md "Base link").
bool linked(const checl_image* e, const Parsed& E, const checl_image* d, const Parsed& D) {
  return D.flags == 1 && D.base_epoch == E.epoch && D.L.n_chunks == E.L.n_chunks && D.L.crc_off == E.L.crc_off &&
         D.source_device == E.source_device &&
         D.base_table_crc == host_crc32c(e->host + E.L.crc_off, 4 * E.L.n_chunks) &&
         std::memcmp(d->host + kHeaderBytes, e->host + kHeaderBytes, D.L.crc_off - kHeaderBytes) == 0;
}

// Restore of a chain [F, D1, ..., Dn] of host images: F's payload is copied into
// the new allocation (laid out like the full payload), each delta's present spans
// are scattered over it in chain order (kOpScatter from the staging slots), and
// one in-place verify (kOpCheck) checks every chunk against the last CRC table.
// All-or-nothing like checl_restore.
checl_status do_restore_chain(checl_ctx* ctx, const checl_image* const* chain, uint32_t n_img, int device,
                              void* stream, checl_report* rep) {
  const double t0 = now_ms();
  if (rep) std::memset(rep, 0, sizeof(*rep)), rep->first_bad_chunk = ~0ull;
  const double tp = now_ms();
  std::vector<Parsed> Ps(n_img);
  for (uint32_t i = 0; i < n_img; ++i) {
    if (chain[i]->location != CHECL_IMAGE_HOST) return CHECL_ERR_INVALID_VALUE;
    checl_status st = parse_image(chain[i]->host, chain[i]->image_bytes, false, &Ps[i]);
    if (st) return st;
    if ((i == 0) != (Ps[i].flags == 0)) return CHECL_ERR_BAD_IMAGE;
    if (i > 0 && !linked(chain[i - 1], Ps[i - 1], chain[i], Ps[i])) return CHECL_ERR_BAD_IMAGE;
  }
  const Parsed& F = Ps[0];
  const Parsed& Z = Ps[n_img - 1];
  DeviceGuard g(device);
  DevState& ds = ctx->dev(device);
  const uint64_t aux0 = ds.aux_launches;
  begin_events(ctx, ds);
  KernelTimer kt;
  checl_timing tm{};
  const double ts = now_ms();
  ck(cudaDeviceSynchronize());
  tm.sync_ms = now_ms() - ts;
  if (rep) set_report(rep, Z, 0, 0);

  // r2: segments laid out like the full payload
  const double ta = now_ms();
  stream = stream_on(stream, device);
  RestoreAlloc A;
  if (!new_alloc(ctx, device, stream, F.bufs, F.full_payload, &A)) return CHECL_ERR_OUT_OF_DEVICE_MEMORY;
  order_after(ds, stream);
  tm.alloc_ms = now_ms() - ta;
  const uint64_t nch = F.L.n_chunks;

  // descriptors of every delta's present chunks: ptr = destination in the arena,
  // img_off = position in that delta's compacted payload; stages per delta
  struct DStage {
    uint32_t img;
    uint64_t c0, c1, lo, hi;
  };
  std::vector<ChunkDesc> hdesc;
  std::vector<DStage> dst;
  for (uint32_t i = 1; i < n_img; ++i) {
    const Parsed& D = Ps[i];
    const uint8_t* map = chain[i]->host + D.map_off;
    uint64_t pos = 0;
    bool open = false;
    DStage cur{i, 0, 0, 0, 0};
    for (size_t b = 0; b < D.bufs.size(); ++b) {
      const uint64_t nb = chunks_of(D.bufs[b].size);
      for (uint64_t j = 0; j < nb; ++j) {
        if (!bit_set(map, D.bufs[b].first_chunk + j)) continue;
        uint64_t a, z;
        chunk_span(D.bufs, b, j, D.full_payload, &a, &z);
        const uint32_t len = (uint32_t)std::min<uint64_t>(kChunkBytes, D.bufs[b].size - (uint64_t)kChunkBytes * j);
        if (open && pos + (z - a) - cur.lo > ctx->slot_bytes) {
          dst.push_back(cur);
          open = false;
        }
        if (!open) {
          cur = DStage{i, hdesc.size(), hdesc.size(), pos, pos};
          open = true;
        }
        hdesc.push_back(ChunkDesc{reinterpret_cast<uint64_t>(A.at(a)), (uint32_t)(pos / kBufferAlign),
                                  make_len_pad(len, (uint32_t)(z - a - len))});
        pos += z - a;
        cur.c1 = hdesc.size();
        cur.hi = pos;
      }
    }
    if (open) dst.push_back(cur);
  }
  ds.scratch_gen = 0;  // the scratch list is overwritten (no longer described)
  ds.status_clean = false;
  ds.desc_scratch.ensure(std::max<uint64_t>(std::max<uint64_t>(nch, hdesc.size()), 1));
  ds.cdesc.ensure(std::max<size_t>(hdesc.size(), 1));
  ds.crc_scratch.ensure(std::max<uint64_t>(nch, 1));
  ds.h_recs.ensure(std::max<size_t>(F.bufs.size(), 1));
  ds.recs_scratch.ensure(std::max<size_t>(F.bufs.size(), 1));
  const uint64_t rounds = build_records(F.bufs, [&](size_t b) { return A.buf(F.bufs, b); }, ds.h_recs.p);
  ds.round_scratch.ensure(nch + 1);
  tm.plan_ms = now_ms() - tp;

  cudaEvent_t c_begin = ds.events.get(), c_end = ds.events.get(), base_in = ds.events.get();
  ck(cudaEventRecord(c_begin, ds.copy));
  // r3: F's payload straight into the segments; the last CRC table; the delta chunk list
  for (size_t k = 0; k < A.segs.size(); ++k)
    if (A.segs[k].hi > A.segs[k].lo)
      ck(cudaMemcpyAsync(A.arenas[k]->base, chain[0]->host + F.L.payload_off + A.segs[k].lo, A.segs[k].hi - A.segs[k].lo,
                         cudaMemcpyHostToDevice, ds.copy));
  ck(cudaEventRecord(base_in, ds.copy));
  if (nch)
    ck(cudaMemcpyAsync(ds.crc_scratch.p, chain[n_img - 1]->host + Z.L.crc_off, 4 * nch, cudaMemcpyHostToDevice, ds.copy));
  if (!hdesc.empty())
    ck(cudaMemcpyAsync(ds.cdesc.p, hdesc.data(), hdesc.size() * sizeof(ChunkDesc), cudaMemcpyHostToDevice, ds.copy));
  if (nch) {  // the expansion also initialises the verify status
    ck(cudaMemcpyAsync(ds.recs_scratch.p, ds.h_recs.p, F.bufs.size() * sizeof(BufferRecord), cudaMemcpyHostToDevice,
                       ds.compute));
    ++ds.aux_launches;
    ck(launch_expand(ds.recs_scratch.p, (uint32_t)F.bufs.size(), F.full_payload, nch, ds.desc_scratch.p,
                     ds.round_scratch.p, rounds, ds.status.p, ds.n_sms, ds.compute));
  }
  ck(cudaStreamWaitEvent(ds.compute, base_in, 0));
  // deltas in chain order: fill slot k over PCIe, scatter its spans (later deltas
  // overwrite earlier ones: every scatter runs on the compute stream in order)
  ds.ensure_slots(ctx->slot_bytes, ctx->n_slots);
  std::vector<cudaEvent_t> filled(ds.n_slots), done(ds.n_slots);
  for (uint32_t i = 0; i < ds.n_slots; ++i) {
    filled[i] = ds.events.get();
    done[i] = ds.events.get();
  }
  LaunchParams lp = base_params(ds);
  lp.desc = ds.cdesc.p;
  lp.round_base = nullptr;  // host-built list: grid-stride kernels
  for (size_t s = 0; s < dst.size(); ++s) {
    const DStage& S = dst[s];
    const uint32_t k = (uint32_t)(s % ds.n_slots);
    if (s >= ds.n_slots) ck(cudaStreamWaitEvent(ds.copy, done[k], 0));
    ck(cudaMemcpyAsync(ds.slot(k), chain[S.img]->host + Ps[S.img].L.payload_off + S.lo, S.hi - S.lo,
                       cudaMemcpyHostToDevice, ds.copy));
    ck(cudaEventRecord(filled[k], ds.copy));
    ck(cudaStreamWaitEvent(ds.compute, filled[k], 0));
    lp.c0 = S.c0;
    lp.c1 = S.c1;
    lp.image = ds.slot(k);
    lp.image_base = S.lo;
    timed_launch(ds, kt, kOpScatter, lp, ds.compute);
    ck(cudaEventRecord(done[k], ds.compute));
  }
  ck(cudaEventRecord(c_end, ds.copy));
  ck(cudaStreamWaitEvent(ds.compute, c_end, 0));
  // r4: every chunk of the result against the last CRC table, in place
  lp.desc = ds.desc_scratch.p;
  lp.round_base = ds.round_scratch.p;
  lp.crc = ds.crc_scratch.p;
  lp.c0 = 0;
  lp.c1 = nch;
  lp.image = nullptr;
  lp.image_base = 0;
  if (nch) {
    lp.status_host = ds.status_host_dev;
    timed_launch(ds, kt, kOpCheck, lp, ds.compute);
    if (!lp.status_host) ck(cudaMemcpyAsync(ds.h_status.p, ds.status.p, 16, cudaMemcpyDeviceToHost, ds.compute));
  } else {
    ds.h_status.p[0] = ~0ull;
    ds.h_status.p[1] = 0;
  }
  ck(cudaStreamSynchronize(ds.compute));
  ck(cudaStreamSynchronize(ds.copy));
  ds.status_clean = nch && lp.status_host;
  const uint64_t first_bad = ds.h_status.p[0], n_bad = ds.h_status.p[1];
  tm.n_kernels = kt.spans.size() + (ds.aux_launches - aux0);
  tm.n_stages = dst.size() + 1;
  if (rep) set_report(rep, Z, n_bad, first_bad);
  if (n_bad) {
    tm.total_ms = now_ms() - t0;
    defer_timing(ctx, ds, tm, kt, c_begin, c_end, CHECL_STATS_CHAIN);
    return CHECL_ERR_CRC_MISMATCH;
  }
  const double tc = now_ms();
  commit(ctx, Z, device, A, 0);
  tm.commit_ms = now_ms() - tc;
  tm.total_ms = now_ms() - t0;
  defer_timing(ctx, ds, tm, kt, c_begin, c_end, CHECL_STATS_CHAIN);
  return CHECL_SUCCESS;
}

}  // namespace

// ============================== C ABI =========================================

extern "C" {

checl_status checl_create(const checl_allocator* a, checl_ctx** out) {
  if (!out) return CHECL_ERR_INVALID_VALUE;
  return guarded([&]() -> checl_status {
    auto* c = new checl_ctx();
    if (a) c->alloc = *a;
    if (const char* s = std::getenv("CHECL_STAGING_BYTES")) {
      const unsigned long long v = std::strtoull(s, nullptr, 10);
      if (v >= kChunkBytes + kBufferAlign && v % kChunkBytes == 0) c->slot_bytes = v;
    }
    *out = c;
    return CHECL_SUCCESS;
  });
}

checl_status checl_destroy(checl_ctx* ctx) {
  if (!ctx) return CHECL_ERR_INVALID_VALUE;
  return guarded([&]() -> checl_status {
    {
      // delete in the reverse of creation order (L19-L20)
      std::lock_guard<std::mutex> lk(ctx->mu);
      bool synced[kMaxDevices] = {};
      for (Binding* b : ctx->bindings)
        for (auto& a : b->seg_arena)
          if (a && a->base && !synced[a->device]) {  // no kernel may still touch them
            int prev = -1;
            cudaGetDevice(&prev);
            cudaSetDevice(a->device);
            cudaDeviceSynchronize();
            if (prev >= 0) cudaSetDevice(prev);
            synced[a->device] = true;
          }
      ctx->entries.clear();
      for (Binding* b : ctx->bindings) delete b;  // (frees the segments)
      ctx->bindings.clear();
      ctx->bind.binding = nullptr;
      for (auto& n : ctx->n_live) n = 0;
      for (auto& sp : ctx->spares) sp.clear();
      ctx->deferred.clear();
    }
    for (auto*& d : ctx->devs) {
      if (d) {
        d->destroy();
        delete d;
        d = nullptr;
      }
    }
    for (auto& c : g_signal_ctx) {
      checl_ctx* expect = ctx;
      c.compare_exchange_strong(expect, nullptr);
    }
    delete ctx;
    return CHECL_SUCCESS;
  });
}

checl_status checl_set_staging(checl_ctx* ctx, size_t slot_bytes, uint32_t n_slots) {
  if (!ctx || slot_bytes < kChunkBytes + kBufferAlign || slot_bytes % kChunkBytes || n_slots < 1 ||
      n_slots > kMaxSlots)
    return CHECL_ERR_INVALID_VALUE;
  std::lock_guard<std::mutex> lk(ctx->mu);
  ctx->slot_bytes = slot_bytes;
  ctx->n_slots = n_slots;
  return CHECL_SUCCESS;
}

checl_status checl_register_buffer(checl_ctx* ctx, int device, void* dev_ptr, size_t bytes, uint32_t flags,
                                   checl_handle* out) {
  if (!ctx || !out || (bytes > 0 && !dev_ptr)) return CHECL_ERR_INVALID_VALUE;
  if (!valid_device(device)) return CHECL_ERR_INVALID_DEVICE;
  const uintptr_t lo = reinterpret_cast<uintptr_t>(dev_ptr);
  if (bytes && lo > ~(uintptr_t)0 - bytes) return CHECL_ERR_INVALID_VALUE;
  return guarded([&]() -> checl_status {
    std::lock_guard<std::mutex> lk(ctx->mu);
    if (bytes) {
      auto& m = ctx->by_addr[device];
      auto it = m.upper_bound(lo);  // first range starting after lo
      if (it != m.end() && it->first < lo + bytes) return CHECL_ERR_INVALID_VALUE;
      if (it != m.begin()) {
        --it;  // range starting at or before lo
        if (it->first + it->second.bytes > lo) return CHECL_ERR_INVALID_VALUE;
      }
      // the library's own live segments (a few per restore; not in the range map, so
      // that a commit does not update it per segment)
      for (Binding* b : ctx->bindings)
        for (auto& a : b->seg_arena)
          if (a && a->base && a->device == device) {
            const uintptr_t s0 = reinterpret_cast<uintptr_t>(a->base);
            if (lo < s0 + a->bytes && s0 < lo + bytes) return CHECL_ERR_INVALID_VALUE;
          }
    }
    const uint64_t h = ctx->next_id++;
    Entry e;
    e.device = device;
    e.ptr = static_cast<uint8_t*>(dev_ptr);
    e.bytes = bytes;
    e.flags = flags;
    e.owned = false;
    e.bind = nullptr;
    e.idx = 0;
    ctx->entries.emplace(h, std::move(e));
    ctx->n_live[device]++;
    if (bytes) ctx->by_addr[device][lo] = {bytes, h};
    ctx->version[device]++;
    *out = h;
    return CHECL_SUCCESS;
  });
}

checl_status checl_release(checl_ctx* ctx, checl_handle h) {
  if (!ctx) return CHECL_ERR_INVALID_VALUE;
  return guarded([&]() -> checl_status {
    std::shared_ptr<Arena> drop;
    int dev = -1;
    {
      std::lock_guard<std::mutex> lk(ctx->mu);
      auto it = ctx->entries.find(h);
      if (it == ctx->entries.end()) return CHECL_ERR_INVALID_HANDLE;
      Entry& e = it->second;
      dev = e.device;
      if (!e.owned && e.bytes) ctx->by_addr[e.device].erase(reinterpret_cast<uintptr_t>(e.ptr));
      std::vector<std::shared_ptr<Arena>> d;
      release_slot(ctx, e, d);  // the segment's last handle: d holds it
      if (!d.empty()) {
        drop = std::move(d.front());
        // a checkpoint / restore / migrate running on another thread may have planned
        // reads of it: that call frees it when it ends (BusyGuard)
        if (ctx->busy.load()) ctx->deferred.push_back(std::move(drop));
      }
      ctx->version[e.device]++;
      ctx->n_live[e.device]--;
      ctx->entries.erase(it);
    }
    (void)dev;
    std::vector<std::shared_ptr<Arena>> v;
    if (drop) v.push_back(std::move(drop));
    free_arenas(v);  // (after the device is idle)
    return CHECL_SUCCESS;
  });
}

checl_status checl_translate(const checl_ctx* ctx, checl_handle h, void** dev_ptr, size_t* bytes, int* device) {
  if (!ctx) return CHECL_ERR_INVALID_VALUE;
  std::lock_guard<std::mutex> lk(ctx->mu);
  auto it = ctx->entries.find(h);
  if (it == ctx->entries.end()) return CHECL_ERR_INVALID_HANDLE;
  if (dev_ptr) *dev_ptr = entry_ptr(it->second);
  if (bytes) *bytes = it->second.bytes;
  if (device) *device = it->second.device;
  return CHECL_SUCCESS;
}

checl_status checl_count(const checl_ctx* ctx, int device, uint64_t* n_buffers, uint64_t* total_bytes) {
  if (!ctx) return CHECL_ERR_INVALID_VALUE;
  if (!valid_device(device)) return CHECL_ERR_INVALID_DEVICE;
  std::lock_guard<std::mutex> lk(ctx->mu);
  uint64_t n = 0, t = 0;
  for (auto& kv : ctx->entries)
    if (kv.second.device == device) ++n, t += kv.second.bytes;
  if (n_buffers) *n_buffers = n;
  if (total_bytes) *total_bytes = t;
  return CHECL_SUCCESS;
}

static checl_status checkpoint_common(checl_ctx* ctx, int device, void* stream, uint64_t epoch, checl_image* img,
                                      bool to_device) {
  BusyGuard b(ctx);
  if (!b.ok) return CHECL_ERR_BUSY;
  return guarded([&]() { return do_checkpoint(ctx, device, stream, epoch, img, to_device); });
}

checl_status checl_checkpoint(checl_ctx* ctx, int device, void* cuda_stream, uint64_t epoch, checl_image** out) {
  if (!ctx || !out) return CHECL_ERR_INVALID_VALUE;
  if (!valid_device(device)) return CHECL_ERR_INVALID_DEVICE;
  checl_image* img = new (std::nothrow) checl_image();
  if (!img) return CHECL_ERR_OUT_OF_HOST_MEMORY;
  checl_status st = checkpoint_common(ctx, device, cuda_stream, epoch, img, false);
  if (st) {
    checl_image_free(img);
    return st;
  }
  *out = img;
  return CHECL_SUCCESS;
}

checl_status checl_checkpoint_device(checl_ctx* ctx, int device, void* cuda_stream, uint64_t epoch,
                                     checl_image** out) {
  if (!ctx || !out) return CHECL_ERR_INVALID_VALUE;
  if (!valid_device(device)) return CHECL_ERR_INVALID_DEVICE;
  checl_image* img = new (std::nothrow) checl_image();
  if (!img) return CHECL_ERR_OUT_OF_HOST_MEMORY;
  checl_status st = checkpoint_common(ctx, device, cuda_stream, epoch, img, true);
  if (st) {
    checl_image_free(img);
    return st;
  }
  *out = img;
  return CHECL_SUCCESS;
}

checl_status checl_checkpoint_into(checl_ctx* ctx, int device, void* cuda_stream, uint64_t epoch,
                                   checl_image* reuse) {
  if (!ctx || !reuse || !reuse->owned) return CHECL_ERR_INVALID_VALUE;
  if (!valid_device(device)) return CHECL_ERR_INVALID_DEVICE;
  return checkpoint_common(ctx, device, cuda_stream, epoch, reuse, reuse->location == CHECL_IMAGE_DEVICE);
}

checl_status checl_image_view(const checl_image* img, const void** bytes, size_t* nbytes) {
  if (!img || !bytes || !nbytes) return CHECL_ERR_INVALID_VALUE;
  *bytes = img->host;
  *nbytes = img->location == CHECL_IMAGE_DEVICE ? img->payload_off : img->image_bytes;
  return CHECL_SUCCESS;
}

checl_status checl_image_info(const checl_image* img, int* location, int* device, uint64_t* image_bytes,
                              void** device_payload) {
  if (!img) return CHECL_ERR_INVALID_VALUE;
  if (location) *location = img->location;
  if (device) *device = img->location == CHECL_IMAGE_DEVICE ? img->device : -1;
  if (image_bytes) *image_bytes = img->image_bytes;
  if (device_payload) *device_payload = img->d_payload;
  return CHECL_SUCCESS;
}

checl_status checl_image_wrap(const void* bytes, size_t nbytes, checl_image** out) {
  if (!out || (!bytes && nbytes)) return CHECL_ERR_INVALID_VALUE;
  checl_image* img = new (std::nothrow) checl_image();
  if (!img) return CHECL_ERR_OUT_OF_HOST_MEMORY;
  img->owned = false;
  img->host = static_cast<const uint8_t*>(bytes);
  img->host_cap = nbytes;
  img->image_bytes = nbytes;  // validated against the header at restore
  img->payload_off = nbytes >= 64 ? get_u64(static_cast<const uint8_t*>(bytes) + 56) : 0;
  *out = img;
  return CHECL_SUCCESS;
}

checl_status checl_image_to_host(const checl_image* img, checl_image** out) {
  if (!img || !out) return CHECL_ERR_INVALID_VALUE;
  return guarded([&]() -> checl_status {
    checl_image* h = new checl_image();
    try {
      if (img->location == CHECL_IMAGE_HOST) {
        h->ensure_host(img->image_bytes, false);
        std::memcpy(h->host_mut, img->host, img->image_bytes);
      } else {
        DeviceGuard g(img->device);
        h->ensure_host(img->image_bytes, true);
        std::memcpy(h->host_mut, img->host, img->payload_off);
        if (img->image_bytes > img->payload_off)
          ck(cudaMemcpy(h->host_mut + img->payload_off, img->d_payload, img->image_bytes - img->payload_off,
                        cudaMemcpyDeviceToHost));
      }
    } catch (...) {
      h->free_host();
      delete h;
      throw;
    }
    h->image_bytes = img->image_bytes;
    h->payload_off = img->payload_off;
    *out = h;
    return CHECL_SUCCESS;
  });
}

checl_status checl_image_free(checl_image* img) {
  if (!img) return CHECL_SUCCESS;
  img->free_device();
  img->free_host();
  delete img;
  return CHECL_SUCCESS;
}

checl_status checl_restore(checl_ctx* ctx, const checl_image* img, int device, void* cuda_stream, checl_report* rep) {
  if (!ctx || !img) return CHECL_ERR_INVALID_VALUE;
  if (!valid_device(device)) return CHECL_ERR_INVALID_DEVICE;
  if (img->location == CHECL_IMAGE_DEVICE && !valid_device(img->device)) return CHECL_ERR_INVALID_DEVICE;
  BusyGuard b(ctx);
  if (!b.ok) return CHECL_ERR_BUSY;
  return guarded([&]() { return do_restore(ctx, img, device, cuda_stream, rep, false); });
}

checl_status checl_migrate(checl_ctx* ctx, int src_device, int dst_device, void* cuda_stream, checl_report* rep) {
  if (!ctx) return CHECL_ERR_INVALID_VALUE;
  if (!valid_device(src_device) || !valid_device(dst_device)) return CHECL_ERR_INVALID_DEVICE;
  BusyGuard b(ctx);
  if (!b.ok) return CHECL_ERR_BUSY;
  return guarded([&]() -> checl_status {
    const double t0 = now_ms();
    // m1: the image of src's buffers in src's HBM, allocated through the context's
    // allocator and freed as soon as K2 on dst has read it (a move: the source GPU
    // keeps nothing, L41 §IV-C), so it returns to the caller's memory pool
    checl_image img;
    img.dalloc = ctx->alloc;
    img.dstream = stream_on(cuda_stream, src_device);
    struct Drop {
      checl_image& i;
      ~Drop() {
        i.free_device();
        i.free_host();
      }
    } drop{img};
    checl_status st = do_checkpoint(ctx, src_device, cuda_stream, 0, &img, true);
    settle(ctx);
    checl_timing ck_t = ctx->last;
    // m2-m3: verify + scatter on dst reading src's HBM over NVLink, rebind to dst
    if (st == CHECL_SUCCESS) st = do_restore(ctx, &img, dst_device, cuda_stream, rep, true);
    settle(ctx);
    std::lock_guard<std::mutex> lk(ctx->tmu);
    checl_timing& t = ctx->last;
    t.sync_ms += ck_t.sync_ms;
    t.plan_ms += ck_t.plan_ms;
    t.kernel_ms += ck_t.kernel_ms;
    t.copy_ms += ck_t.copy_ms;
    t.n_kernels += ck_t.n_kernels;
    t.n_stages += ck_t.n_stages;
    t.total_ms = now_ms() - t0;
    return st;
  });
}

checl_status checl_checkpoint_incremental(checl_ctx* ctx, int device, void* cuda_stream, uint64_t epoch,
                                          const checl_image* base, checl_image** out) {
  return checl_checkpoint_incremental_ex(ctx, device, cuda_stream, epoch, base, CHECL_DIRTY_BYTES, out);
}

checl_status checl_checkpoint_incremental_ex(checl_ctx* ctx, int device, void* cuda_stream, uint64_t epoch,
                                             const checl_image* base, uint32_t dirty_rule, checl_image** out) {
  if (!ctx || !out || !base || !base->host || dirty_rule > CHECL_DIRTY_BYTES) return CHECL_ERR_INVALID_VALUE;
  if (!valid_device(device)) return CHECL_ERR_INVALID_DEVICE;
  checl_image* img = new (std::nothrow) checl_image();
  if (!img) return CHECL_ERR_OUT_OF_HOST_MEMORY;
  BusyGuard b(ctx);
  checl_status st = b.ok ? guarded([&]() {
    return do_checkpoint_incremental(ctx, device, cuda_stream, epoch, base, img, dirty_rule);
  })
                         : CHECL_ERR_BUSY;
  if (st) {
    checl_image_free(img);
    return st;
  }
  *out = img;
  return CHECL_SUCCESS;
}

checl_status checl_restore_chain(checl_ctx* ctx, const checl_image* const* chain, uint32_t n, int device,
                                 void* cuda_stream, checl_report* rep) {
  if (!ctx || !chain || n == 0) return CHECL_ERR_INVALID_VALUE;
  for (uint32_t i = 0; i < n; ++i)
    if (!chain[i]) return CHECL_ERR_INVALID_VALUE;
  if (!valid_device(device)) return CHECL_ERR_INVALID_DEVICE;
  if (n == 1) return checl_restore(ctx, chain[0], device, cuda_stream, rep);
  BusyGuard b(ctx);
  if (!b.ok) return CHECL_ERR_BUSY;
  return guarded([&]() { return do_restore_chain(ctx, chain, n, device, cuda_stream, rep); });
}

checl_status checl_image_merge(const checl_image* full, const checl_image* delta, checl_image** out) {
  if (!full || !delta || !out) return CHECL_ERR_INVALID_VALUE;
  if (full->location != CHECL_IMAGE_HOST || delta->location != CHECL_IMAGE_HOST) return CHECL_ERR_INVALID_VALUE;
  return guarded([&]() -> checl_status {
    Parsed Fp, Dp;
    checl_status st = parse_image(full->host, full->image_bytes, false, &Fp);
    if (!st) st = parse_image(delta->host, delta->image_bytes, false, &Dp);
    if (st) return st;
    if (Fp.flags != 0 || !linked(full, Fp, delta, Dp)) return CHECL_ERR_BAD_IMAGE;
    checl_image* m = new checl_image();
    try {
      m->ensure_host(Fp.L.image_bytes, false);
    } catch (...) {
      delete m;
      throw;
    }
    uint8_t* o = m->host_mut;
    // FORMAT.md "Merge": F's bytes; D's header with flags 0 and the full-image
    // fields; D's CRC table; every present chunk's span from D, in ascending order
    std::memcpy(o, full->host, Fp.L.image_bytes);
    std::memcpy(o, delta->host, kHeaderBytes);
    put_u32(o + 84, 0);
    put_u64(o + 56, Fp.L.payload_off);
    put_u64(o + 64, Fp.L.payload_bytes);
    put_u64(o + 72, Fp.L.image_bytes);
    std::memset(o + 96, 0, 28);
    std::memcpy(o + Fp.L.crc_off, delta->host + Dp.L.crc_off, 4 * Fp.L.n_chunks);
    const uint8_t* map = delta->host + Dp.map_off;
    uint64_t pos = Dp.L.payload_off;
    for (size_t b = 0; b < Fp.bufs.size(); ++b) {
      const uint64_t nb = chunks_of(Fp.bufs[b].size);
      for (uint64_t j = 0; j < nb; ++j) {
        if (!bit_set(map, Fp.bufs[b].first_chunk + j)) continue;
        uint64_t a, z;
        chunk_span(Fp.bufs, b, j, Fp.full_payload, &a, &z);
        std::memcpy(o + Fp.L.payload_off + a, delta->host + pos, z - a);
        pos += z - a;
      }
    }
    put_u32(o + 124, meta_crc(o, Fp.L.payload_off));
    m->image_bytes = Fp.L.image_bytes;
    m->payload_off = Fp.L.payload_off;
    *out = m;
    return CHECL_SUCCESS;
  });
}

// ---- delayed checkpointing mode (L16 §III-C) ----------------

namespace {
void on_checkpoint_signal(int signo) {  // async-signal-safe: one lock-free atomic store
  if (signo <= 0 || signo >= kMaxSignal) return;
  checl_ctx* c = g_signal_ctx[signo].load(std::memory_order_relaxed);
  if (c) c->requested.store(1, std::memory_order_relaxed);
}
}  // namespace

checl_status checl_request_checkpoint(checl_ctx* ctx) {
  if (!ctx) return CHECL_ERR_INVALID_VALUE;
  ctx->requested.store(1, std::memory_order_relaxed);
  return CHECL_SUCCESS;
}

checl_status checl_checkpoint_pending(const checl_ctx* ctx, int* pending) {
  if (!ctx || !pending) return CHECL_ERR_INVALID_VALUE;
  *pending = ctx->requested.load(std::memory_order_relaxed) ? 1 : 0;
  return CHECL_SUCCESS;
}

checl_status checl_install_signal(checl_ctx* ctx, int signo) {
  if (signo <= 0 || signo >= kMaxSignal || signo == SIGKILL || signo == SIGSTOP) return CHECL_ERR_INVALID_VALUE;
  struct sigaction sa;
  std::memset(&sa, 0, sizeof sa);
  sigemptyset(&sa.sa_mask);
  sa.sa_flags = SA_RESTART;
  sa.sa_handler = ctx ? on_checkpoint_signal : SIG_DFL;
  g_signal_ctx[signo].store(ctx);
  if (sigaction(signo, &sa, nullptr) != 0) {
    g_signal_ctx[signo].store(nullptr);
    return CHECL_ERR_INVALID_VALUE;
  }
  return CHECL_SUCCESS;
}

checl_status checl_sync_point(checl_ctx* ctx, int device, void* cuda_stream, uint64_t epoch, checl_image* reuse,
                              checl_image** out) {
  if (!ctx || !out) return CHECL_ERR_INVALID_VALUE;
  if (reuse && !reuse->owned) return CHECL_ERR_INVALID_VALUE;
  if (!valid_device(device)) return CHECL_ERR_INVALID_DEVICE;
  *out = nullptr;
  checl_status st = guarded([&]() -> checl_status {
    DeviceGuard g(device);
    ck(cudaStreamSynchronize(static_cast<cudaStream_t>(cuda_stream)));  // the clFinish the application asked for
    return CHECL_SUCCESS;
  });
  if (st) return st;
  if (!ctx->requested.exchange(0, std::memory_order_relaxed)) return CHECL_SUCCESS;
  if (reuse) {
    st = checl_checkpoint_into(ctx, device, cuda_stream, epoch, reuse);
    if (!st) *out = reuse;
  } else {
    st = checl_checkpoint(ctx, device, cuda_stream, epoch, out);
  }
  if (st) ctx->requested.store(1, std::memory_order_relaxed);  // still owed
  return st;
}

// ---- writing phase: image <-> file (L16 step 3 analogue; Table I) ----

namespace {
constexpr size_t kIoPiece = 64ull << 20;

bool write_all(int fd, const uint8_t* p, size_t n, uint64_t off) {
  while (n) {
    const ssize_t w = pwrite(fd, p, n, (off_t)off);
    if (w <= 0) return false;
    p += w;
    n -= (size_t)w;
    off += (uint64_t)w;
  }
  return true;
}

// Writes [p, p+n) at file offset `off`: the 4 KiB-multiple part through the O_DIRECT
// descriptor when both are usable (page-aligned source), the rest buffered.
bool write_span(int dfd, int bfd, const uint8_t* p, size_t n, uint64_t off) {
  size_t direct = 0;
  if (dfd >= 0 && (reinterpret_cast<uintptr_t>(p) & 4095u) == 0 && (off & 4095u) == 0) direct = n & ~(size_t)4095;
  if (direct && !write_all(dfd, p, direct, off)) return false;
  return write_all(bfd, p + direct, n - direct, off + direct);
}
}  // namespace

// Runs fn(lo, hi) over [0, n) split into up to kIoThreads 4 KiB-aligned pieces on
// parallel threads (one thread's memcpy into the page cache / tmpfs tops out at a few
// GB/s); true iff every piece succeeded.
extern "C++" {
constexpr int kIoThreads = 8;
template <typename F>
static bool parallel_io(uint64_t n, F fn) {
  const uint64_t per = std::max<uint64_t>(align_up((n + kIoThreads - 1) / kIoThreads, 4096), kIoPiece);
  std::vector<std::thread> th;
  std::atomic<bool> ok{true};
  for (uint64_t lo = 0; lo < n; lo += per) {
    const uint64_t hi = std::min(n, lo + per);
    th.emplace_back([&, lo, hi] {
      if (!fn(lo, hi)) ok.store(false);
    });
  }
  for (auto& t : th) t.join();
  return ok.load();
}
}  // extern "C++"

checl_status checl_image_write(const checl_image* img, const char* path, uint32_t flags) {
  if (!img || !path || flags & ~3u) return CHECL_ERR_INVALID_VALUE;
  return guarded([&]() -> checl_status {
    // (read-write: a MAP_SHARED PROT_WRITE mapping needs a descriptor opened for reading too)
    const int bfd = ::open(path, O_RDWR | O_CREAT | O_TRUNC, 0644);
    if (bfd < 0) return CHECL_ERR_INVALID_VALUE;
    int dfd = (flags & CHECL_IO_DIRECT) ? ::open(path, O_WRONLY | O_DIRECT) : -1;
    bool ok = true;
    if (img->location == CHECL_IMAGE_HOST && img->image_bytes) {
      const bool direct = dfd >= 0 && (reinterpret_cast<uintptr_t>(img->host) & 4095u) == 0;
      // blocks allocated up front: the parallel pieces overwrite in place, and a page
      // fault of the shared mapping below cannot run out of space (ENOSPC inside a
      // mapping is SIGBUS, not an error return). Without the reservation the file is
      // written with pwrite, whose errors come back as INVALID_VALUE.
      const bool reserved = posix_fallocate(bfd, 0, (off_t)img->image_bytes) == 0;
      if (!reserved) ok = ::ftruncate(bfd, (off_t)img->image_bytes) == 0;
      void* map = MAP_FAILED;
      if (ok && !direct && reserved) map = ::mmap(nullptr, img->image_bytes, PROT_WRITE, MAP_SHARED, bfd, 0);
      if (!ok) {
      } else if (map != MAP_FAILED) {
        // page-cache / tmpfs target: parallel copies into the shared mapping (write(2)
        // on one file serialises on the inode lock; page faults of a mapping do not)
        uint8_t* m = static_cast<uint8_t*>(map);
        parallel_io(img->image_bytes, [&](uint64_t lo, uint64_t hi) {
          std::memcpy(m + lo, img->host + lo, hi - lo);
          return true;
        });
        if (flags & CHECL_IO_SYNC) ok = ::msync(map, img->image_bytes, MS_SYNC) == 0;
        ::munmap(map, img->image_bytes);
      } else {
        ok = parallel_io(img->image_bytes, [&](uint64_t lo, uint64_t hi) {
          for (uint64_t o = lo; o < hi; o += kIoPiece)
            if (!write_span(dfd, bfd, img->host + o, std::min<uint64_t>(kIoPiece, hi - o), o)) return false;
          return true;
        });
      }
    } else if (img->location == CHECL_IMAGE_DEVICE) {
      // device image: the host mirror, then the payload through a pinned bounce buffer
      ok = write_span(dfd, bfd, img->host, img->payload_off, 0);
      DeviceGuard g(img->device);
      PinnedBuf<uint8_t> bounce;
      const uint64_t pay = img->image_bytes - img->payload_off;
      bounce.ensure(std::min<uint64_t>(kIoPiece, std::max<uint64_t>(pay, 1)));
      for (uint64_t o = 0; ok && o < pay; o += kIoPiece) {
        const uint64_t n = std::min<uint64_t>(kIoPiece, pay - o);
        ck(cudaMemcpy(bounce.p, img->d_payload + o, n, cudaMemcpyDeviceToHost));
        ok = write_span(dfd, bfd, bounce.p, n, img->payload_off + o);
      }
      bounce.release();
    }
    if (ok && (flags & CHECL_IO_SYNC)) ok = ::fsync(bfd) == 0;
    if (dfd >= 0) ::close(dfd);
    if (::close(bfd) != 0) ok = false;
    return ok ? CHECL_SUCCESS : CHECL_ERR_INVALID_VALUE;
  });
}

checl_status checl_image_read(const char* path, uint32_t flags, checl_image** out) {
  if (!path || !out || flags & ~1u) return CHECL_ERR_INVALID_VALUE;
  return guarded([&]() -> checl_status {
    struct stat sb;
    if (::stat(path, &sb) != 0 || sb.st_size < (off_t)kHeaderBytes) return CHECL_ERR_BAD_IMAGE;
    const uint64_t size = (uint64_t)sb.st_size, cap = pinned_class(align_up(size, 4096));
    checl_image* img = new checl_image();
    void* p = nullptr;
    size_t pcap = cap;
    // pinned when a device is present (restore then fills over PCIe at full rate)
    if (device_count() > 0 && ((p = pinned_pool().take(cap, &pcap)) != nullptr || (p = pin_alloc(cap)) != nullptr)) {
      img->pinned = true;
    } else {
      cudaGetLastError();
      p = nullptr;
      if (posix_memalign(&p, 4096, cap) != 0) {
        delete img;
        throw std::bad_alloc();
      }
      img->pinned = false;
    }
    img->owned = true;
    img->host = img->host_mut = static_cast<uint8_t*>(p);
    img->host_cap = img->pinned ? pcap : cap;
    int fd = (flags & CHECL_IO_DIRECT) ? ::open(path, O_RDONLY | O_DIRECT) : -1;
    if (fd < 0) fd = ::open(path, O_RDONLY);
    bool ok = fd >= 0 && parallel_io(size, [&](uint64_t lo, uint64_t hi) {
      // pieces start 4 KiB-aligned; the last one may read up to `cap` (aligned length)
      const uint64_t end = hi == size ? cap : hi;
      for (uint64_t o = lo; o < hi;) {
        const ssize_t r = pread(fd, img->host_mut + o, (size_t)std::min<uint64_t>(kIoPiece, end - o), (off_t)o);
        if (r <= 0) return false;
        o += (uint64_t)r;
      }
      return true;
    });
    if (fd >= 0) ::close(fd);
    Parsed P;
    checl_status st = ok ? parse_image(img->host, size, false, &P) : CHECL_ERR_BAD_IMAGE;
    if (st) {
      img->free_host();
      delete img;
      return st;
    }
    img->image_bytes = P.L.image_bytes;
    img->payload_off = P.L.payload_off;
    *out = img;
    return CHECL_SUCCESS;
  });
}

checl_status checl_trim(checl_ctx* ctx) {
  if (!ctx) return CHECL_ERR_INVALID_VALUE;
  return guarded([&]() -> checl_status {
    std::vector<std::shared_ptr<Arena>> drop;
    {
      std::lock_guard<std::mutex> lk(ctx->mu);
      for (int d = 0; d < kMaxDevices; ++d) {
        for (auto& a : ctx->spares[d]) drop.push_back(std::move(a));
        ctx->spares[d].clear();
      }
    }
    free_arenas(drop);
    // the exact incremental rule's device copy of the last delta's state: the next exact
    // delta reseeds it from a full base, or writes a full image (reading 25)
    BusyGuard b(ctx);
    if (b.ok)
      for (DevState* ds : ctx->devs)
        if (ds && ds->shadow.p) {
          DeviceGuard g(ds->dev);
          ck(cudaDeviceSynchronize());
          ds->shadow.release();
          ds->shadow_ok = false;
        }
    pinned_pool().trim();
    return CHECL_SUCCESS;
  });
}

checl_status checl_last_timing(const checl_ctx* ctx, checl_timing* out) {
  if (!ctx || !out) return CHECL_ERR_INVALID_VALUE;
  settle(ctx);
  std::lock_guard<std::mutex> lk(ctx->tmu);
  *out = ctx->last;
  return CHECL_SUCCESS;
}

checl_status checl_stats_get(const checl_ctx* ctx, int kind, checl_stats* out) {
  if (!ctx || !out || kind < 0 || kind >= CHECL_STATS_KINDS) return CHECL_ERR_INVALID_VALUE;
  settle(ctx);
  std::lock_guard<std::mutex> lk(ctx->tmu);
  *out = ctx->stats[kind];
  return CHECL_SUCCESS;
}

checl_status checl_stats_reset(checl_ctx* ctx) {
  if (!ctx) return CHECL_ERR_INVALID_VALUE;
  settle(ctx);
  std::lock_guard<std::mutex> lk(ctx->tmu);
  for (auto& st : ctx->stats) st = checl_stats{};
  return CHECL_SUCCESS;
}

const char* checl_status_string(checl_status s) {
  switch (s) {
    case CHECL_SUCCESS: return "CHECL_SUCCESS";
    case CHECL_ERR_INVALID_VALUE: return "CHECL_ERR_INVALID_VALUE";
    case CHECL_ERR_INVALID_HANDLE: return "CHECL_ERR_INVALID_HANDLE";
    case CHECL_ERR_INVALID_DEVICE: return "CHECL_ERR_INVALID_DEVICE";
    case CHECL_ERR_OUT_OF_DEVICE_MEMORY: return "CHECL_ERR_OUT_OF_DEVICE_MEMORY";
    case CHECL_ERR_OUT_OF_HOST_MEMORY: return "CHECL_ERR_OUT_OF_HOST_MEMORY";
    case CHECL_ERR_BAD_IMAGE: return "CHECL_ERR_BAD_IMAGE";
    case CHECL_ERR_CRC_MISMATCH: return "CHECL_ERR_CRC_MISMATCH";
    case CHECL_ERR_CUDA: return "CHECL_ERR_CUDA";
    case CHECL_ERR_PEER_ACCESS: return "CHECL_ERR_PEER_ACCESS";
    case CHECL_ERR_BUSY: return "CHECL_ERR_BUSY";
    default: return "CHECL_ERR_UNKNOWN";
  }
}

const char* checl_last_cuda_error(void) { return t_last_cuda_error.c_str(); }

uint32_t checl_version(void) { return 0x00010000u; }

checl_status checl_debug_fill(int device, void* dev_ptr, size_t bytes, uint64_t seed, uint64_t stream_id, int kind,
                              void* cuda_stream) {
  if ((!dev_ptr && bytes) || kind < 0 || kind > 2) return CHECL_ERR_INVALID_VALUE;
  if (!valid_device(device)) return CHECL_ERR_INVALID_DEVICE;
  return guarded([&]() -> checl_status {
    DeviceGuard g(device);
    int sms = 0;
    ck(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device));
    auto mix = [](uint64_t z) {
      z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
      z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
      return z ^ (z >> 31);
    };
    const uint64_t key = mix((seed * 0x9E3779B97F4A7C15ull) ^ ((stream_id + 1) * 0xD1B54A32D192ED03ull));
    ck(launch_fill(static_cast<uint8_t*>(dev_ptr), bytes, key, kind, sms, static_cast<cudaStream_t>(cuda_stream)));
    return CHECL_SUCCESS;
  });
}

checl_status checl_debug_compare(int device, const void* a, const void* b, size_t bytes, uint64_t* n_diff) {
  if (!n_diff || ((!a || !b) && bytes)) return CHECL_ERR_INVALID_VALUE;
  if (!valid_device(device)) return CHECL_ERR_INVALID_DEVICE;
  return guarded([&]() -> checl_status {
    DeviceGuard g(device);
    int sms = 0;
    ck(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device));
    unsigned long long* d = nullptr;
    ck(cudaMalloc(&d, 8));
    unsigned long long h = 0;
    cudaError_t e = cudaMemset(d, 0, 8);
    if (e == cudaSuccess)
      e = launch_compare(static_cast<const uint8_t*>(a), static_cast<const uint8_t*>(b), bytes, d, sms, nullptr);
    if (e == cudaSuccess) e = cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
    cudaFree(d);
    ck(e);
    *n_diff = h;
    return CHECL_SUCCESS;
  });
}

checl_status checl_debug_corrupt(checl_image* img, uint64_t image_offset, uint8_t mask) {
  if (!img) return CHECL_ERR_INVALID_VALUE;
  if (image_offset >= img->image_bytes) return CHECL_ERR_INVALID_VALUE;
  return guarded([&]() -> checl_status {
    if (img->location == CHECL_IMAGE_DEVICE && image_offset >= img->payload_off) {
      DeviceGuard g(img->device);
      uint8_t* p = img->d_payload + (image_offset - img->payload_off);
      uint8_t v = 0;
      ck(cudaMemcpy(&v, p, 1, cudaMemcpyDeviceToHost));
      v ^= mask;
      ck(cudaMemcpy(p, &v, 1, cudaMemcpyHostToDevice));
      return CHECL_SUCCESS;
    }
    if (!img->owned) return CHECL_ERR_INVALID_VALUE;  // wrapped bytes are the caller's
    img->host_mut[image_offset] ^= mask;
    img->meta_valid = false;  // (the next checkpoint into it rewrites its manifest)
    return CHECL_SUCCESS;
  });
}

}  // extern "C"
