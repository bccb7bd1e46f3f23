// K3/K4/K5: copy kernels of the migration engine (DESIGN.md §6 "migrate").
//
// One kernel serves every byte move of a transition that is not a plain DMA:
//   K3 gather-pack   scattered arena ranges -> contiguous device staging (then one DMA D2H)
//   K4 scatter-unpack contiguous staging -> scattered arena ranges (compaction, R11/R12)
//   K5 zero-copy     arena <-> pinned *mapped* host memory over PCIe (small tensors: one launch
//                    replaces one DMA per tensor; measured 51-54 GB/s vs 1 GB/s for 4 KiB DMAs)
//   D2D carry        half 1-m -> half m (R8)
// The host splits every segment into work items of <= `chunk` bytes; CTAs take items in a
// grid-stride loop and move them with 16-byte vector loads/stores, 4 in flight per thread.
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdlib>
#include <cstring>

#include "dyo_internal.h"

namespace dyo {

constexpr int kCopyThreads = 512;

__global__ void __launch_bounds__(kCopyThreads)
copy_segments_kernel(const CopySeg* __restrict__ segs, int n) {
  for (int it = blockIdx.x; it < n; it += gridDim.x) {
    const CopySeg sg = segs[it];
    const char* src = sg.src;
    char* dst = sg.dst;
    const int64_t nbytes = sg.bytes;
    const bool vec = ((((uintptr_t)src) | ((uintptr_t)dst)) & 15) == 0;
    int64_t done = 0;
    if (vec) {
      const int64_t n16 = nbytes >> 4;
      const int4* s4 = reinterpret_cast<const int4*>(src);
      int4* d4 = reinterpret_cast<int4*>(dst);
      const int64_t stride = blockDim.x;
      int64_t i = threadIdx.x;
      for (; i + 3 * stride < n16; i += 4 * stride) {
        const int4 v0 = s4[i], v1 = s4[i + stride], v2 = s4[i + 2 * stride], v3 = s4[i + 3 * stride];
        d4[i] = v0;
        d4[i + stride] = v1;
        d4[i + 2 * stride] = v2;
        d4[i + 3 * stride] = v3;
      }
      for (; i < n16; i += stride) d4[i] = s4[i];
      done = n16 << 4;
    }
    for (int64_t i = done + threadIdx.x; i < nbytes; i += blockDim.x) dst[i] = src[i];
  }
}

// ---- TMA bulk variant (device<->device moves: pack / unpack / carry / compaction) ----------
// One elected thread per CTA streams its work items through a ring of kTmaStages shared-memory
// buffers: cp.async.bulk global->shared (mbarrier complete_tx), then cp.async.bulk
// shared->global (bulk_group); a buffer is reused only after its store has read it
// (cp.async.bulk.wait_group.read). The copy engine of the SM does the byte moving, so a few
// CTAs saturate HBM and the SMs stay free for the DyNN's compute. Unaligned heads/tails (not
// multiples of 16 bytes) are copied by the CTA's threads.
// Ring shapes (stages x chunk): 4 x 16 KiB lets three copy kernels share an SM; the deeper rings
// keep more bytes in flight per SM when one copy kernel has the GPU (DYO_TMA_RING selects, for
// measurement; DESIGN.md §6 records which one is the default and why).
constexpr int kTmaStages = 4;
constexpr int kTmaChunk = 16 << 10;

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

// The device<->device moves of a transition are driven straight from the plan's records, which
// the planner left in device memory: the host never builds or ships work items for them (it
// would have to send them over a PCIe link that the transition's own DMAs keep saturated in
// both directions; measured: a zero-copy descriptor read under that load stretched 220 MB
// launches from ~40 to 100-150 us).
//
// Records i < n (filtered by `late` when f_late >= 0) define copies
//   src_base + rec[i][f_src]  ->  dst_base + rec[i][f_dst] - dst_bias,  rec[i][f_bytes] bytes.
// Each record's 16-byte-aligned body (0 when src or dst is not 16-byte aligned) is a piece of
// one virtual stream of `total` bytes; CTA b copies the contiguous slice [b*per, (b+1)*per) of
// it (per = total/grid rounded up to 16 bytes), so one large record spreads over every SM. The
// remaining < 16-byte tails (and unaligned records) are copied by the CTAs' threads.

constexpr int kRecThreads = 128;
constexpr unsigned long long kStampCap = (1ull << 22) - 1;   // DYO_COPY_STAMPS log entries

template <int CHUNK>
struct RecCursor {
  const RecCopyArgs* a;
  int i;                       // current record
  int64_t off, body, pos, hi;  // offset in its body; position in the stream; slice end
  const char* src;
  char* dst;
  __device__ int64_t body_of(int k, const char** s, char** d) const {
    const int64_t* r = a->rec + (int64_t)k * a->stride;
    if (a->f_late >= 0 && r[a->f_late] != a->late_val) return 0;
    *s = a->src_base + r[a->f_src];
    *d = a->dst_base + (r[a->f_dst] - a->dst_bias);
    const bool al = ((((uintptr_t)*s) | ((uintptr_t)*d)) & 15) == 0;
    return al ? (r[a->f_bytes] & ~(int64_t)15) : 0;
  }
  __device__ void settle() {   // skip exhausted / empty records
    while (pos < hi && off >= body) {
      ++i;
      off = 0;
      body = i < a->n ? body_of(i, &src, &dst) : 0;
      if (i >= a->n) { pos = hi; return; }
    }
  }
  __device__ void init(const RecCopyArgs* aa, int i0, int64_t off0, int64_t lo, int64_t hi_) {
    a = aa; i = i0; off = off0; pos = lo; hi = hi_;
    if (a->rec == nullptr) { src = a->src_base; dst = a->dst_base; body = hi_; off = lo; return; }
    body = (i < a->n) ? body_of(i, &src, &dst) : 0;
    settle();
  }
  __device__ bool valid() const { return pos < hi; }
  __device__ uint32_t len() const {
    int64_t l = body - off;
    if (hi - pos < l) l = hi - pos;
    return (uint32_t)(l < CHUNK ? l : CHUNK);
  }
  __device__ void next() {
    const uint32_t l = len();
    off += l;
    pos += l;
    if (a->rec != nullptr) settle();
  }
};

// Grid barrier of a cooperative multi-wave launch: every CTA's copies of the wave have read
// their sources (the elected thread waited for its bulk stores, the threads' byte tails are
// done) before any CTA starts the next wave, whose destinations may overlap them (a compaction
// wave ends where a later move's destination meets an earlier move's source).
__device__ __forceinline__ void copy_grid_barrier(unsigned int* ctr, unsigned int target) {
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    atomicAdd(ctr, 1u);
    unsigned int v;
    do {
      asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory");
    } while ((int)(v - target) < 0);
  }
  __syncthreads();
}

template <int kTmaStages, int kTmaChunk>
__global__ void __launch_bounds__(kRecThreads)
copy_records_tma_kernel(const __grid_constant__ RecCopyArgs args) {
  extern __shared__ __align__(128) unsigned char sbuf[];
  __shared__ __align__(8) uint64_t bar[kTmaStages];
  __shared__ int64_t wsum[kRecThreads / 32];
  __shared__ int s_i0;
  __shared__ int64_t s_off0;
  constexpr int L = kTmaStages - 1;          // loads kept in flight ahead of the store cursor
  unsigned long long t_enter = 0, t_scan = 0;
  if (args.stamps != nullptr && threadIdx.x == 0) asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_enter));
  const int nwaves = args.n_waves > 1 ? args.n_waves : 1;
  for (int wv = 0; wv < nwaves; ++wv) {
  RecCopyArgs aw = args;
  if (nwaves > 1) {
    const int r0 = wv ? args.wave_end[wv - 1] : 0;
    aw.rec = args.rec + (int64_t)r0 * args.stride;
    aw.n = args.wave_end[wv] - r0;
    aw.total = args.wave_total[wv];
  }
  const RecCopyArgs* a = &aw;
  // the stream: the records' bodies, or the single range's body (0 when unaligned)
  const bool single = a->rec == nullptr;
  const int64_t T = !single ? a->total
                  : (((((uintptr_t)a->src_base) | ((uintptr_t)a->dst_base)) & 15) == 0 ? a->total & ~(int64_t)15 : 0);
  int64_t per = (T + gridDim.x - 1) / gridDim.x;
  per = (per + 15) & ~(int64_t)15;
  const int64_t lo = (int64_t)blockIdx.x * per;
  const int64_t hi = lo + per < T ? lo + per : T;

  // the record holding stream position lo: exclusive scan of the bodies, a tile at a time
  if (threadIdx.x == 0) { s_i0 = a->n; s_off0 = 0; }
  __syncthreads();
  if (a->rec != nullptr && lo < hi) {
    int64_t carry = 0;
    for (int t0 = 0; t0 < a->n; t0 += blockDim.x) {
      const int k = t0 + threadIdx.x;
      int64_t v = 0;
      if (k < a->n) { const char* s_; char* d_; RecCursor<kTmaChunk> c; c.a = a; v = c.body_of(k, &s_, &d_); }
      const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
      int64_t x = v;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int64_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
      }
      if (lane == 31) wsum[w] = x;
      __syncthreads();
      int64_t before = carry, tile = 0;
      for (int q = 0; q < (int)(blockDim.x >> 5); ++q) {
        if (q < w) before += wsum[q];
        tile += wsum[q];
      }
      const int64_t start = before + x - v;   // exclusive prefix of record k
      if (k < a->n && v > 0 && start <= lo && lo < start + v) { s_i0 = k; s_off0 = lo - start; }
      carry += tile;
      __syncthreads();
      if (s_i0 < a->n || carry > lo) break;   // found (uniform: shared flag / uniform carry)
    }
  }

  if (a->stamps != nullptr && threadIdx.x == 0) asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_scan));
  if (threadIdx.x == 0 && lo < hi) {
    for (int q = 0; q < kTmaStages; ++q)
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar[q])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    RecCursor<kTmaChunk> lc, sc;
    lc.init(a, s_i0, s_off0, lo, hi);
    sc.init(a, s_i0, s_off0, lo, hi);
    auto issue_load = [&](uint32_t k) {
      const uint32_t st = k % kTmaStages;
      const uint32_t len = lc.len();
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar[st])), "r"(len) : "memory");
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                   ::"r"(su32(sbuf + st * kTmaChunk)), "l"(lc.src + lc.off), "r"(len), "r"(su32(&bar[st])) : "memory");
      lc.next();
    };
    uint32_t issued = 0;
    for (; issued < (uint32_t)L && lc.valid(); ++issued) issue_load(issued);
    for (uint32_t k = 0; sc.valid(); ++k) {
      const uint32_t st = k % kTmaStages;
      const uint32_t par = (k / kTmaStages) & 1;
      asm volatile("{\n.reg .pred P1;\nWAIT_%=:\nmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n@!P1 bra WAIT_%=;\n}\n"
                   ::"r"(su32(&bar[st])), "r"(par) : "memory");
      asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(sc.dst + sc.off),
                   "r"(su32(sbuf + st * kTmaChunk)), "r"(sc.len()) : "memory");
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      sc.next();
      if (lc.valid()) {
        // the next load reuses the buffer of chunk issued+1-kTmaStages = k: wait until every
        // store but the newest kTmaStages-L ones has read its buffer
        asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(kTmaStages - L) : "memory");
        issue_load(issued++);
      }
    }
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    // the next wave initialises the barriers again
    for (int q = 0; q < kTmaStages; ++q) asm volatile("mbarrier.inval.shared::cta.b64 [%0];" ::"r"(su32(&bar[q])) : "memory");
  }
  // < 16-byte tails and unaligned records: byte copies, record k by CTA k % grid
  if (single) {
    for (int64_t x = T + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; x < a->total; x += (int64_t)gridDim.x * blockDim.x)
      a->dst_base[x] = a->src_base[x];
  } else {
    for (int k = blockIdx.x; k < a->n; k += gridDim.x) {
      const int64_t* r = a->rec + (int64_t)k * a->stride;
      if (a->f_late >= 0 && r[a->f_late] != a->late_val) continue;
      const char* sp = a->src_base + r[a->f_src];
      char* dp = a->dst_base + (r[a->f_dst] - a->dst_bias);
      const int64_t nb = r[a->f_bytes];
      const bool al = ((((uintptr_t)sp) | ((uintptr_t)dp)) & 15) == 0;
      for (int64_t x = (al ? nb & ~(int64_t)15 : 0) + threadIdx.x; x < nb; x += blockDim.x) dp[x] = sp[x];
    }
  }
  if (wv + 1 < nwaves) copy_grid_barrier(args.gbar, args.gbar_base + (unsigned)(wv + 1) * gridDim.x);
  }   // waves
  const RecCopyArgs* a = &args;
  // exit stamp after every copy of the CTA, the byte tails included
  if (a->stamps != nullptr) {
    __syncthreads();
    if (threadIdx.x == 0) {
      unsigned long long t_end, slot;
      uint32_t smid;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_end));
      asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
      slot = atomicAdd(a->stamps, 1ull);
      if (slot < kStampCap) {
        unsigned long long* e = a->stamps + 4 * (slot + 1);
        e[0] = ((unsigned long long)a->launch << 32) | ((unsigned long long)blockIdx.x << 8) | (smid & 255u);
        e[1] = t_enter; e[2] = t_scan; e[3] = t_end;
      }
    }
  }
}

template <int S, int C>
static cudaError_t launch_ring(const RecCopyArgs& a, int grid, cudaStream_t s, int* grid_used) {
  static uint64_t attr_done = 0;                  // bit d: attributes set on device d
  const uint64_t bit = 1ull << current_device();
  const int smem = S * C;
  if (!(attr_done & bit)) {
    cudaError_t e = cudaFuncSetAttribute(copy_records_tma_kernel<S, C>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    // DYO_TMA_CARVEOUT=1: ask for the maximum shared-memory carveout (measurement of whether a
    // carveout change between this kernel and its neighbours delays its start)
    if (const char* v = getenv("DYO_TMA_CARVEOUT"))
      if (v[0] == '1') {
        e = cudaFuncSetAttribute(copy_records_tma_kernel<S, C>, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
        if (e != cudaSuccess) return e;
      }
    attr_done |= bit;
  }
  if (a.n_waves > 1) {
    // multi-wave: the whole grid, co-resident (cooperative launch) for the grid barriers
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(kRecThreads);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeCooperative;
    at[0].val.cooperative = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    if (grid_used) *grid_used = grid;
    return cudaLaunchKernelEx(&cfg, copy_records_tma_kernel<S, C>, a);
  }
  // at least one chunk per CTA; enough CTAs for the tail loop over the records
  int64_t g = (a.total + C - 1) / C;
  if (a.rec != nullptr && g < a.n) g = a.n;
  if (g > grid) g = grid;
  if (g < 1) g = 1;
  if (grid_used) *grid_used = (int)g;
  copy_records_tma_kernel<S, C><<<(int)g, kRecThreads, smem, s>>>(a);
  return cudaGetLastError();
}

// DYO_TMA_RING = "4x16" (default) | "8x16" | "4x32" | "6x32" | "3x64" (stages x KiB)
static int tma_ring() {
  static int r = -1;
  if (r < 0) {
    r = 0;
    if (const char* e = getenv("DYO_TMA_RING")) {
      const char* names[] = {"4x16", "8x16", "4x32", "6x32", "3x64"};
      for (int q = 0; q < 5; ++q)
        if (strcmp(e, names[q]) == 0) r = q;
    }
  }
  return r;
}

// DYO_TMA_CTAS_PER_SM = 1 (default) | 2 | 3: CTAs per SM of the record copy grid
static int tma_ctas_per_sm() {
  static int c = 0;
  if (c == 0) {
    c = 1;
    if (const char* e = getenv("DYO_TMA_CTAS_PER_SM")) c = atoi(e) >= 2 && atoi(e) <= 3 ? atoi(e) : 1;
  }
  return c;
}

// DYO_COPY_STAMPS=1 (measurement aid): every record-copy CTA appends {launch<<32 | cta<<8 | smid,
// globaltimer at entry, after the record scan, at the end} to a device log (slot 0 = count; up to
// 2^22 - 1 entries), read back by dyo_debug_copy_stamps.
// The log is per device (a process may drive several GPUs, one ctx each).
static unsigned long long* g_stamps_dev[64] = {};
static unsigned long long*& stamps_of_current_device() { return g_stamps_dev[current_device()]; }

// DYO_COPY_STAMPS=2 also brackets each record-copy launch with a one-thread marker kernel on the
// same stream (entry cta field 0xFFF, smid field 0 = before, 1 = after): it locates the time
// between the CUDA events and the copy kernel's CTAs.
__global__ void copy_mark_kernel(unsigned long long* stamps, int64_t launch, int which) {
  unsigned long long t, slot;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  slot = atomicAdd(stamps, 1ull);
  if (slot < kStampCap) {
    unsigned long long* e = stamps + 4 * (slot + 1);
    e[0] = ((unsigned long long)launch << 32) | (0xFFFull << 8) | (unsigned)which;
    e[1] = t; e[2] = t; e[3] = t;
  }
}
static int64_t g_launch = 0;
int64_t copy_stamps_read(unsigned long long* host, int64_t cap) {
  unsigned long long* g_stamps = stamps_of_current_device();
  if (g_stamps == nullptr) return 0;
  if (host == nullptr && cap == 0) return cudaMemset(g_stamps, 0, 8) == cudaSuccess ? 0 : -1;   // reset
  unsigned long long n = 0;
  if (cudaMemcpy(&n, g_stamps, 8, cudaMemcpyDeviceToHost) != cudaSuccess) return -1;
  if (n > kStampCap) n = kStampCap;
  if ((int64_t)n > cap) n = (unsigned long long)cap;
  if (host != nullptr && n > 0 &&
      cudaMemcpy(host, g_stamps + 4, n * 32, cudaMemcpyDeviceToHost) != cudaSuccess) return -1;
  return (int64_t)n;
}

cudaError_t launch_copy_records(const RecCopyArgs& a0, int grid, cudaStream_t s, int* grid_used) {
  if (a0.total <= 0 && (a0.rec == nullptr || a0.n <= 0)) return cudaSuccess;
  RecCopyArgs a = a0;
  static int stamps_on = -1;
  if (stamps_on < 0) {
    const char* e = getenv("DYO_COPY_STAMPS");
    stamps_on = (e != nullptr && (e[0] == '1' || e[0] == '2')) ? (e[0] - '0') : 0;
  }
  unsigned long long*& g_stamps = stamps_of_current_device();
  if (stamps_on && g_stamps == nullptr) {
    if (cudaMalloc(&g_stamps, (size_t)32 * (kStampCap + 1)) != cudaSuccess) return cudaGetLastError();
    cudaMemset(g_stamps, 0, 8);
  }
  if (stamps_on) { a.stamps = g_stamps; a.launch = g_launch++; }
  if (stamps_on == 2) copy_mark_kernel<<<1, 1, 0, s>>>(g_stamps, a.launch, 0);
  grid *= tma_ctas_per_sm();
  cudaError_t e;
  switch (tma_ring()) {
    case 1: e = launch_ring<8, 16 << 10>(a, grid, s, grid_used); break;
    case 2: e = launch_ring<4, 32 << 10>(a, grid, s, grid_used); break;
    case 3: e = launch_ring<6, 32 << 10>(a, grid, s, grid_used); break;
    case 4: e = launch_ring<3, 64 << 10>(a, grid, s, grid_used); break;
    default: e = launch_ring<kTmaStages, kTmaChunk>(a, grid, s, grid_used); break;
  }
  if (e == cudaSuccess && stamps_on == 2) {
    copy_mark_kernel<<<1, 1, 0, s>>>(g_stamps, a.launch, 1);
    e = cudaGetLastError();
  }
  return e;
}

cudaError_t launch_copy_segments(const CopySeg* segs, int n, int64_t /*chunk*/, int grid,
                                 cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  if (grid > n) grid = n;
  copy_segments_kernel<<<grid, kCopyThreads, 0, s>>>(segs, n);
  return cudaGetLastError();
}

}  // namespace dyo
