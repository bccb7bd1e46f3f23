// K3/K4/K5: segment-list copy kernels (DESIGN.md §6 "migrate").
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
// One elected thread per CTA streams each work item through a ring of kStages shared-memory
// buffers: cp.async.bulk global->shared (mbarrier complete_tx), then cp.async.bulk
// shared->global (bulk_group); a buffer is reused only after its store has read it
// (cp.async.bulk.wait_group.read). The copy engine of the SM does the byte moving, so a few
// CTAs saturate HBM and the SMs stay free for the DyNN's compute. Unaligned heads/tails (not
// multiples of 16 bytes) are copied by the CTA's threads.
constexpr int kTmaStages = 4;
constexpr int kTmaChunk = 32 << 10;

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

// A cursor over the 32 KiB chunks of this CTA's work items (items blockIdx.x, +gridDim.x, ...;
// only their 16-byte-aligned bodies).
struct ChunkCursor {
  const CopySeg* segs;
  int n, it;
  int64_t off, body;
  const char* src;
  char* dst;
  __device__ void load_item() {
    while (it < n) {
      const CopySeg sg = segs[it];
      src = sg.src;
      dst = sg.dst;
      const bool aligned = ((((uintptr_t)src) | ((uintptr_t)dst)) & 15) == 0;
      body = aligned ? (sg.bytes & ~(int64_t)15) : 0;
      if (body > 0) return;
      it += gridDim.x;
    }
  }
  __device__ void init(const CopySeg* s, int nn) { segs = s; n = nn; it = blockIdx.x; off = 0; load_item(); }
  __device__ bool valid() const { return it < n; }
  __device__ uint32_t len() const { return (uint32_t)((body - off) < kTmaChunk ? (body - off) : kTmaChunk); }
  __device__ void next() {
    off += kTmaChunk;
    if (off >= body) { it += gridDim.x; off = 0; load_item(); }
  }
};

__global__ void __launch_bounds__(128)
copy_segments_tma_kernel(const CopySeg* __restrict__ segs, int n) {
  extern __shared__ __align__(128) unsigned char sbuf[];
  __shared__ __align__(8) uint64_t bar[kTmaStages];
  constexpr int L = kTmaStages - 1;          // loads kept in flight ahead of the store cursor
  if (threadIdx.x == 0) {
    for (int i = 0; i < kTmaStages; ++i)
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar[i])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    ChunkCursor lc, sc;
    lc.init(segs, n);
    sc.init(segs, n);
    auto issue_load = [&](int k) {
      const int st = k % kTmaStages;
      const uint32_t len = lc.len();
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar[st])), "r"(len) : "memory");
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                   ::"r"(su32(sbuf + st * kTmaChunk)), "l"(lc.src + lc.off), "r"(len), "r"(su32(&bar[st])) : "memory");
      lc.next();
    };
    int issued = 0;
    for (; issued < L && lc.valid(); ++issued) issue_load(issued);
    for (int k = 0; sc.valid(); ++k) {
      const int st = k % kTmaStages;
      const uint32_t par = (uint32_t)((k / kTmaStages) & 1);
      asm volatile("{\n.reg .pred P1;\nWAIT_%=:\nmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n@!P1 bra WAIT_%=;\n}\n"
                   ::"r"(su32(&bar[st])), "r"(par) : "memory");
      asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(sc.dst + sc.off),
                   "r"(su32(sbuf + st * kTmaChunk)), "r"(sc.len()) : "memory");
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      sc.next();
      if (lc.valid()) {
        // the next load reuses the buffer of chunk issued+1-kTmaStages = k: wait until every
        // store but the newest one (chunk k's, L - ... >= that) has read its buffer
        asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(kTmaStages - L) : "memory");
        issue_load(issued++);
      }
    }
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
  // unaligned items and the < 16-byte tails: plain byte copies by the CTA's threads
  for (int it = blockIdx.x; it < n; it += gridDim.x) {
    const CopySeg sg = segs[it];
    const bool aligned = ((((uintptr_t)sg.src) | ((uintptr_t)sg.dst)) & 15) == 0;
    const int64_t body = aligned ? (sg.bytes & ~(int64_t)15) : 0;
    for (int64_t i = body + threadIdx.x; i < sg.bytes; i += blockDim.x) sg.dst[i] = sg.src[i];
  }
}

cudaError_t launch_copy_segments_tma(const CopySeg* segs, int n, int grid, cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  static bool attr = false;
  const int smem = kTmaStages * kTmaChunk;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(copy_segments_tma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  if (grid > n) grid = n;
  copy_segments_tma_kernel<<<grid, 128, smem, s>>>(segs, n);
  return cudaGetLastError();
}

cudaError_t launch_copy_segments(const CopySeg* segs, int n, int64_t /*chunk*/, int grid,
                                 cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  if (grid > n) grid = n;
  copy_segments_kernel<<<grid, kCopyThreads, 0, s>>>(segs, n);
  return cudaGetLastError();
}

}  // namespace dyo
