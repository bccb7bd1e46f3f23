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

cudaError_t launch_copy_segments(const CopySeg* segs, int n, int64_t /*chunk*/, int grid,
                                 cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  if (grid > n) grid = n;
  copy_segments_kernel<<<grid, kCopyThreads, 0, s>>>(segs, n);
  return cudaGetLastError();
}

}  // namespace dyo
