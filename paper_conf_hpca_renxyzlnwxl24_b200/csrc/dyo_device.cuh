// Block-level device helpers shared by the decode and planner kernels.
#pragma once
#include <cuda_runtime.h>
#include <cstdint>

namespace dyo {

// Programmatic dependent launch (PDL) for kernel chains on one stream: a kernel launched with
// launch_pdl may be scheduled while its predecessor finishes; pdl_enter() at its top waits for
// the predecessor grid's completion and memory flush (griddepcontrol.wait) before anything
// reads its outputs, then lets this kernel's own successor be scheduled (every CTA has started,
// so a waiting successor never holds slots the primary still needs). DYO_PDL=0 disables it.
__device__ __forceinline__ void pdl_enter() {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

int pdl_enabled();   // api / launch side: 1 unless DYO_PDL=0

template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*k)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                              Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl_enabled() ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, k, static_cast<KArgs>(args)...);
}

// Exclusive scan of one int per thread over the block; *total gets the sum (all threads).
// warp_tmp: >= 32 ints of shared memory. Contains three __syncthreads().
__device__ __forceinline__ int block_scan(int v, int* warp_tmp, int* total) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
  int x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) warp_tmp[w] = x;
  __syncthreads();
  if (w == 0) {
    int s = lane < nw ? warp_tmp[lane] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(0xffffffffu, s, o);
      if (lane >= o) s += y;
    }
    if (lane < nw) warp_tmp[lane] = s;
  }
  __syncthreads();
  const int base = w > 0 ? warp_tmp[w - 1] : 0;
  const int tot = warp_tmp[nw - 1];
  __syncthreads();
  if (total) *total = tot;
  return base + x - v;
}

// Sum of one int64 per thread over the block, returned to every thread. No atomics: 64-bit
// shared-memory atomicAdd compiles to a CAS spin loop (ATOMS.CAST.SPIN.64) that serialises
// under contention. tmp: >= 32 long longs of shared memory. Contains two __syncthreads().
__device__ __forceinline__ long long block_sum64(long long v, long long* tmp) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  if (lane == 0) tmp[w] = v;
  __syncthreads();
  long long t = 0;
  for (int i = 0; i < nw; ++i) t += tmp[i];
  __syncthreads();
  return t;
}

// Exclusive scan of arr[0..n) in place (block-wide, chunks of blockDim); returns the total.
__device__ __forceinline__ int block_scan_array(int* arr, int n, int* warp_tmp) {
  int carry = 0;
  for (int i0 = 0; i0 < n; i0 += blockDim.x) {
    const int i = i0 + threadIdx.x;
    const int v = i < n ? arr[i] : 0;
    int tot = 0;
    const int p = block_scan(v, warp_tmp, &tot);
    if (i < n) arr[i] = carry + p;
    carry += tot;
    __syncthreads();
  }
  return carry;
}

// Ascending bitonic sort of key[0..n) (pads to a power of two with ~0); key has room for it.
__device__ __forceinline__ void block_sort_u64(uint64_t* key, int n) {
  int np2 = 1;
  while (np2 < n) np2 <<= 1;
  for (int i = n + threadIdx.x; i < np2; i += blockDim.x) key[i] = ~0ull;
  __syncthreads();
  for (int k = 2; k <= np2; k <<= 1) {
    for (int j = k >> 1; j > 0; j >>= 1) {
      for (int i = threadIdx.x; i < np2; i += blockDim.x) {
        const int ixj = i ^ j;
        if (ixj > i) {
          const uint64_t x = key[i], z = key[ixj];
          const bool up = (i & k) == 0;
          if ((x > z) == up) { key[i] = z; key[ixj] = x; }
        }
      }
      __syncthreads();
    }
  }
}

// bitonic sort of 64 keys held two per lane (index lane -> x, lane + 32 -> z), ascending
__device__ __forceinline__ void warp_sort64(uint64_t& x, uint64_t& z, int lane) {
#pragma unroll
  for (int k = 2; k <= 64; k <<= 1) {
#pragma unroll
    for (int j = k >> 1; j > 0; j >>= 1) {
      if (j == 32) {
        const uint64_t lo = x < z ? x : z, hi = x < z ? z : x;
        x = lo;
        z = hi;
      } else {
        const uint64_t px = __shfl_xor_sync(0xffffffffu, x, j);
        const uint64_t pz = __shfl_xor_sync(0xffffffffu, z, j);
        const bool lower = (lane & j) == 0;
        const bool upx = (lane & k) == 0, upz = ((lane + 32) & k) == 0;
        x = (lower == upx) ? (x < px ? x : px) : (x < px ? px : x);
        z = (lower == upz) ? (z < pz ? z : pz) : (z < pz ? pz : z);
      }
    }
  }
}

}  // namespace dyo
