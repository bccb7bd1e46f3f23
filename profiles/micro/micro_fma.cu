// DFMA / FFMA / F2F throughput per SM (tools/, not product code). All results stored.
#include <cuda_runtime.h>
#include <cstdio>
__global__ void kd(double* out, double y, int n) {
  double z0 = threadIdx.x, z1 = z0 + 1, z2 = z0 + 2, z3 = z0 + 3, z4 = z0 + 4, z5 = z0 + 5, z6 = z0 + 6, z7 = z0 + 7;
  for (int i = 0; i < n; ++i) {
    z0 = fma(z0, y, 1e-9); z1 = fma(z1, y, 1e-9); z2 = fma(z2, y, 1e-9); z3 = fma(z3, y, 1e-9);
    z4 = fma(z4, y, 1e-9); z5 = fma(z5, y, 1e-9); z6 = fma(z6, y, 1e-9); z7 = fma(z7, y, 1e-9);
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = z0 + z1 + z2 + z3 + z4 + z5 + z6 + z7;
}
__global__ void kf(float* out, float y, int n) {
  float z0 = threadIdx.x, z1 = z0 + 1, z2 = z0 + 2, z3 = z0 + 3, z4 = z0 + 4, z5 = z0 + 5, z6 = z0 + 6, z7 = z0 + 7;
  for (int i = 0; i < n; ++i) {
    z0 = fmaf(z0, y, 1e-9f); z1 = fmaf(z1, y, 1e-9f); z2 = fmaf(z2, y, 1e-9f); z3 = fmaf(z3, y, 1e-9f);
    z4 = fmaf(z4, y, 1e-9f); z5 = fmaf(z5, y, 1e-9f); z6 = fmaf(z6, y, 1e-9f); z7 = fmaf(z7, y, 1e-9f);
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = z0 + z1 + z2 + z3 + z4 + z5 + z6 + z7;
}
__global__ void kc(double* out, const float* in, int n) {
  double acc = 0; float x = in[threadIdx.x];
  for (int i = 0; i < n; ++i) { x = x * 1.0000001f; acc = fma((double)x, 1.5, acc); }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}
int main() {
  double* od; float* of; float* in;
  cudaMalloc(&od, 148 * 1024 * 8); cudaMalloc(&of, 148 * 1024 * 4); cudaMalloc(&in, 4096); cudaMemset(in, 0, 4096);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b); float ms;
  int n = 1 << 14;
  for (int rep = 0; rep < 2; ++rep) {
    cudaEventRecord(a); kd<<<148, 1024>>>(od, 0.9999, n); cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b);
    printf("DFMA: %.2f TFLOPS (%.1f FMA/clk/SM at 1.965 GHz)\n", 148.0 * 1024 * 8 * n * 2 / ms / 1e9, 148.0 * 1024 * 8 * n / (ms * 1e-3) / 148 / 1.965e9);
    cudaEventRecord(a); kf<<<148, 1024>>>(of, 0.9999f, n); cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b);
    printf("FFMA: %.2f TFLOPS (%.1f FMA/clk/SM)\n", 148.0 * 1024 * 8 * n * 2 / ms / 1e9, 148.0 * 1024 * 8 * n / (ms * 1e-3) / 148 / 1.965e9);
    cudaEventRecord(a); kc<<<148, 1024>>>(od, in, n); cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b);
    printf("F2F+DFMA chain: %.1f conv/clk/SM\n", 148.0 * 1024 * n / (ms * 1e-3) / 148 / 1.965e9);
  }
  return 0;
}
