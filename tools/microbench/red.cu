// Global RED.ADD.F32 throughput into L2-resident per-CTA regions (long-row numeric design probe)
#include <cstdio>
#include <cuda_runtime.h>
__global__ void k_red(float* base, int region_words, int iters, int spacing, int mode) {
  float* r = base + (size_t)blockIdx.x * region_words;
  unsigned x = blockIdx.x * 7919u + threadIdx.x * 104729u + 1u;
  for (int i = 0; i < iters; ++i) {
    unsigned idx;
    if (mode == 0) { x = x * 1664525u + 1013904223u; idx = x % region_words; }           // random
    else { idx = ((unsigned)i * 32u * spacing + (threadIdx.x & 31) * spacing + (threadIdx.x >> 5) * 7919u) % region_words; } // strided within warp
    atomicAdd(r + idx, 1.0f);
  }
}
__global__ void k_sts(float* base, int region_words, int iters) {
  float* r = base + (size_t)blockIdx.x * region_words;
  unsigned x = blockIdx.x * 7919u + threadIdx.x * 104729u + 1u;
  for (int i = 0; i < iters; ++i) { x = x * 1664525u + 1013904223u; r[x % region_words] = 1.0f; }
}
int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int regions[] = {16384, 65536, 262144};
  float* buf; cudaMalloc(&buf, (size_t)sms * 2 * 262144 * 4);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  for (int rw : regions) for (int mode = 0; mode < 2; ++mode) for (int ctas = 1; ctas <= 2; ++ctas) {
    int iters = 2000, T = 1024 / ctas;
    int grid = sms * ctas;
    k_red<<<grid, T>>>(buf, rw, 10, 15, mode);
    cudaEventRecord(a);
    k_red<<<grid, T>>>(buf, rw, iters, 15, mode);
    cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    double ops = (double)grid * T * iters;
    printf("RED.F32 region %7d words/CTA (%.1f MB total) %s ctas/SM=%d: %8.1f Gop/s\n", rw, grid * (double)rw * 4 / 1e6,
           mode ? "warp-strided(15)" : "random          ", ctas, ops / ms / 1e6);
  }
  for (int rw : regions) {
    int iters = 2000; k_sts<<<sms, 1024>>>(buf, rw, 10);
    cudaEventRecord(a); k_sts<<<sms, 1024>>>(buf, rw, iters); cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    printf("STG random region %7d: %8.1f Gop/s\n", rw, (double)sms * 1024 * iters / ms / 1e6);
  }
  return 0;
}
