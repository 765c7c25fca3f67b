// FP64 microbenchmarks for B200 (sm_100a): DFMA pipe peak, DMMA (mma.sync m8n8k4 f64)
// peak, and a check of the m8n8k4 f64 fragment layout. Standalone tool; not part of the
// library. Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o fp64_peaks fp64_peaks.cu
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); exit(1);} } while (0)

template <int CHAINS>
__global__ void dfma_kernel(double* out, int iters, double a, double b) {
  double acc[CHAINS];
#pragma unroll
  for (int c = 0; c < CHAINS; ++c) acc[c] = threadIdx.x * 1e-9 + c;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int u = 0; u < 16; ++u)
#pragma unroll
      for (int c = 0; c < CHAINS; ++c) acc[c] = fma(acc[c], a, b);
  }
  double s = 0;
#pragma unroll
  for (int c = 0; c < CHAINS; ++c) s += acc[c];
  if (s == 12345.678) out[0] = s;
}

__device__ __forceinline__ void dmma(double& d0, double& d1, double a, double b) {
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
               : "+d"(d0), "+d"(d1) : "d"(a), "d"(b));
}

template <int ACC>
__global__ void dmma_kernel(double* out, int iters) {
  double c0[ACC], c1[ACC];
  double a = 1.0 + threadIdx.x * 1e-12, b = 1.0 - threadIdx.x * 1e-12;
#pragma unroll
  for (int i = 0; i < ACC; ++i) { c0[i] = i; c1[i] = -i; }
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int u = 0; u < 4; ++u)
#pragma unroll
      for (int i = 0; i < ACC; ++i) dmma(c0[i], c1[i], a, b);
  }
  double s = 0;
#pragma unroll
  for (int i = 0; i < ACC; ++i) s += c0[i] + c1[i];
  if (s == 12345.678) out[0] = s;
}

// Layout probe: lane l supplies A[l>>2][l&3] and B[l&3][l>>2]; writes its two C values.
__global__ void layout_kernel(const double* A, const double* B, double* C) {
  int l = threadIdx.x;
  double a = A[(l >> 2) * 4 + (l & 3)];   // A row-major 8x4
  double b = B[(l & 3) * 8 + (l >> 2)];   // B row-major 4x8
  double d0 = 0, d1 = 0;
  dmma(d0, d1, a, b);
  C[(l >> 2) * 8 + (l & 3) * 2 + 0] = d0;  // C row-major 8x8
  C[(l >> 2) * 8 + (l & 3) * 2 + 1] = d1;
}

int main() {
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, 0));
  int clk = 0; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("{\"device\":\"%s\",\"sms\":%d,\"l2_bytes\":%d,\"smem_optin\":%zu,\"smem_per_sm\":%zu,"
         "\"regs_per_sm\":%d,\"clock_khz\":%d,\"cc\":\"%d.%d\",\"mem_bytes\":%zu}\n",
         p.name, p.multiProcessorCount, p.l2CacheSize, p.sharedMemPerBlockOptin,
         p.sharedMemPerMultiprocessor, p.regsPerMultiprocessor, clk, p.major, p.minor,
         p.totalGlobalMem);
  double* out; CK(cudaMalloc(&out, 64));
  // layout probe
  {
    double hA[32], hB[32], hC[64], ref[64];
    for (int i = 0; i < 32; ++i) { hA[i] = i + 1; hB[i] = (i * 7) % 11 - 5; }
    for (int i = 0; i < 8; ++i) for (int j = 0; j < 8; ++j) {
      double s = 0; for (int k = 0; k < 4; ++k) s += hA[i * 4 + k] * hB[k * 8 + j]; ref[i * 8 + j] = s; }
    double *dA, *dB, *dC; CK(cudaMalloc(&dA, 256)); CK(cudaMalloc(&dB, 256)); CK(cudaMalloc(&dC, 512));
    CK(cudaMemcpy(dA, hA, 256, cudaMemcpyHostToDevice)); CK(cudaMemcpy(dB, hB, 256, cudaMemcpyHostToDevice));
    layout_kernel<<<1, 32>>>(dA, dB, dC); CK(cudaDeviceSynchronize());
    CK(cudaMemcpy(hC, dC, 512, cudaMemcpyDeviceToHost));
    int bad = 0; for (int i = 0; i < 64; ++i) bad += hC[i] != ref[i];
    printf("{\"dmma_layout_mismatches\":%d}\n", bad);
  }
  cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
  int sms = p.multiProcessorCount;
  for (int blocks_per_sm : {4, 8}) {
    int iters = 4096, threads = 256, grid = sms * blocks_per_sm;
    dfma_kernel<8><<<grid, threads>>>(out, 16, 1.0000001, 1e-9); CK(cudaDeviceSynchronize());
    float best = 1e30f;
    for (int r = 0; r < 5; ++r) {
      CK(cudaEventRecord(e0)); dfma_kernel<8><<<grid, threads>>>(out, iters, 1.0000001, 1e-9);
      CK(cudaEventRecord(e1)); CK(cudaEventSynchronize(e1));
      float ms; CK(cudaEventElapsedTime(&ms, e0, e1)); if (ms < best) best = ms;
    }
    double flops = 2.0 * grid * threads * (double)iters * 16 * 8;
    printf("{\"kernel\":\"dfma\",\"blocks_per_sm\":%d,\"ms\":%.4f,\"tflops\":%.3f}\n", blocks_per_sm, best, flops / best / 1e9);
  }
  for (int warps_per_sm : {8, 16, 32}) {
    int iters = 2048, threads = 256, grid = sms * warps_per_sm / 8;
    dmma_kernel<8><<<grid, threads>>>(out, 16); CK(cudaDeviceSynchronize());
    float best = 1e30f;
    for (int r = 0; r < 5; ++r) {
      CK(cudaEventRecord(e0)); dmma_kernel<8><<<grid, threads>>>(out, iters);
      CK(cudaEventRecord(e1)); CK(cudaEventSynchronize(e1));
      float ms; CK(cudaEventElapsedTime(&ms, e0, e1)); if (ms < best) best = ms;
    }
    double flops = 2.0 * 256 * (grid * threads / 32) * (double)iters * 4 * 8;
    printf("{\"kernel\":\"dmma_m8n8k4\",\"warps_per_sm\":%d,\"ms\":%.4f,\"tflops\":%.3f}\n", warps_per_sm, best, flops / best / 1e9);
  }
  return 0;
}
