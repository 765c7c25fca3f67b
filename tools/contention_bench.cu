// Microbenchmark (tool): cost of the POTF2 diagonal-block routine when several warps of an SM
// run it at once (P warps per SM) and when other warps keep the FP64 pipe busy with DMMA
// (D warps per SM), to separate the pivot chain's own latency from pipe contention.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include -o tools/contention_bench tools/contention_bench.cu
#include "../paper_conf_ipps_abdelfattahhtd16_b200/csrc/potrf.cu"
#include <cstdio>

using namespace vb;

__global__ void cont_kernel(double* out, long long* cyc, int P, int reps, int mode) {
  extern __shared__ double sm[];
  __shared__ volatile int stop;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) stop = 0;
  __syncthreads();
  if (warp < P) {
    double* T = sm + warp * (32 * 36 + 64 + 64 + 64);
    double *ws = T + 32 * 36, *sv = ws + 64, *tv = sv + 64;
    double* g = out + ((size_t)blockIdx.x * 64 + warp) * 32 * 32;
    long long tot = 0;
    double x = 0;
    for (int r = 0; r < reps; ++r) {
      for (int c = 0; c < 32; ++c) T[c * 36 + lane] = (c == lane) ? 40.0 + lane : 0.25 / (1 + ((lane * 7 + c * 3) % 5));
      __syncwarp();
      const long long t0 = clock64();
      int info;
      if (mode == 0) {
        info = potf2_block32(T, 36, 32, lane, g, 32, ws, sv, tv);
      } else if (mode == 1) {  // rcp_nr chain of 32 (the pivot reciprocal alone)
        double d = T[lane * 36 + lane];
        for (int j = 0; j < 32; ++j) { d = rcp_nr(d) + 1.0; asm volatile("" : "+d"(d)); }
        info = (int)d;
      } else if (mode == 2) {  // 256 dependent DFMA
        double d = T[lane * 36 + lane];
        for (int j = 0; j < 256; ++j) asm volatile("fma.rn.f64 %0, %0, %1, %2;" : "+d"(d) : "d"(0.999), "d"(1e-9));
        info = (int)d;
      } else if (mode == 3) {  // 256 dependent FFMA (fp32)
        float d = (float)T[lane * 36 + lane];
        for (int j = 0; j < 256; ++j) asm volatile("fma.rn.f32 %0, %0, %1, %2;" : "+f"(d) : "f"(0.999f), "f"(1e-9f));
        info = (int)d;
      } else if (mode == 4) {  // 256 dependent IADD
        int d = lane;
        for (int j = 0; j < 256; ++j) asm volatile("add.s32 %0, %0, %1;" : "+r"(d) : "r"(j));
        info = d & 1;
      } else if (mode == 6) {  // 64 dependent DMMA (one accumulator)
        double acc[2] = {T[lane], 0.0};
        for (int j = 0; j < 64; ++j) dmma(acc, 1e-3, 1e-3);
        info = (int)acc[0];
      } else {  // 64 dependent MUFU.RCP64H
        double d = T[lane * 36 + lane];
        for (int j = 0; j < 64; ++j) asm volatile("rcp.approx.ftz.f64 %0, %0;" : "+d"(d));
        info = (int)d;
      }
      __syncwarp();
      tot += clock64() - t0;
      x += info;
    }
    if (lane == 0) cyc[blockIdx.x * 64 + warp] = tot / reps;
    if (lane == 0) atomicAdd((int*)&stop, 1);
    out[lane] += x;
  } else {
    // DMMA hog: 16 independent accumulators until all POTF2 warps are done
    double acc[16][2];
    for (int i = 0; i < 16; ++i) acc[i][0] = acc[i][1] = lane;
    while (stop < P) {
      for (int it = 0; it < 16; ++it)
#pragma unroll
        for (int i = 0; i < 16; ++i) dmma(acc[i], 1e-3, 1e-3);
    }
    double s = 0;
    for (int i = 0; i < 16; ++i) s += acc[i][0] + acc[i][1];
    out[4096 * 64 + threadIdx.x] = s;
  }
}

int main() {
  double* out;
  long long* cyc;
  cudaMalloc(&out, 8ull * 148 * 64 * 1024 + 8 * 4096 * 128);
  cudaMalloc(&cyc, 8 * 148 * 64);
  cudaFuncSetAttribute(cont_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  const int Ps[] = {1, 4};
  const int Ds[] = {0, 4, 8, 12};
  const char* names[] = {"potf2_block32", "rcp_nr_chain32", "dfma_chain256", "ffma_chain256",
                         "iadd_chain256", "mufu_rcp64h_chain64", "dmma_chain64"};
  for (int mode = 6; mode < 7; ++mode)
    for (int P : Ps)
      for (int D : Ds) {
        if (P + D > 32) continue;
        const size_t smem = (size_t)P * (32 * 36 + 192) * 8;
        cont_kernel<<<148, 32 * (P + D), smem>>>(out, cyc, P, 8, mode);
        if (cudaDeviceSynchronize() != cudaSuccess) { printf("launch failed P=%d D=%d\n", P, D); return 1; }
        long long h[148 * 64];
        cudaMemcpy(h, cyc, sizeof h, cudaMemcpyDeviceToHost);
        double s = 0;
        int c = 0;
        for (int b = 0; b < 148; ++b)
          for (int w = 0; w < P; ++w) s += h[b * 64 + w], ++c;
        printf("{\"op\":\"%s\",\"potf2_warps_per_sm\":%d,\"dmma_warps_per_sm\":%d,\"cycles\":%.0f}\n",
               names[mode], P, D, s / c);
      }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
