// Microbenchmark (tool): which sub-partitions' DMMA streams slow a latency-bound FP64 chain?
// One CTA of 8 warps per SM (warp w on SMSP w % 4). Warp 0 runs a chain (POTF2(32), a DFMA
// chain, a SHFL chain or an LDS chain); the warps in `hog_mask` stream independent DMMAs (or
// L2 loads, hog kind 1) until the chain warp is done. Prints the chain's cycles per case.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/pipe_share_bench tools/pipe_share_bench.cu
#include "../paper_conf_ipps_abdelfattahhtd16_b200/csrc/potrf.cu"
#include "quad_experiment.cuh"
#include <cstdio>

using namespace vb;

__global__ void share_kernel(double* out, const double* src, long long* cyc, int hog_mask, int mode,
                             int hog_kind, int reps) {
  __shared__ double T[32 * 36 + 192];
  __shared__ volatile int stop;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) stop = 0;
  __syncthreads();
  if (warp == 0) {
    double *ws = T + 32 * 36, *sv = ws + 64, *tv = sv + 64;
    double* g = out + (size_t)blockIdx.x * 32 * 32;
    long long tot = 0;
    double x = 0;
    for (int r = 0; r < reps; ++r) {
      for (int c = 0; c < 32; ++c) T[c * 36 + lane] = (c == lane) ? 40.0 + lane : 0.25 / (1 + ((lane * 7 + c * 3) % 5));
      __syncwarp();
      const long long t0 = clock64();
      int info = 0;
      if (mode == 0) {
        info = potf2_block32<false>(T, 36, 32, lane, g, 32, ws, sv, tv);
      } else if (mode == 1) {
        double d = T[lane * 36 + lane];
        for (int j = 0; j < 256; ++j) asm volatile("fma.rn.f64 %0, %0, %1, %2;" : "+d"(d) : "d"(0.999), "d"(1e-9));
        info = (int)d;
      } else if (mode == 2) {
        double d = T[lane * 36 + lane];
        for (int j = 0; j < 256; ++j) d = __shfl_sync(kFull, d, (lane + 1) & 31);
        info = (int)d;
      } else {
        int idx = lane;
        const int* Ti = reinterpret_cast<const int*>(T);
        for (int j = 0; j < 256; ++j) idx = (Ti[idx] & 31) + lane * 0;
        info = idx;
      }
      __syncwarp();
      tot += clock64() - t0;
      x += info;
    }
    if (lane == 0) cyc[blockIdx.x] = tot / reps;
    if (lane == 0) stop = 1;
    out[(size_t)gridDim.x * 1024 + lane] += x;
  } else if ((hog_mask >> warp) & 1) {
    if (hog_kind == 0) {
      double acc[16][2];
      for (int i = 0; i < 16; ++i) acc[i][0] = acc[i][1] = lane;
      while (!stop) {
        for (int it = 0; it < 16; ++it)
#pragma unroll
          for (int i = 0; i < 16; ++i) dmma(acc[i], 1e-3, 1e-3);
      }
      double s = 0;
      for (int i = 0; i < 16; ++i) s += acc[i][0] + acc[i][1];
      out[(size_t)gridDim.x * 1024 + 64 + threadIdx.x] = s;
    } else if (hog_kind == 2) {  // the quad kernel's strip k-loop: L2 fragments + DMMA
      double acc[2][4][2] = {};
      const double* A = src + (((size_t)blockIdx.x * 8 + warp) * 4096) % ((1 << 20) - 4096);
      while (!stop) strip_kloop_t<false, double, 2, 4, -1>(acc, A, 64, 64, 0, 16, 0, 48, lane);
      double s = 0;
      for (int i = 0; i < 2; ++i)
        for (int j = 0; j < 4; ++j) s += acc[i][j][0] + acc[i][j][1];
      out[(size_t)gridDim.x * 1024 + 64 + threadIdx.x] = s;
    } else {  // L2 load stream (LDG.64 __ldcg), 8 in flight per lane
      double s = 0;
      size_t off = ((size_t)blockIdx.x * 8 + warp) * 4096 + lane;
      while (!stop) {
#pragma unroll
        for (int i = 0; i < 8; ++i) s += __ldcg(src + ((off + i * 32) & ((1 << 20) - 1)));
        off += 256;
      }
      out[(size_t)gridDim.x * 1024 + 64 + threadIdx.x] = s;
    }
  }
}

int main() {
  double *out, *src;
  long long* cyc;
  cudaMalloc(&out, 8ull * (148 * 1024 + 4096));
  cudaMalloc(&src, 8ull << 20);
  cudaMemset(src, 0, 8ull << 20);
  cudaMalloc(&cyc, 8 * 148);
  const char* modes[] = {"potf2_block32", "dfma_chain256", "shfl_chain256", "lds_chain256"};
  struct H { int mask; const char* what; };
  const H hogs[] = {{0, "none"},
                    {1 << 4, "SMSP0 (same as chain)"},
                    {1 << 1, "SMSP1"},
                    {1 << 2, "SMSP2"},
                    {(1 << 2) | (1 << 3), "SMSP2+3"},
                    {(1 << 1) | (1 << 2) | (1 << 3), "SMSP1+2+3"},
                    {(1 << 1) | (1 << 2) | (1 << 3) | (1 << 5) | (1 << 6) | (1 << 7), "SMSP1+2+3 x2"},
                    {0xFE, "all incl SMSP0"}};
  for (int kind = 0; kind < 3; ++kind)
    for (int mode = 0; mode < (kind == 2 ? 1 : 4); ++mode)
      for (const H& h : hogs) {
        share_kernel<<<148, 256>>>(out, src, cyc, h.mask, mode, kind, 8);
        if (cudaDeviceSynchronize() != cudaSuccess) { printf("launch failed\n"); return 1; }
        long long c[148];
        cudaMemcpy(c, cyc, sizeof c, cudaMemcpyDeviceToHost);
        double s = 0;
        for (int b = 0; b < 148; ++b) s += c[b];
        printf("{\"chain\":\"%s\",\"hog\":\"%s\",\"hog_warps\":\"%s\",\"cycles\":%.0f}\n", modes[mode],
               kind == 2 ? "strip_kloop" : (kind ? "ldg_l2" : "dmma"), h.what, s / 148);
      }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
