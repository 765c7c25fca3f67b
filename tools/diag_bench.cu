// Microbenchmark (tool): latency of the diagonal-block routines of potrf.cu (POTF2 32,
// TRTRI 32, the 64x64 diag_block64v2) on one SM, with and without DMMA-heavy co-runners.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I ../include -o diag_bench diag_bench.cu
#include "../paper_conf_ipps_abdelfattahhtd16_b200/csrc/potrf.cu"
#include <cstdio>

using namespace vb;

__global__ void __launch_bounds__(256) diag_kernel(double* gA, int ld, int reps, long long* out,
                                                   int which) {
  extern __shared__ __align__(128) unsigned char sm[];
  Smem2<Cfg64d>& s = *reinterpret_cast<Smem2<Cfg64d>*>(sm);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  long long t_tot = 0;
  for (int it = 0; it < reps; ++it) {
    // SPD 64x64 block: diag 64 + 0.5 elsewhere (lower), into T
    for (int e = threadIdx.x; e < 64 * 64; e += blockDim.x) {
      const int c = e / 64, r = e % 64;
      s.T[c][r] = (r == c) ? 64.0 + r : 0.5 / (1 + ((r * 7 + c * 3) % 5));
    }
    __syncthreads();
    long long t0 = clock64();
    if (which == 0) {
      if (warp == 0) potf2_block32(&s.T[0][0], Cfg64d::LDT, 32, lane, gA, ld, s.wbuf, s.sv, s.tv);
    } else if (which == 1) {
      if (warp == 0) {
        potf2_block32(&s.T[0][0], Cfg64d::LDT, 32, lane, gA, ld, s.wbuf, s.sv, s.tv);
        t0 = clock64();
        trtri32_dmma_warp(&s.T[0][0], Cfg64d::LDT, s.tv, &s.T[32][0], Cfg64d::LDT, s.S, LDS_T, lane);
      }
    } else {
      if (warp < 4) diag_block64v2(s, 64, warp, lane, gA, ld, true);
    }
    __syncthreads();
    t_tot += clock64() - t0;
  }
  if (threadIdx.x == 0) out[blockIdx.x] = t_tot / reps;
}

// co-runner: DMMA-heavy loop with LDS operands (like the k-loop)
__global__ void __launch_bounds__(256) hog_kernel(double* sink, int iters) {
  __shared__ double b[16][68];
  double acc[2][8][2] = {};
  const int lane = threadIdx.x & 31, g = lane >> 2, q = lane & 3;
  for (int i = threadIdx.x; i < 16 * 68; i += 256) (&b[0][0])[i] = 1e-9 * i;
  __syncthreads();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int kk = 0; kk < 4; ++kk) {
      double fa[2], fb[8];
      for (int mt = 0; mt < 2; ++mt) fa[mt] = b[kk * 4 + q][mt * 8 + g];
      for (int nt = 0; nt < 8; ++nt) fb[nt] = b[kk * 4 + q][nt * 8 + g];
      for (int mt = 0; mt < 2; ++mt)
        for (int nt = 0; nt < 8; ++nt) dmma(acc[mt][nt], fa[mt], fb[nt]);
    }
  }
  double k = 0;
  for (int mt = 0; mt < 2; ++mt) for (int nt = 0; nt < 8; ++nt) k += acc[mt][nt][0];
  if (k == 1.234) sink[0] = k;
}

int main() {
  double* gA; long long* out; double* sink;
  cudaMalloc(&gA, 64 * 64 * 8 * 4); cudaMalloc(&out, 8 * 1024); cudaMalloc(&sink, 64);
  int smem = sizeof(Smem2<Cfg64d>);
  cudaFuncSetAttribute(diag_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const char* names[3] = {"potf2_block32", "trtri32", "diag_block64v2"};
  for (int which = 0; which < 3; ++which) {
    for (int hog = 0; hog < 2; ++hog) {
      cudaStream_t s1, s2; cudaStreamCreate(&s1); cudaStreamCreate(&s2);
      if (hog) hog_kernel<<<148, 256, 0, s2>>>(sink, 200000);
      diag_kernel<<<148, 256, smem, s1>>>(gA, 64, 50, out, which);
      cudaDeviceSynchronize();
      long long h[148]; cudaMemcpy(h, out, sizeof h, cudaMemcpyDeviceToHost);
      double avg = 0; for (int i = 0; i < 148; ++i) avg += h[i]; avg /= 148;
      printf("{\"routine\":\"%s\",\"corunner\":%d,\"cycles\":%.0f,\"err\":\"%s\"}\n", names[which], hog, avg,
             cudaGetErrorString(cudaGetLastError()));
    }
  }
#ifdef VB_DIAG_PROF
  {
    cudaMemset(out, 0, 8);
    unsigned long long z[16] = {};
    cudaMemcpyToSymbol(g_dprof, z, sizeof z);
    diag_kernel<<<148, 256, smem>>>(gA, 64, 50, out, 2);
    cudaDeviceSynchronize();
    unsigned long long h[16];
    cudaMemcpyFromSymbol(h, g_dprof, sizeof h);
    const char* st[8] = {"potf2_1", "trtri_1", "bar_1", "l21_mm_store", "syrk22", "potf2_2", "trtri_2", "bar_end"};
    for (int i = 0; i < 8; ++i) printf("{\"diag64_step\":\"%s\",\"cycles\":%.0f}\n", st[i], h[i] / (148.0 * 50));
  }
#endif
  return 0;
}
