// Microbenchmark (tool): cycles of the pivot-chain routines (POTF2 / TRTRI of a 32x32 tile) on
// one warp, alone and with 1/3 other warps of the SAME sub-partition running the same routine
// (the quad kernel puts four CTAs' chain warps on SMSP 0). One CTA per SM, warps 0,4,8,12 = SMSP 0.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/chain_bench tools/chain_bench.cu
#include "../paper_conf_ipps_abdelfattahhtd16_b200/csrc/potrf.cu"
#include "quad_experiment.cuh"
#include <cstdio>

using namespace vb;

namespace vb {
// DMMA-free variants of the pivot-chain routines (measured slower than the DMMA ones: these
// numbers are why the product keeps potf2_block32 / trtri32_dmma_warp). A DMMA stream starves every FP64 latency chain
// issued on the same SM sub-partition (tools/pipe_share_bench.cu, profiles/r02: a 256-long DFMA
// chain 2.2 K -> 120 K cycles, POTF2(32) 5.8 K -> 237 K cycles beside one DMMA-streaming warp of
// the same SMSP; DMMA streams on the other three SMSPs cost nothing). The small kernel keeps its
// chain warps on a sub-partition of their own, so their own routines must not issue DMMAs
// either (one chain warp's TRTRI on DMMA starved the other chain warps' POTF2 2.9x).

// POTF2 of the nb x nb (nb <= 32) lower block in T (T[c*ldt + r]) by one warp, the whole block
// in registers (lane r = row r; potf2_regs_warp<32>, DFMA only), written back to T and to global
// (Ag, lda) — columns < nb, on failure up to and including the failing column. sv/tv receive
// l_cc and 1/l_cc. Returns info.
template <bool UP, typename E = double>
VB_DEVINL int potf2_tile32_dfma(double* T, int ldt, int nb, int lane, E* Ag, int lda, double* ws,
                                double* sv, double* tv) {
  double a[32];
#pragma unroll
  for (int c = 0; c < 32; ++c)
    a[c] = (c < nb && lane < nb) ? T[c * ldt + lane] : selp(c == lane, 1.0, 0.0);
  const int info = potf2_regs_warp<32>(a, nb, lane, ws, sv, tv);
  const int ncol = info ? info : nb;
#pragma unroll
  for (int c = 0; c < 32; ++c)
    if (c < ncol && lane >= c && lane < nb) {
      T[c * ldt + lane] = a[c];
      Ag[gix<UP>(lane, c, lda)] = a[c];
    }
  __syncwarp();
  return info;
}

// Inverse of a 32x32 lower-triangular L (T[c*ldt + r] = L[r][c], tv[c] = 1/L[c][c]) by one warp
// with DFMA only: lane c computes column c of X = L^-1 by forward substitution in right-looking
// order (after x_j is known, every pending sum s_i, i > j, takes its term: 31 - j independent
// FMAs per step, so the dependent chain is one DMUL + one DFMA per column). Output
// INV[k*ldi + n] = X[n][k] (the TRSM's B-operand layout), the full 32x32 block written (zeros
// above the diagonal of X).
VB_DEVINL void trtri32_dfma_warp(const double* T, int ldt, const double* tv, double* INV, int ldi,
                                 int lane) {
  double sacc[32];
#pragma unroll
  for (int i = 0; i < 32; ++i) sacc[i] = 0.0;
#pragma unroll
  for (int j = 0; j < 32; ++j) {
    const double xj = (j < lane) ? 0.0 : ((j == lane) ? tv[j] : -sacc[j] * tv[j]);
    INV[lane * ldi + j] = xj;
#pragma unroll
    for (int i = j + 1; i < 32; ++i) sacc[i] = fma(T[j * ldt + i], xj, sacc[i]);
  }
  __syncwarp();
}

}  // namespace vb

__global__ void __launch_bounds__(512, 1) chain_kernel(double* out, long long* cyc, int nwarps_smsp0, int mode, int reps,
                                                       int nbr, int hogs, const double* src) {
  extern __shared__ double sm[];
  __shared__ volatile int stop;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) stop = 0;
  __syncthreads();
  if (warp % 4 != 0) {  // hogs on SMSPs 1-3: the quad kernel's strip k-loop (L2 fragments + DMMA)
    if (!hogs || warp / 4 >= nwarps_smsp0) return;
    double acc[2][4][2] = {};
    const double* A = src + (((size_t)blockIdx.x * 16 + warp) * 4096) % ((1 << 20) - 4096);
    while (stop < nwarps_smsp0) strip_kloop_t<false, double, 2, 4, -1>(acc, A, 64, 64, 0, 16, 0, 48, lane);
    double s = 0;
    for (int i = 0; i < 2; ++i)
      for (int j = 0; j < 4; ++j) s += acc[i][j][0] + acc[i][j][1];
    out[(size_t)gridDim.x * 16 * 1024 + 512 + threadIdx.x] = s;
    return;
  }
  if (warp / 4 >= nwarps_smsp0) return;
  double* T = sm + (warp / 4) * (32 * 36 * 2 + 64 + 64 + 64 + 16 * LDS_T);
  double *INV = T + 32 * 36, *ws = INV + 32 * 36, *sv = ws + 64, *tv = sv + 64, *S = tv + 64;
  double* g = out + ((size_t)blockIdx.x * 16 + warp) * 32 * 32;
  long long tot = 0;
  double x = 0;
  for (int r = 0; r < reps; ++r) {
    for (int c = 0; c < 32; ++c) T[c * 36 + lane] = (c == lane) ? 40.0 + lane : 0.25 / (1 + ((lane * 7 + c * 3) % 5));
    for (int c = 0; c < 32; ++c) tv[c] = 1.0 / (40.0 + c);
    __syncwarp();
    const long long t0 = clock64();
    int info = 0;
    if (mode == 0) info = potf2_block32<false>(T, 36, nbr, lane, g, 32, ws, sv, tv);
    else if (mode == 1) info = potf2_tile32_dfma<false>(T, 36, nbr, lane, g, 32, ws, sv, tv);
    else if (mode == 2) trtri32_dmma_warp(T, 36, tv, INV, 36, S, LDS_T, lane);
    else trtri32_dfma_warp(T, 36, tv, INV, 36, lane);
    __syncwarp();
    tot += clock64() - t0;
    x += info + INV[lane];
  }
  if (lane == 0) cyc[blockIdx.x * 16 + warp / 4] = tot / reps;
  if (lane == 0) atomicAdd((int*)&stop, 1);
  out[(size_t)gridDim.x * 16 * 1024 + threadIdx.x] = x;
}

int main() {
  double *out, *src;
  long long* cyc;
  cudaMalloc(&src, 8ull << 20);
  cudaMemset(src, 0, 8ull << 20);
  cudaMalloc(&out, 8ull * (148 * 16 * 1024 + 1024));
  cudaMalloc(&cyc, 8 * 148 * 16);
  const int smem = 4 * (32 * 36 * 2 + 192 + 16 * LDS_T) * 8;
  cudaFuncSetAttribute(chain_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const char* names[] = {"potf2_block32 (dmma syrk)", "potf2_tile32_dfma", "trtri32_dmma", "trtri32_dfma"};
  for (int hogs = 0; hogs < 2; ++hogs)
  for (int mode = 0; mode < 4; ++mode)
    for (int w : {1, 2, 4}) {
      chain_kernel<<<148, 512, smem>>>(out, cyc, w, mode, 16, 32, hogs, src);
      if (cudaDeviceSynchronize() != cudaSuccess || cudaGetLastError() != cudaSuccess) { printf("fail\n"); return 1; }
      long long h[148 * 16];
      cudaMemcpy(h, cyc, sizeof h, cudaMemcpyDeviceToHost);
      double s = 0;
      for (int b = 0; b < 148; ++b)
        for (int i = 0; i < w; ++i) s += h[b * 16 + i];
      printf("{\"routine\":\"%s\",\"warps_on_smsp0\":%d,\"strip_kloop_hogs_smsp123\":%d,\"cycles\":%.0f}\n", names[mode], w, hogs ? 3 * w : 0, s / (148 * w));
    }
  return 0;
}
