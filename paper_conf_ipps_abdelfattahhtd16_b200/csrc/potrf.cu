// potrf.cu — the factorisation kernels of vbatched_dpotrf (steps a2-a7 of SURVEY.md §8(a)).
//
// One persistent kernel drains the work list written by scan_bin (matrices sorted by n
// descending = flops descending):
//   * blocked CTA path, n > 32 (one CTA of 256 threads per matrix): the left-looking
//     blocked Cholesky of PAPER.md Algorithm 1 with panel width NB=32:
//       for each panel j0 (columns j0..j0+NB-1), for each block of MB=128 rows r0 >= j0:
//         panel update   C = A[r0:, j0:j0+NB] - L[r0:, 0:j0] L[j0:j0+NB, 0:j0]^T
//                        (SYRK on the diagonal block + GEMM below, "customized syrk"
//                         with B a part of A, Fig. 2) on DMMA tensor
//                         cores, operands staged by a 3-stage cp.async pipeline
//                         (double buffering);
//         tile factorize L11 = chol(C1)  (POTF2 by one warp, register-resident rows,
//                        warp shuffles for pivot broadcast and column scaling);
//         panel factorize C2 <- C2 L11^-T (TRSM as TRTRI of L11 in shared memory + a
//                        DMMA GEMM, the design of PAPER.md:760-772).
//     Every element of L is written once; previously computed columns are re-read from
//     L2/HBM once per panel (left-looking).
//   * warp path, n <= 32 (one warp per matrix, lane r holds row r in registers): the fused
//     POTF2 of PAPER.md:551-560 with the whole matrix on chip; one HBM read + one write.
// Failed matrices (non-positive or NaN pivot) stop at the failing column and report the
// LAPACK info (SURVEY.md §8(c) readings #2-#3); nothing else is touched again (a7).
#include <algorithm>

#include "common.cuh"
#include "internal.h"

namespace vb {

constexpr int NB = 32;       // panel width (Algorithm 1's nb)
constexpr int MB = 128;      // rows per GEMM/TRSM pass (8 warps x 16 rows)
constexpr int KC = 16;       // k-chunk per pipeline stage
constexpr int STAGES = 3;    // cp.async pipeline depth
constexpr int kThreads = 256;
constexpr int LDA_S = MB + 4;  // padded smem leading dims (conflict-free DMMA fragment loads)
constexpr int LDB_S = NB + 4;
constexpr int LDI = NB + 4;

struct BigSmem {
  union {
    struct {
      double a[STAGES][KC][LDA_S];  // A chunk: [k][row]
      double b[STAGES][KC][LDB_S];  // B chunk: [k][panel row]
    } pipe;
    double tile[NB][LDA_S];  // C tile: [col][row], aliases the pipeline after the k loop
  } u;
  double inv[NB][LDI];  // inv[k][n] = (L11^-1)[n][k]  (DMMA B operand of the TRSM)
  double rdiag[NB];
  int item;
  int info;
};

// ---------------------------------------------------------------------------------------
// POTF2 of an n x n (n <= 32) lower block held one row per lane: a[c] = A[lane][c], c<=lane.
// Right-looking; pivot broadcast and l_kj exchange by shuffles. sqrt is IEEE correctly
// rounded (required so that exact integer families stay exact, SURVEY §8(c) reading #12).
// Returns LAPACK info (1-based failing column) or 0. On failure the pivot stays at (j,j).
VB_DEVINL int potf2_warp_regs(double (&a)[32], int n, int lane) {
  int info = 0;
#pragma unroll
  for (int j = 0; j < 32; ++j) {
    if (j >= n) break;
    const double piv = __shfl_sync(kFull, a[j], j);
    if (!(piv > 0.0)) {  // NaN or <= 0: leading minor of order j+1 not PD
      info = j + 1;
      break;
    }
    const double ljj = sqrt(piv);
    const double rinv = 1.0 / ljj;
    if (lane == j) a[j] = ljj;
    else if (lane > j) a[j] *= rinv;
#pragma unroll
    for (int k = j + 1; k < 32; ++k) {
      if (k >= n) break;
      const double lkj = __shfl_sync(kFull, a[j], k);
      if (lane >= k) a[k] = fma(-a[j], lkj, a[k]);
    }
  }
  return info;
}

// Warp path: one matrix (n <= 32) per warp, whole matrix in registers.
VB_DEVINL void potrf_warp_matrix(double* __restrict__ A, int n, int ld, int* info_out, int lane) {
  double a[32];
#pragma unroll
  for (int c = 0; c < 32; ++c) {
    a[c] = 0.0;
    if (c < n && lane >= c && lane < n) a[c] = A[(size_t)c * ld + lane];
  }
  const int info = potf2_warp_regs(a, n, lane);
#pragma unroll
  for (int c = 0; c < 32; ++c)
    if (c < n && lane >= c && lane < n) A[(size_t)c * ld + lane] = a[c];
  if (lane == 0 && info) *info_out = info;
}

// Stage k-chunk kc of the panel-update operands: A rows r0..r0+MB-1 and the panel rows
// j0..j0+NB-1 (the "B" of Fig. 2), columns kc*KC..kc*KC+KC-1. Rows >= n are zero-filled.
VB_DEVINL void load_stage(BigSmem& s, int st, int kc, const double* __restrict__ A, int n, int ld,
                          int r0, int j0) {
  const int tid = threadIdx.x;
  const int k0 = kc * KC;
#pragma unroll
  for (int e = 0; e < (MB * KC) / kThreads; ++e) {
    const int idx = tid + e * kThreads;
    const int c = idx / MB, r = idx % MB;
    const int row = r0 + r;
    const bool p = row < n;
    cp_async8(&s.u.pipe.a[st][c][r], A + (p ? (size_t)(k0 + c) * ld + row : 0), p);
  }
#pragma unroll
  for (int e = 0; e < (NB * KC) / kThreads; ++e) {
    const int idx = tid + e * kThreads;
    const int c = idx / NB, r = idx % NB;
    const int row = j0 + r;
    const bool p = row < n;
    cp_async8(&s.u.pipe.b[st][c][r], A + (p ? (size_t)(k0 + c) * ld + row : 0), p);
  }
}

// Warp 0: factor the nb x nb diagonal block held in s.u.tile rows/cols 0..nb-1, store L11
// to global, and build inv(L11)^T in s.inv. Sets s.info (0 or local 1-based column).
VB_DEVINL void diag_factor_invert(BigSmem& s, int nb, int lane, double* __restrict__ A, int ld,
                                  int j0) {
  double a[32];
#pragma unroll
  for (int c = 0; c < 32; ++c) a[c] = (c <= lane && lane < nb) ? s.u.tile[c][lane] : 0.0;
  const int info = potf2_warp_regs(a, nb, lane);
  double* Ad = A + (size_t)j0 * ld + j0;
#pragma unroll
  for (int c = 0; c < 32; ++c)
    if (c <= lane && lane < nb) {
      s.u.tile[c][lane] = a[c];
      Ad[(size_t)c * ld + lane] = a[c];
    }
  if (info) {
    if (lane == 0) s.info = info;
    return;
  }
  __syncwarp();
  if (lane < nb) s.rdiag[lane] = 1.0 / s.u.tile[lane][lane];
  __syncwarp();
  // Column `lane` of inv(L11) by forward substitution: x_i = -(sum_{k<i} L_ik x_k) / L_ii.
  double x[32];
#pragma unroll
  for (int i = 0; i < 32; ++i) {
    if (i < nb) {
      double s0 = 0.0, s1 = 0.0;
#pragma unroll
      for (int k = 0; k < i; ++k) {
        if (k & 1) s1 = fma(s.u.tile[k][i], x[k], s1);
        else s0 = fma(s.u.tile[k][i], x[k], s0);
      }
      const double r = s.rdiag[i];
      x[i] = (i < lane) ? 0.0 : ((i == lane) ? r : -(s0 + s1) * r);
    } else {
      x[i] = 0.0;
    }
  }
#pragma unroll
  for (int i = 0; i < 32; ++i) s.inv[lane][i] = x[i];
  if (lane == 0) s.info = 0;
}

// Blocked left-looking Cholesky of one matrix by the whole CTA.
VB_DEVINL void potrf_big_matrix(BigSmem& s, double* __restrict__ A, int n, int ld,
                                int* info_out) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int g = lane >> 2, q = lane & 3;
  for (int j0 = 0; j0 < n; j0 += NB) {
    const int nb = min(NB, n - j0);
    const int nk = j0 / KC;
    for (int r0 = j0; r0 < n; r0 += MB) {
      const bool first = (r0 == j0);
      const bool warp_active = (r0 + warp * 16) < n;
      // ---- panel update (SYRK/GEMM on DMMA): acc = L[r0:r0+MB, 0:j0] L[j0:j0+NB, 0:j0]^T
      double acc[2][4][2];
#pragma unroll
      for (int mt = 0; mt < 2; ++mt)
#pragma unroll
        for (int nt = 0; nt < 4; ++nt) acc[mt][nt][0] = acc[mt][nt][1] = 0.0;
      if (nk > 0) {
#pragma unroll
        for (int st = 0; st < STAGES - 1; ++st) {
          if (st < nk) load_stage(s, st, st, A, n, ld, r0, j0);
          cp_async_commit();
        }
        for (int kc = 0; kc < nk; ++kc) {
          cp_async_wait<STAGES - 2>();
          __syncthreads();
          const int pf = kc + STAGES - 1;
          if (pf < nk) load_stage(s, pf % STAGES, pf, A, n, ld, r0, j0);
          cp_async_commit();
          const int st = kc % STAGES;
          if (warp_active) {
#pragma unroll
            for (int kk = 0; kk < KC / 4; ++kk) {
              const double* sa = &s.u.pipe.a[st][kk * 4 + q][warp * 16 + g];
              const double a0 = sa[0], a1 = sa[8];
              const double* sb = &s.u.pipe.b[st][kk * 4 + q][g];
              double b[4];
#pragma unroll
              for (int nt = 0; nt < 4; ++nt) b[nt] = sb[nt * 8];
#pragma unroll
              for (int nt = 0; nt < 4; ++nt) {
                dmma(acc[0][nt], a0, b[nt]);
                dmma(acc[1][nt], a1, b[nt]);
              }
            }
          }
        }
        cp_async_wait<0>();
      }
      __syncthreads();  // pipeline buffers are free: reuse as the C tile
#pragma unroll
      for (int mt = 0; mt < 2; ++mt)
#pragma unroll
        for (int nt = 0; nt < 4; ++nt) {
          const int r = warp * 16 + mt * 8 + g, c = nt * 8 + 2 * q;
          s.u.tile[c][r] = -acc[mt][nt][0];
          s.u.tile[c + 1][r] = -acc[mt][nt][1];
        }
      __syncthreads();
      // C = A - acc  (coalesced read of the panel's original values, L2-only load)
      for (int idx = tid; idx < NB * MB; idx += kThreads) {
        const int c = idx / MB, r = idx % MB;
        if (c < nb && r0 + r < n) s.u.tile[c][r] += __ldcg(A + (size_t)(j0 + c) * ld + (r0 + r));
      }
      __syncthreads();
      if (first) {
        if (warp == 0) diag_factor_invert(s, nb, lane, A, ld, j0);
        __syncthreads();
        if (s.info) {
          if (tid == 0) *info_out = j0 + s.info;
          return;
        }
        if (r0 + nb >= n) continue;  // no rows below the diagonal block in this pass
      }
      // ---- panel factorize (TRSM): X = C inv(L11)^T on DMMA
      double x[2][4][2];
#pragma unroll
      for (int mt = 0; mt < 2; ++mt)
#pragma unroll
        for (int nt = 0; nt < 4; ++nt) x[mt][nt][0] = x[mt][nt][1] = 0.0;
      if (warp_active) {
#pragma unroll
        for (int k4 = 0; k4 < NB / 4; ++k4) {
          const double a0 = s.u.tile[k4 * 4 + q][warp * 16 + g];
          const double a1 = s.u.tile[k4 * 4 + q][warp * 16 + 8 + g];
          double b[4];
#pragma unroll
          for (int nt = 0; nt < 4; ++nt) b[nt] = s.inv[k4 * 4 + q][nt * 8 + g];
#pragma unroll
          for (int nt = 0; nt < 4; ++nt) {
            dmma(x[0][nt], a0, b[nt]);
            dmma(x[1][nt], a1, b[nt]);
          }
        }
      }
      __syncthreads();
#pragma unroll
      for (int mt = 0; mt < 2; ++mt)
#pragma unroll
        for (int nt = 0; nt < 4; ++nt) {
          const int r = warp * 16 + mt * 8 + g, c = nt * 8 + 2 * q;
          s.u.tile[c][r] = x[mt][nt][0];
          s.u.tile[c + 1][r] = x[mt][nt][1];
        }
      __syncthreads();
      const int row_lo = first ? j0 + nb : r0;
      for (int idx = tid; idx < NB * MB; idx += kThreads) {
        const int c = idx / MB, r = idx % MB;
        const int row = r0 + r;
        if (c < nb && row < n && row >= row_lo) A[(size_t)(j0 + c) * ld + row] = s.u.tile[c][r];
      }
      __syncthreads();
    }
  }
}

template <bool kBig>
__global__ void __launch_bounds__(kThreads, 2)
    potrf_persistent_kernel(const int* __restrict__ d_n, double* const* __restrict__ dA,
                            const int* __restrict__ d_ldda, int* __restrict__ d_info,
                            const Ctrl* __restrict__ ctrl_c, const int* __restrict__ order) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  Ctrl* ctrl = const_cast<Ctrl*>(ctrl_c);
  pdl_wait();  // the scan's outputs (order, ctrl, info) are complete and visible
  const int count_big = ctrl->count_big;
  const int count_warp = ctrl->count_warp;
  const int tid = threadIdx.x, lane = tid & 31;
  if constexpr (kBig) {
    BigSmem& s = *reinterpret_cast<BigSmem*>(smem_raw);
    for (;;) {
      if (tid == 0) s.item = atomicAdd(&ctrl->head_big, 1);
      __syncthreads();
      const int it = s.item;
      __syncthreads();
      if (it >= count_big) break;
      const int m = order[it];
      potrf_big_matrix(s, dA[m], d_n[m], d_ldda[m], d_info + m);
      __syncthreads();
    }
  }
  for (;;) {
    int w = 0;
    if (lane == 0) w = atomicAdd(&ctrl->head_warp, 1);
    w = __shfl_sync(kFull, w, 0);
    if (w >= count_warp) break;
    const int m = order[count_big + w];
    potrf_warp_matrix(dA[m], d_n[m], d_ldda[m], d_info + m, lane);
  }
}

static int g_num_sms = 0;
static int g_occ_big = 0;

static cudaError_t init_device_info() {
  if (g_num_sms) return cudaSuccess;
  int dev;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  e = cudaDeviceGetAttribute(&g_num_sms, cudaDevAttrMultiProcessorCount, dev);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(potrf_persistent_kernel<true>,
                           cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(BigSmem));
  if (e != cudaSuccess) return e;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&g_occ_big, potrf_persistent_kernel<true>,
                                                    kThreads, sizeof(BigSmem));
  if (e != cudaSuccess) return e;
  if (g_occ_big < 1) g_occ_big = 1;
  return cudaSuccess;
}

cudaError_t launch_potrf_paths(const int* d_n, double* const* dA, const int* d_ldda, int* d_info,
                               int batch, int max_n_hint, const Ctrl* ctrl, const int* order,
                               cudaStream_t stream) {
  cudaError_t e = init_device_info();
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg = {};
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  cfg.stream = stream;
  cfg.blockDim = dim3(kThreads);
  if (max_n_hint > kWarpMaxN) {
    const int grid = std::max(1, std::min(batch, g_num_sms * g_occ_big));
    cfg.gridDim = dim3(grid);
    cfg.dynamicSmemBytes = sizeof(BigSmem);
    return cudaLaunchKernelEx(&cfg, potrf_persistent_kernel<true>, d_n, dA, d_ldda, d_info, ctrl,
                              order);
  }
  // Only warp-path matrices: one warp per matrix, 8 warps per CTA.
  const int warps = std::max(1, batch);
  const int grid = std::max(1, std::min((warps + 7) / 8, g_num_sms * 8));
  cfg.gridDim = dim3(grid);
  cfg.dynamicSmemBytes = 0;
  return cudaLaunchKernelEx(&cfg, potrf_persistent_kernel<false>, d_n, dA, d_ldda, d_info, ctrl,
                            order);
}

}  // namespace vb
