// potrf.cu — the factorisation kernels of vbatched_dpotrf (steps a2-a7 of SURVEY.md §8(a)).
//
// Two persistent kernels drain the work list written by scan_bin (matrices sorted by n
// descending = flops descending, i.e. longest-processing-time first):
//
//  * potrf_blocked_kernel, n > 32: one CTA (8 warps) per matrix, the left-looking blocked
//    Cholesky of PAPER.md Algorithm 1 with panel width NB = 32:
//      for each panel j0 (columns j0..j0+NB-1), for each block of MB = 128 rows r0 >= j0:
//        panel update    C = A[r0:, j0:j0+NB] - L[r0:, 0:j0] L[j0:j0+NB, 0:j0]^T
//                        ("customized syrk" with B a part of A, Fig. 2) on
//                        the FP64 tensor cores (DMMA), operands staged by a 3-stage cp.async
//                        pipeline (double buffering); the accumulators start
//                        from A's panel values, loaded before the k loop;
//        tile factorize  L11 = chol(C1): POTF2 by one warp on the 32x32 block in shared
//                        memory (row-owner lanes, LDL^T-form right-looking update so that
//                        sqrt and the column scaling are off the column-to-column chain);
//        panel factorize C2 <- C2 L11^-T: TRTRI of L11 by recursive doubling on DMMA in
//                        shared memory, then a DMMA GEMM — the trtri + gemm TRSM design of
//                        PAPER.md:760-772.
//    Every element of L is written once; earlier columns are re-read once per panel.
//  * potrf_warp_kernel, n <= 32: one warp per matrix, whole matrix in shared memory
//    (the fused on-chip POTF2 of PAPER.md:551-560; one HBM read, one HBM write). It is
//    launched after the blocked kernel with programmatic dependent launch and starts on the
//    SMs the blocked kernel's CTAs free once its work list is empty (the smallest matrices
//    come last in LPT order anyway).
// Failed matrices (pivot <= 0 or NaN) stop at the failing column and report the LAPACK info
// (SURVEY.md §8(c) readings #2-#3); nothing of them is touched again (a7).
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
constexpr int LDS_S = 20;      // TRTRI scratch

struct BigSmem {
  union {
    struct {
      double a[STAGES][KC][LDA_S];  // A chunk: [k][row]
      double b[STAGES][KC][LDB_S];  // B chunk: [k][panel row]
    } pipe;
    struct {
      double tile[NB][LDA_S];  // C tile: [col][row], aliases the pipeline after the k loop
      double scratch[16 * LDS_S * 2];  // TRTRI scratch
    } e;
  } u;
  double inv[NB][LDI];      // inv[k][n] = (L11^-1)[n][k]  (DMMA B operand of the TRSM)
  double wbuf[2 * NB];
  double sv[NB];
  double tv[NB];
  int item;
  int info;
};

// ---------------------------------------------------------------------------------------
// POTF2 of an nb x nb (nb <= NM <= 32) lower block by one warp, lane r holding row r in
// registers (a[c] = A[r][c], c <= r; entries c > r are don't-care). Right-looking in LDL^T
// form: with d_j the j-th pivot and u_rj the updated column, a_rk -= u_rj * w_kj where
// w_kj = u_kj / d_j. The next pivot d_{j+1} = a_{j+1,j+1} - u_{j+1,j} w_{j+1,j} needs only
// lane j+1's own values, so the column-to-column chain is shfl -> rcp -> mul -> fma -> shfl;
// the multipliers w_kj reach the other lanes through a double-buffered shared-memory row
// (ws[2][32]). sqrt (IEEE correctly rounded, SURVEY §8(c) reading #12) and the scaling
// l_rj = u_rj / l_jj happen in one parallel pass at the end.
// Returns LAPACK info (1-based failing column; pivot !(d > 0) incl. NaN) or 0. On failure
// columns < j hold L, the pivot d_j stays at (j,j) (lane j's a[j] == d_j), later entries are
// partially updated. sv/tv (shared, >= NM doubles) receive l_cc and 1/l_cc.
template <int NM>
VB_DEVINL int potf2_regs_warp(double (&a)[NM], int nb, int lane, double* ws, double* sv,
                              double* tv) {
  int info = 0;
  double myd = 1.0;
  double dn = a[0];  // candidate next pivot (meaningful in lane j+1)
#pragma unroll
  for (int j = 0; j < NM; ++j) {
    if (j >= nb) break;
    const double d = __shfl_sync(kFull, dn, j);
    if (!(d > 0.0)) {
      info = j + 1;
      break;
    }
    if (lane == j) myd = d;
    const double rd = 1.0 / d;
    const double u = a[j];
    const double w = u * rd;
    double* wb = ws + (j & 1) * 32;
    wb[lane] = w;
    if (j + 1 < NM) dn = fma(-u, w, a[(j + 1) < NM ? j + 1 : 0]);
    __syncwarp();
#pragma unroll
    for (int k = j + 1; k < NM; ++k) a[k] = fma(-u, wb[k], a[k]);
  }
  const int ncols = info ? info - 1 : nb;
  const double sq = sqrt(myd);
  const double isq = 1.0 / sq;
  if (lane < ncols) {
    sv[lane] = sq;
    tv[lane] = isq;
  }
  __syncwarp();
#pragma unroll
  for (int c = 0; c < NM; ++c) {
    if (c < ncols) {
      if (c < lane) a[c] *= tv[c];
      else if (c == lane) a[c] = sq;
    }
  }
  return info;
}

// ---------------------------------------------------------------------------------------
// Inverse of the 32x32 lower-triangular L (T[c*ldt+r] = L[r][c], tv[c] = 1/L[c][c]) by one
// warp: 8x8 diagonal blocks by substitution (lane = block column), then two levels of
// recursive doubling inv([[A,0],[B,C]]) = [[inv A, 0], [-inv C B inv A, inv C]] on DMMA.
// Output INV[k*ldi + n] = X[n][k], X = L^-1 (the TRSM's B operand layout).
VB_DEVINL void trtri32_dmma_warp(const double* T, int ldt, const double* tv, double* INV,
                                 int ldi, double* S, int lane) {
  const int g = lane >> 2, q = lane & 3;
  for (int e = lane; e < NB * NB; e += 32) INV[(e >> 5) * ldi + (e & 31)] = 0.0;
  __syncwarp();
  {  // level 0: column c of inv(D_b), D_b = L[8b:8b+8, 8b:8b+8]
    const int b = lane >> 3, c = lane & 7, o = 8 * b;
    double x[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      double s = 0.0;
#pragma unroll
      for (int k = 0; k < i; ++k) s = fma(T[(o + k) * ldt + o + i], x[k], s);
      const double r = tv[o + i];
      x[i] = (i < c) ? 0.0 : ((i == c) ? r : -s * r);
    }
#pragma unroll
    for (int i = 0; i < 8; ++i) INV[(o + c) * ldi + o + i] = x[i];
  }
  __syncwarp();
  // level 1: blocks (2p, 2p+1), p = 0, 1: X[16p+8:, 16p:16p+8] = -inv(D_{2p+1}) B inv(D_{2p})
  {
    double t[2][2] = {{0.0, 0.0}, {0.0, 0.0}};
#pragma unroll
    for (int p = 0; p < 2; ++p) {
      const int o = 16 * p;
#pragma unroll
      for (int ks = 0; ks < 2; ++ks) {
        const double a = T[(o + ks * 4 + q) * ldt + o + 8 + g];   // B[g][k]
        const double bb = INV[(o + g) * ldi + o + ks * 4 + q];    // invA[k][g]
        dmma(t[p], a, bb);
      }
    }
#pragma unroll
    for (int p = 0; p < 2; ++p) {
      S[p * 8 * LDS_S + g * LDS_S + 2 * q] = t[p][0];
      S[p * 8 * LDS_S + g * LDS_S + 2 * q + 1] = t[p][1];
    }
    __syncwarp();
    double r[2][2] = {{0.0, 0.0}, {0.0, 0.0}};
#pragma unroll
    for (int p = 0; p < 2; ++p) {
      const int o = 16 * p;
#pragma unroll
      for (int ks = 0; ks < 2; ++ks) {
        const double a = INV[(o + 8 + ks * 4 + q) * ldi + o + 8 + g];  // invC[g][k]
        const double bb = S[p * 8 * LDS_S + (ks * 4 + q) * LDS_S + g];  // Tm[k][g]
        dmma(r[p], a, bb);
      }
    }
#pragma unroll
    for (int p = 0; p < 2; ++p) {
      const int o = 16 * p;
      INV[(o + 2 * q) * ldi + o + 8 + g] = -r[p][0];
      INV[(o + 2 * q + 1) * ldi + o + 8 + g] = -r[p][1];
    }
  }
  __syncwarp();
  // level 2: X[16:32, 0:16] = -inv(C16) L[16:32, 0:16] inv(A16)
  {
    double t[2][2][2];
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
#pragma unroll
      for (int nt = 0; nt < 2; ++nt) t[mt][nt][0] = t[mt][nt][1] = 0.0;
#pragma unroll
    for (int ks = 0; ks < 4; ++ks) {
      double a[2], bb[2];
#pragma unroll
      for (int mt = 0; mt < 2; ++mt) a[mt] = T[(ks * 4 + q) * ldt + 16 + mt * 8 + g];
#pragma unroll
      for (int nt = 0; nt < 2; ++nt) bb[nt] = INV[(nt * 8 + g) * ldi + ks * 4 + q];
#pragma unroll
      for (int mt = 0; mt < 2; ++mt)
#pragma unroll
        for (int nt = 0; nt < 2; ++nt) dmma(t[mt][nt], a[mt], bb[nt]);
    }
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
#pragma unroll
      for (int nt = 0; nt < 2; ++nt) {
        S[(mt * 8 + g) * LDS_S + nt * 8 + 2 * q] = t[mt][nt][0];
        S[(mt * 8 + g) * LDS_S + nt * 8 + 2 * q + 1] = t[mt][nt][1];
      }
    __syncwarp();
    double r[2][2][2];
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
#pragma unroll
      for (int nt = 0; nt < 2; ++nt) r[mt][nt][0] = r[mt][nt][1] = 0.0;
#pragma unroll
    for (int ks = 0; ks < 4; ++ks) {
      double a[2], bb[2];
#pragma unroll
      for (int mt = 0; mt < 2; ++mt) a[mt] = INV[(16 + ks * 4 + q) * ldi + 16 + mt * 8 + g];
#pragma unroll
      for (int nt = 0; nt < 2; ++nt) bb[nt] = S[(ks * 4 + q) * LDS_S + nt * 8 + g];
#pragma unroll
      for (int mt = 0; mt < 2; ++mt)
#pragma unroll
        for (int nt = 0; nt < 2; ++nt) dmma(r[mt][nt], a[mt], bb[nt]);
    }
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
#pragma unroll
      for (int nt = 0; nt < 2; ++nt)
#pragma unroll
        for (int h = 0; h < 2; ++h)
          INV[(nt * 8 + 2 * q + h) * ldi + 16 + mt * 8 + g] = -r[mt][nt][h];
  }
  __syncwarp();
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
      // ---- accumulators start from A's panel values (lower triangle only)
      double acc[2][4][2];
#pragma unroll
      for (int mt = 0; mt < 2; ++mt)
#pragma unroll
        for (int nt = 0; nt < 4; ++nt)
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            const int row = r0 + warp * 16 + mt * 8 + g, col = j0 + nt * 8 + 2 * q + h;
            const bool v = row < n && col < j0 + nb && row >= col;
            acc[mt][nt][h] = v ? __ldcg(A + (size_t)col * ld + row) : 0.0;
          }
      // ---- panel update on DMMA: acc -= L[r0:r0+MB, 0:j0] L[j0:j0+NB, 0:j0]^T
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
              const double a0 = -sa[0], a1 = -sa[8];
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
          s.u.e.tile[c][r] = acc[mt][nt][0];
          s.u.e.tile[c + 1][r] = acc[mt][nt][1];
        }
      __syncthreads();
      if (first) {
        const bool below = r0 + nb < n;
        if (warp == 0) {
          double a[NB];
#pragma unroll
          for (int c = 0; c < NB; ++c) a[c] = s.u.e.tile[c][lane];
          const int info = potf2_regs_warp<NB>(a, nb, lane, s.wbuf, s.sv, s.tv);
          // store the factored diagonal block (lower part; on failure incl. the pivot)
          double* Ad = A + (size_t)j0 * ld + j0;
          const int ncol = info ? info : nb;
#pragma unroll
          for (int c = 0; c < NB; ++c)
            if (c < ncol && lane >= c && lane < nb) {
              s.u.e.tile[c][lane] = a[c];
              Ad[(size_t)c * ld + lane] = a[c];
            }
          __syncwarp();
          if (!info && below) trtri32_dmma_warp(&s.u.e.tile[0][0], LDA_S, s.tv, &s.inv[0][0], LDI,
                                                s.u.e.scratch, lane);
          if (lane == 0) s.info = info;
        }
        __syncthreads();
        if (s.info) {
          if (tid == 0) *info_out = j0 + s.info;
          return;
        }
        if (!below) continue;  // no rows below the diagonal block in this pass
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
          const double a0 = s.u.e.tile[k4 * 4 + q][warp * 16 + g];
          const double a1 = s.u.e.tile[k4 * 4 + q][warp * 16 + 8 + g];
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
          s.u.e.tile[c][r] = x[mt][nt][0];
          s.u.e.tile[c + 1][r] = x[mt][nt][1];
        }
      __syncthreads();
      const int row_lo = first ? j0 + nb : r0;
      for (int idx = tid; idx < NB * MB; idx += kThreads) {
        const int c = idx / MB, r = idx % MB;
        const int row = r0 + r;
        if (c < nb && row < n && row >= row_lo) A[(size_t)(j0 + c) * ld + row] = s.u.e.tile[c][r];
      }
      __syncthreads();
    }
  }
}

__global__ void __launch_bounds__(kThreads, 3)
    potrf_blocked_kernel(const int* __restrict__ d_n, double* const* __restrict__ dA,
                         const int* __restrict__ d_ldda, int* __restrict__ d_info,
                         const Ctrl* __restrict__ ctrl_c, const int* __restrict__ order) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  BigSmem& s = *reinterpret_cast<BigSmem*>(smem_raw);
  Ctrl* ctrl = const_cast<Ctrl*>(ctrl_c);
  pdl_wait();  // the scan's outputs (order, ctrl, info) are complete and visible
  const int count_big = ctrl->count_big;
  const int tid = threadIdx.x;
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
  // work list empty: let the warp-path kernel start on this SM
  pdl_launch_dependents();
}

// ---------------------------------------------------------------------------------------
constexpr int kWarpsPerCta = 2;
struct WarpSmem {
  double w[kWarpsPerCta][64];
  double sv[kWarpsPerCta][32];
  double tv[kWarpsPerCta][32];
};

// One matrix (n <= NM) by one warp, rows in registers: one HBM read, one HBM write.
template <int NM>
VB_DEVINL void potrf_warp_matrix(double* __restrict__ A, int n, int ld, int* info_out, int lane,
                                 double* ws, double* sv, double* tv) {
  double a[NM];
#pragma unroll
  for (int c = 0; c < NM; ++c)
    a[c] = (c < n && lane >= c && lane < n) ? A[(size_t)c * ld + lane] : 0.0;
  const int info = potf2_regs_warp<NM>(a, n, lane, ws, sv, tv);
  const int ncol = info ? info : n;
#pragma unroll
  for (int c = 0; c < NM; ++c)
    if (c < ncol && lane >= c && lane < n) A[(size_t)c * ld + lane] = a[c];
  if (lane == 0 && info) *info_out = info;
  __syncwarp();
}

// Warp path: one matrix (n <= 32) per warp, whole matrix in registers.
// wait_upstream: 1 when launched directly after the scan (the only factorisation kernel),
// 0 when launched after potrf_blocked_kernel (whose CTAs passed the scan's completion
// before releasing this grid, so the scan's outputs are already visible).
__global__ void __launch_bounds__(32 * kWarpsPerCta)
    potrf_warp_kernel(const int* __restrict__ d_n, double* const* __restrict__ dA,
                      const int* __restrict__ d_ldda, int* __restrict__ d_info,
                      const Ctrl* __restrict__ ctrl_c, const int* __restrict__ order,
                      int wait_upstream) {
  __shared__ WarpSmem s;
  Ctrl* ctrl = const_cast<Ctrl*>(ctrl_c);
  if (wait_upstream) pdl_wait();
  const int count_big = *(volatile const int*)&ctrl->count_big;
  const int count_warp = *(volatile const int*)&ctrl->count_warp;
  const int lane = threadIdx.x & 31, wi = threadIdx.x >> 5;
  for (;;) {
    int w = 0;
    if (lane == 0) w = atomicAdd(&ctrl->head_warp, 1);
    w = __shfl_sync(kFull, w, 0);
    if (w >= count_warp) break;
    const int m = order[count_big + w];
    const int n = d_n[m], ld = d_ldda[m];
    if (n <= 8)
      potrf_warp_matrix<8>(dA[m], n, ld, d_info + m, lane, s.w[wi], s.sv[wi], s.tv[wi]);
    else if (n <= 16)
      potrf_warp_matrix<16>(dA[m], n, ld, d_info + m, lane, s.w[wi], s.sv[wi], s.tv[wi]);
    else
      potrf_warp_matrix<32>(dA[m], n, ld, d_info + m, lane, s.w[wi], s.sv[wi], s.tv[wi]);
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
  e = cudaFuncSetAttribute(potrf_blocked_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                           (int)sizeof(BigSmem));
  if (e != cudaSuccess) return e;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&g_occ_big, potrf_blocked_kernel, kThreads,
                                                    sizeof(BigSmem));
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
  const bool big = max_n_hint > kWarpMaxN;
  if (big) {
    cfg.blockDim = dim3(kThreads);
    cfg.gridDim = dim3(std::max(1, std::min(batch, g_num_sms * g_occ_big)));
    cfg.dynamicSmemBytes = sizeof(BigSmem);
    e = cudaLaunchKernelEx(&cfg, potrf_blocked_kernel, d_n, dA, d_ldda, d_info, ctrl, order);
    if (e != cudaSuccess) return e;
  }
  const int warps = std::max(1, batch);
  cfg.blockDim = dim3(32 * kWarpsPerCta);
  cfg.gridDim = dim3(std::max(1, std::min((warps + kWarpsPerCta - 1) / kWarpsPerCta,
                                          g_num_sms * 8)));
  cfg.dynamicSmemBytes = 0;
  return cudaLaunchKernelEx(&cfg, potrf_warp_kernel, d_n, dA, d_ldda, d_info, ctrl, order,
                            big ? 0 : 1);
}

}  // namespace vb
