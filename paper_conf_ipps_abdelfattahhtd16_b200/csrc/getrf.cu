// getrf.cu — vbatched LU with partial pivoting (DGETRF): the extension
// to LU that the paper names as future work ("the extension of this work to the LU and QR
// factorizations ... where many of the BLAS kernels proposed here can be reused out of the
// box", §V; "these kernels are a foundation for other variable-size batched
// factorizations (LU and QR)", §III-E).
//
// Built the paper's "separated" way: a host loop over panels of NB columns,
// each step = an aux kernel that derives the per-matrix sub-problem sizes and pointers on the
// GPU (the size arrays live there), a fused panel kernel (getf2 with partial
// pivoting, rows in registers), the row interchanges fused with the unit-lower solve
// A12 <- L11^-1 A12 (laswp + trsm, one warp per column), and then the SAME vbatched GEMM and
// TRSM kernels that vbatched_dgemm / vbatched_dtrsm export, in two levels, so that the trailing
// matrix is streamed once per 64 columns instead of once per 16 (rank-16 updates are HBM-bound):
//   inner step j (16 columns of the 64-column block [j0, j0 + 64), restricted to the block):
//     panel j; interchanges on the block's other columns; solve of rows j..j+15 of the block's
//     columns right of the panel; A[j+16:, j+16:j0+64] -= A21 A12 (vbatched GEMM, k = 16)
//   after the block (LAPACK DGETRF's blocked step, the block playing the panel):
//     the block's interchanges on the trailing columns (lu_laswp_block_kernel);
//     A[j0:j0+64, j0+64:] <- L11^-1 A[j0:j0+64, j0+64:] (vbatched DTRSM, unit lower 64 x 64);
//     A[j0+64:, j0+64:] -= A[j0+64:, j0:j0+64] A[j0:j0+64, j0+64:] (vbatched GEMM, k = 64).
// The interchanges of later blocks reach the columns of earlier blocks once, after the last
// step. Matrices whose panel is exhausted get size 0 in the step arrays and cost no tiles.
#include <algorithm>

#include "../../include/vbatched.h"
#include "common.cuh"
#include "internal.h"

namespace vb {
namespace {

constexpr int kLuNB = 16;        // panel width (the inner GEMMs' k)
constexpr int kLuOB = 64;        // outer block width (the trailing GEMM's k)
constexpr int kLuThreads = 256;  // panel kernel CTA
constexpr int kLuMaxRPT = 4;     // rows per thread held in registers: m - j <= 1024

struct LuStep {
  int* pm;   // panel rows (m_i - j), 0 when the matrix has no panel at step j
  int* pn;   // panel width (<= NB)
  double** P;  // panel top-left A_i(j, j)
  // BLAS problems, 2 x batch entries: inner step [0, batch) the GEMM in the block; after a
  // block [0, batch) the k = 64 trailing GEMM and [batch, 2 batch) the TRSM (gm x gn right-hand
  // side at gB, unit lower gA)
  int* gm;
  int* gn;
  int* gk;
  int* gld;  // ldda_i, twice
  double** gA;
  double** gB;
  double** gC;
};

// info: -1 m < 0, -2 n < 0, -4 ldda < max(1, m), -9 m > max_m or n > max_n; else 0.
__global__ void lu_validate_kernel(const int* __restrict__ d_m, const int* __restrict__ d_n,
                                   const int* __restrict__ d_ld, int* __restrict__ d_info, int batch,
                                   int max_m, int max_n) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < batch; i += gridDim.x * blockDim.x) {
    const int m = d_m[i], n = d_n[i], ld = d_ld[i];
    int code = 0;
    if (m < 0) code = -1;
    else if (n < 0) code = -2;
    else if (ld < (m > 1 ? m : 1)) code = -4;
    else if (m > max_m || n > max_n) code = -9;
    d_info[i] = code;
  }
}

__global__ void lu_step_kernel(const int* __restrict__ d_m, const int* __restrict__ d_n,
                               double* const* __restrict__ dA, const int* __restrict__ d_ld,
                               const int* __restrict__ d_info, int batch, int j, int j0, LuStep st) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < batch; i += gridDim.x * blockDim.x) {
    const int m = d_m[i], n = d_n[i], ld = d_ld[i];
    const int kmax = m < n ? m : n;
    const bool act = d_info[i] >= 0 && j < kmax;
    const int nb = act ? min(kLuNB, kmax - j) : 0;
    const int oend = min(j0 + kLuOB, n);  // the block's last column + 1
    st.pm[i] = act ? m - j : 0;
    st.pn[i] = nb;
    double* A = dA[i];
    st.P[i] = act ? A + (size_t)j * ld + j : A;
    const int r1 = j + nb;  // first row / column after the panel
    st.gld[i] = st.gld[batch + i] = ld;
    st.gk[i] = nb;
    st.gA[i] = act ? A + (size_t)j * ld + r1 : A;  // L21
    // the block's columns right of the panel, all rows below
    st.gm[i] = act ? m - r1 : 0;
    st.gn[i] = act ? max(0, oend - r1) : 0;
    st.gB[i] = act ? A + (size_t)r1 * ld + j : A;
    st.gC[i] = act ? A + (size_t)r1 * ld + r1 : A;
  }
}

// After the block [j0, j0 + 64): the TRSM of the block's rows of the trailing columns with the
// block's unit lower L11 (entries [batch, 2 batch)), and the k = 64 GEMM below (entries [0, batch)).
__global__ void lu_block_step_kernel(const int* __restrict__ d_m, const int* __restrict__ d_n,
                                     double* const* __restrict__ dA, const int* __restrict__ d_ld,
                                     const int* __restrict__ d_info, int batch, int j0, LuStep st) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < batch; i += gridDim.x * blockDim.x) {
    const int m = d_m[i], n = d_n[i], ld = d_ld[i];
    const int kmax = m < n ? m : n;
    const int e = j0 + kLuOB;
    const int kb = min(kLuOB, kmax - j0);  // the block's panel columns
    const bool tr = d_info[i] >= 0 && kb > 0 && e < n;      // trailing columns exist
    const bool gm = tr && e < m;                            // and rows below the block
    double* A = dA[i];
    st.gm[batch + i] = tr ? kb : 0;
    st.gn[batch + i] = tr ? n - e : 0;
    st.gA[batch + i] = tr ? A + (size_t)j0 * ld + j0 : A;
    st.gB[batch + i] = tr ? A + (size_t)e * ld + j0 : A;
    st.gm[i] = gm ? m - e : 0;
    st.gn[i] = gm ? n - e : 0;
    st.gk[i] = gm ? kLuOB : 0;
    st.gA[i] = gm ? A + (size_t)j0 * ld + e : A;
    st.gB[i] = gm ? A + (size_t)e * ld + j0 : A;
    st.gC[i] = gm ? A + (size_t)e * ld + e : A;
  }
}

// Panel factorisation with partial pivoting (LAPACK DGETF2 on the pm x pn panel): one CTA per
// matrix, thread t holds rows t, t + 256, ... (RPT of them) x NB columns in registers. Column k:
// block argmax of |a_rk| over rows r >= k (ties -> smallest row, as IDAMAX), the pivot row and
// row k trade places through shared memory, l_rk = a_rk / u_kk (IEEE division), rank-1 update
// of the panel's later columns. A zero pivot (the whole column is zero) records info = j+k+1
// (first only) and is skipped, as in DGETF2. ipiv gets the global 1-based interchanges.
template <int RPT>
__global__ void __launch_bounds__(kLuThreads, RPT == 1 ? 3 : RPT == 2 ? 2 : 1)
    lu_panel_kernel(LuStep st, const int* __restrict__ d_ld, int* const* __restrict__ d_ipiv,
                    int* __restrict__ d_info, int batch, int j) {
  __shared__ double prow[kLuNB], krow[kLuNB];
  __shared__ double wval[kLuThreads / 32];
  __shared__ int wrow[kLuThreads / 32];
  __shared__ int s_piv, s_zero;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  for (int i = blockIdx.x; i < batch; i += gridDim.x) {
    const int pm = st.pm[i], pn = st.pn[i];
    if (pm <= 0 || pn <= 0) continue;
    const int ld = d_ld[i];
    double* P = st.P[i];
    double a[RPT][kLuNB];
#pragma unroll
    for (int s = 0; s < RPT; ++s) {
      const int r = tid + s * kLuThreads;
#pragma unroll
      for (int c = 0; c < kLuNB; ++c) a[s][c] = (r < pm && c < pn) ? P[(size_t)c * ld + r] : 0.0;
    }
    if (tid == 0) s_zero = -1;
#pragma unroll
    for (int k = 0; k < kLuNB; ++k) {
      if (k >= pn) break;
      // ---- pivot search: first row of maximal |a_rk|, r >= k
      double best = -1.0;
      int brow = 0x7fffffff;
#pragma unroll
      for (int s = 0; s < RPT; ++s) {
        const int r = tid + s * kLuThreads;
        const double v = fabs(a[s][k]);
        if (r >= k && r < pm && v > best) {
          best = v;
          brow = r;
        }
      }
#pragma unroll
      for (int o = 16; o; o >>= 1) {
        const double ov = __shfl_xor_sync(kFull, best, o);
        const int orow = __shfl_xor_sync(kFull, brow, o);
        if (ov > best || (ov == best && orow < brow)) {
          best = ov;
          brow = orow;
        }
      }
      if (lane == 0) {
        wval[warp] = best;
        wrow[warp] = brow;
      }
      __syncthreads();
      if (tid == 0) {
        double bv = wval[0];
        int br = wrow[0];
        for (int w = 1; w < kLuThreads / 32; ++w)
          if (wval[w] > bv || (wval[w] == bv && wrow[w] < br)) {
            bv = wval[w];
            br = wrow[w];
          }
        s_piv = br;
        d_ipiv[i][j + k] = j + br + 1;
      }
      __syncthreads();
      const int p = s_piv;
      // ---- the pivot row and row k trade places (through shared memory)
#pragma unroll
      for (int s = 0; s < RPT; ++s) {
        const int r = tid + s * kLuThreads;
        if (r == p)
#pragma unroll
          for (int c = 0; c < kLuNB; ++c) prow[c] = a[s][c];
        if (r == k)
#pragma unroll
          for (int c = 0; c < kLuNB; ++c) krow[c] = a[s][c];
      }
      __syncthreads();
      const double piv = prow[k];
#pragma unroll
      for (int s = 0; s < RPT; ++s) {
        const int r = tid + s * kLuThreads;
        if (r == k)
#pragma unroll
          for (int c = 0; c < kLuNB; ++c) a[s][c] = prow[c];
        else if (r == p)
#pragma unroll
          for (int c = 0; c < kLuNB; ++c) a[s][c] = krow[c];
      }
      if (piv != 0.0) {
#pragma unroll
        for (int s = 0; s < RPT; ++s) {
          const int r = tid + s * kLuThreads;
          if (r > k && r < pm) {
            const double l = a[s][k] / piv;
            a[s][k] = l;
#pragma unroll
            for (int c = k + 1; c < kLuNB; ++c) a[s][c] = fma(-l, prow[c], a[s][c]);
          }
        }
      } else if (tid == 0 && s_zero < 0) {
        s_zero = k;
      }
      __syncthreads();  // prow/krow/wval are rewritten by the next column
    }
#pragma unroll
    for (int s = 0; s < RPT; ++s) {
      const int r = tid + s * kLuThreads;
      if (r < pm)
#pragma unroll
        for (int c = 0; c < kLuNB; ++c)
          if (c < pn) P[(size_t)c * ld + r] = a[s][c];
    }
    if (tid == 0 && s_zero >= 0 && d_info[i] == 0) d_info[i] = j + s_zero + 1;
    __syncthreads();
  }
}

// The composition of a step's pn sequential interchanges (LAPACK DLASWP order, ipiv[k] >= k)
// only moves rows of the set S = {j..j+pn-1} u {ipiv targets} (<= 2 pn <= 64 rows): a
// permutation of S, built by one thread. Slot t holds row srow[t]; after the interchanges row
// srow[t] holds the old value of row srow[ssrc[t]]. Slots 0..pn-1 are rows j..j+pn-1.
template <int CAP = 2 * kLuNB>
__device__ int lu_step_perm(const int* ip, int j, int pn, int* srow, int* ssrc) {
  int cnt = pn;
  int cur[CAP];  // cur[t]: slot whose original value currently sits in S[t]
  for (int t = 0; t < pn; ++t) {
    srow[t] = j + t;
    cur[t] = t;
  }
  for (int k = 0; k < pn; ++k) {
    const int r2 = ip[k] - 1;
    int t2 = -1;
    for (int t = 0; t < cnt; ++t)
      if (srow[t] == r2) t2 = t;
    if (t2 < 0) {
      t2 = cnt++;
      srow[t2] = r2;
      cur[t2] = t2;
    }
    const int x = cur[k];
    cur[k] = cur[t2];
    cur[t2] = x;
  }
  for (int t = 0; t < cnt; ++t) ssrc[t] = cur[t];
  return cnt;
}

// Row interchanges of the step's pivots on the columns right of the panel, fused with the
// triangular solve A12 <- L11^-1 A12 (DTRSM 'L','L','N','U', PAPER.md:760-812 reused as a
// fused step). One warp per column: each lane loads two rows of S (one coalesced run
// j..j+pn-1, the rest scattered), takes the value of row pi(S[t]) by a shuffle, and lanes
// 0..pn-1 (the rows j..j+pn-1, now A12's column) run the unit-lower forward substitution with
// L11 held in registers (lane t: L(j+t, j+k), k < t), one shuffle per column of L11. The
// columns left of the panel are not touched here: their interchanges are applied once, after
// the last step (lu_laswp_left_kernel).
__global__ void __launch_bounds__(256)
    lu_laswp_trsm_kernel(LuStep st, double* const* __restrict__ dA, const int* __restrict__ d_n,
                         const int* __restrict__ d_ld, int* const* __restrict__ d_ipiv, int batch,
                         int j, int j0) {
  __shared__ int srow[2 * kLuNB];  // S
  __shared__ int ssrc[2 * kLuNB];  // for slot t: the slot whose old value moves to S[t]
  __shared__ int s_cnt;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  for (int i = blockIdx.x; i < batch; i += gridDim.x) {
    const int pn = st.pn[i];
    if (pn <= 0) continue;
    const int n = d_n[i], ld = d_ld[i];
    const int cend = min(j0 + kLuOB, n);  // the block's columns only
    if (j + pn >= cend && j == j0) continue;
    double* A = dA[i];
    if (threadIdx.x == 0) s_cnt = lu_step_perm(d_ipiv[i] + j, j, pn, srow, ssrc);
    __syncthreads();
    const int cnt = s_cnt;
    const int r_lo = lane < cnt ? srow[lane] : 0, r_hi = lane + 32 < cnt ? srow[lane + 32] : 0;
    const int f_lo = lane < cnt ? ssrc[lane] : 0, f_hi = lane + 32 < cnt ? ssrc[lane + 32] : 0;
    const double* L11 = A + (size_t)j * ld + j;
    double l11[kLuNB];
#pragma unroll
    for (int k = 0; k < kLuNB; ++k) l11[k] = (k < lane && lane < pn) ? L11[(size_t)k * ld + lane] : 0.0;
    for (int c = j + pn + warp; c < cend; c += nw) {
      double* col = A + (size_t)c * ld;
      const double v_lo = lane < cnt ? col[r_lo] : 0.0;
      const double v_hi = lane + 32 < cnt ? col[r_hi] : 0.0;
      const double a_lo = __shfl_sync(kFull, v_lo, f_lo & 31), b_lo = __shfl_sync(kFull, v_hi, f_lo & 31);
      const double a_hi = __shfl_sync(kFull, v_lo, f_hi & 31), b_hi = __shfl_sync(kFull, v_hi, f_hi & 31);
      double x = f_lo < 32 ? a_lo : b_lo;
#pragma unroll
      for (int k = 0; k < kLuNB - 1; ++k) {
        const double xk = __shfl_sync(kFull, x, k);
        x = fma(-l11[k], xk, x);  // l11[k] = 0 for lanes <= k and lanes >= pn
      }
      if (lane < cnt) col[r_lo] = x;
      if (lane + 32 < cnt) col[r_hi] = f_hi < 32 ? a_hi : b_hi;
    }
    // the block's columns left of the panel: the interchanges only
    for (int c = j0 + warp; c < j; c += nw) {
      double* col = A + (size_t)c * ld;
      const double v_lo = lane < cnt ? col[r_lo] : 0.0;
      const double v_hi = lane + 32 < cnt ? col[r_hi] : 0.0;
      const double a_lo = __shfl_sync(kFull, v_lo, f_lo & 31), b_lo = __shfl_sync(kFull, v_hi, f_lo & 31);
      const double a_hi = __shfl_sync(kFull, v_lo, f_hi & 31), b_hi = __shfl_sync(kFull, v_hi, f_hi & 31);
      if (lane < cnt) col[r_lo] = f_lo < 32 ? a_lo : b_lo;
      if (lane + 32 < cnt) col[r_hi] = f_hi < 32 ? a_hi : b_hi;
    }
    __syncthreads();
  }
}

// After a block: its interchanges on the trailing columns (pure data movement). The block's kb
// pivots are composed into one permutation of the rows they touch (rows j0..j0+kb-1 plus up to kb
// pivot rows below; lu_step_perm over the whole block), so each column costs one round of loads
// and one of stores: one warp per column, the touched rows staged in a per-warp buffer.
__global__ void __launch_bounds__(256)
    lu_laswp_block_kernel(const int* __restrict__ d_m, const int* __restrict__ d_n,
                          double* const* __restrict__ dA, const int* __restrict__ d_ld,
                          int* const* __restrict__ d_ipiv, const int* __restrict__ d_info, int batch,
                          int j0) {
  constexpr int CAP = 2 * kLuOB;
  __shared__ int srow[CAP], ssrc[CAP];
  __shared__ double wbuf[8][CAP];
  __shared__ int s_cnt;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  for (int i = blockIdx.x; i < batch; i += gridDim.x) {
    if (d_info[i] < 0) continue;
    const int m = d_m[i], n = d_n[i], ld = d_ld[i];
    const int kmax = m < n ? m : n;
    const int cbeg = j0 + kLuOB;
    if (cbeg >= n || j0 >= kmax) continue;
    double* A = dA[i];
    const int kb = min(kLuOB, kmax - j0);
    __syncthreads();  // the previous matrix is done with srow / ssrc
    if (threadIdx.x == 0) s_cnt = lu_step_perm<CAP>(d_ipiv[i] + j0, j0, kb, srow, ssrc);
    __syncthreads();
    const int cnt = s_cnt;
    double* wb = wbuf[warp];
    for (int c = cbeg + warp; c < n; c += nw) {
      double* col = A + (size_t)c * ld;
      double v[CAP / 32];
#pragma unroll
      for (int u = 0; u < CAP / 32; ++u) {
        const int t = lane + 32 * u;
        v[u] = t < cnt ? col[srow[t]] : 0.0;
      }
#pragma unroll
      for (int u = 0; u < CAP / 32; ++u) wb[lane + 32 * u] = v[u];
      __syncwarp();
#pragma unroll
      for (int u = 0; u < CAP / 32; ++u) {
        const int t = lane + 32 * u;
        if (t < cnt && ssrc[t] != t) col[srow[t]] = wb[ssrc[t]];
      }
      __syncwarp();
    }
  }
}

// The interchanges on the columns left of each panel, deferred to the end (pure data movement:
// the same result as applying them step by step, LAPACK DGETRF's DLASWP on columns 0..j-1).
// Columns of 16-column step b see the interchanges of every step of the later 64-column blocks
// (those of their own block were applied at once, lu_laswp_trsm_kernel); their composition
// src_b (row r receives the value of row src_b[r]) is built backwards, src = sigma_s o src for
// the steps s of the later blocks, with sigma_s the permutation of step s's set S. Each column
// segment below the block is read once (coalesced) into shared memory and only the moved rows
// are written (measured faster than a warp per column with the moved rows in registers).
__global__ void __launch_bounds__(256)
    lu_laswp_left_kernel(const int* __restrict__ d_m, const int* __restrict__ d_n,
                         double* const* __restrict__ dA, const int* __restrict__ d_ld,
                         int* const* __restrict__ d_ipiv, const int* __restrict__ d_info, int batch) {
  __shared__ int src[kLuThreads * kLuMaxRPT];
  __shared__ double buf[kLuThreads * kLuMaxRPT];
  __shared__ int srow[2 * kLuNB], ssrc[2 * kLuNB];
  __shared__ int s_cnt;
  const int tid = threadIdx.x;
  for (int i = blockIdx.x; i < batch; i += gridDim.x) {
    if (d_info[i] < 0) continue;
    const int m = d_m[i], n = d_n[i], ld = d_ld[i];
    const int kmax = m < n ? m : n;
    const int nblk = (kmax + kLuNB - 1) / kLuNB;
    if (nblk < 2) continue;
    double* A = dA[i];
    const int* ip = d_ipiv[i];
    for (int r = tid; r < m; r += blockDim.x) src[r] = r;
    constexpr int SPB = kLuOB / kLuNB;  // steps per 64-column block
    int folded = nblk;                  // steps >= folded are in src
    for (int b = nblk - 1; b >= 0; --b) {
      // the block of step b received the interchanges of its own block's steps at once
      // (lu_laswp_trsm_kernel); it still needs those of every later block
      const int target = (b / SPB + 1) * SPB;
      while (folded > target) {
        --folded;
        const int j = folded * kLuNB, pn = min(kLuNB, kmax - j);
        __syncthreads();  // src complete, previous block's buf reads done
        if (tid == 0) s_cnt = lu_step_perm(ip + j, j, pn, srow, ssrc);
        __syncthreads();
        const int cnt = s_cnt;
        for (int r = j + tid; r < m; r += blockDim.x) {
          const int x = src[r];
          int y = x;
          for (int t = 0; t < cnt; ++t)
            if (srow[t] == x) y = srow[ssrc[t]];
          src[r] = y;
        }
      }
      if (folded == nblk) continue;  // nothing later
      const int j = folded * kLuNB;   // rows >= j may move
      for (int c = b * kLuNB; c < min((b + 1) * kLuNB, kmax); ++c) {
        double* col = A + (size_t)c * ld;
        __syncthreads();  // src updated; buf free
        for (int r = j + tid; r < m; r += blockDim.x) buf[r] = col[r];
        __syncthreads();
        for (int r = j + tid; r < m; r += blockDim.x) {
          const int y = src[r];
          if (y != r) col[r] = buf[y];
        }
      }
    }
    __syncthreads();
  }
}

template <int RPT>
cudaError_t launch_panel(int grid, LuStep st, const int* d_ld, int* const* d_ipiv, int* d_info,
                         int batch, int j, cudaStream_t stream) {
  lu_panel_kernel<RPT><<<grid, kLuThreads, 0, stream>>>(st, d_ld, d_ipiv, d_info, batch, j);
  return cudaGetLastError();
}

}  // namespace

int getrf_impl(const int* d_m, const int* d_n, double* const* dA, const int* d_ld,
               int* const* d_ipiv, int* d_info, int batch, int max_m, int max_n,
               cudaStream_t stream) {
  if (max_m > kLuThreads * kLuMaxRPT) return -8;  // panel rows are held in registers
  int dev = 0, sms = 148;
  if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  void* ws = nullptr;
  const size_t ibytes = sizeof(int) * (size_t)batch, pbytes = sizeof(double*) * (size_t)batch;
  cudaError_t e = ws_alloc(&ws, 2 * ibytes + pbytes + 8 * ibytes + 6 * pbytes + 64, stream);
  if (e != cudaSuccess) return (int)e;
  char* w = static_cast<char*>(ws);
  LuStep st;
  st.P = reinterpret_cast<double**>(w);
  st.gA = st.P + batch;
  st.gB = st.gA + 2 * batch;
  st.gC = st.gB + 2 * batch;
  st.pm = reinterpret_cast<int*>(st.gC + 2 * batch);
  st.pn = st.pm + batch;
  st.gm = st.pn + batch;
  st.gn = st.gm + 2 * batch;
  st.gk = st.gn + 2 * batch;
  st.gld = st.gk + 2 * batch;
  const int eg = std::max(1, std::min((batch + 255) / 256, 4 * sms));
  lu_validate_kernel<<<eg, 256, 0, stream>>>(d_m, d_n, d_ld, d_info, batch, max_m, max_n);
  e = cudaGetLastError();
  const int kmax = std::min(max_m, max_n);
  const int pg = std::max(1, std::min(batch, 8 * sms));
  for (int j0 = 0; j0 < kmax && e == cudaSuccess; j0 += kLuOB) {
    for (int j = j0; j < std::min(j0 + kLuOB, kmax) && e == cudaSuccess; j += kLuNB) {
      lu_step_kernel<<<eg, 256, 0, stream>>>(d_m, d_n, dA, d_ld, d_info, batch, j, j0, st);
      if ((e = cudaGetLastError()) != cudaSuccess) break;
      const int rows = max_m - j;
      if (rows <= kLuThreads) e = launch_panel<1>(pg, st, d_ld, d_ipiv, d_info, batch, j, stream);
      else if (rows <= 2 * kLuThreads) e = launch_panel<2>(pg, st, d_ld, d_ipiv, d_info, batch, j, stream);
      else e = launch_panel<4>(pg, st, d_ld, d_ipiv, d_info, batch, j, stream);
      if (e != cudaSuccess) break;
      if (j + kLuNB < std::min(j0 + kLuOB, max_n) || j > j0) {
        lu_laswp_trsm_kernel<<<pg, 256, 0, stream>>>(st, dA, d_n, d_ld, d_ipiv, batch, j, j0);
        if ((e = cudaGetLastError()) != cudaSuccess) break;
      }
      if (j + kLuNB < std::min(j0 + kLuOB, max_n)) {
        int rc = gemm_launch('N', 'N', st.gm, st.gn, st.gk, -1.0, st.gA, st.gld, st.gB, st.gld, 1.0,
                             st.gC, st.gld, batch, max_m, max_n, kLuNB, stream);
        if (rc != 0) {
          e = rc > 0 ? (cudaError_t)rc : cudaErrorInvalidValue;
          break;
        }
      }
    }
    if (e == cudaSuccess && j0 + kLuOB < max_n) {
      lu_laswp_block_kernel<<<pg, 256, 0, stream>>>(d_m, d_n, dA, d_ld, d_ipiv, d_info, batch, j0);
      if ((e = cudaGetLastError()) != cudaSuccess) break;
      lu_block_step_kernel<<<eg, 256, 0, stream>>>(d_m, d_n, dA, d_ld, d_info, batch, j0, st);
      if ((e = cudaGetLastError()) != cudaSuccess) break;
      int rc = trsm_launch('L', 'L', 'N', 'U', st.gm + batch, st.gn + batch, 1.0, st.gA + batch,
                           st.gld, st.gB + batch, st.gld, batch, kLuOB, max_n, stream);
      if (rc == 0 && j0 + kLuOB < max_m)
        rc = gemm_launch('N', 'N', st.gm, st.gn, st.gk, -1.0, st.gA, st.gld, st.gB, st.gld, 1.0,
                         st.gC, st.gld, batch, max_m, max_n, kLuOB, stream);
      if (rc != 0) e = rc > 0 ? (cudaError_t)rc : cudaErrorInvalidValue;
    }
  }
  if (e == cudaSuccess && kmax > kLuNB) {
    lu_laswp_left_kernel<<<pg, 256, 0, stream>>>(d_m, d_n, dA, d_ld, d_ipiv, d_info, batch);
    e = cudaGetLastError();
  }
  cudaError_t e2 = ws_free(ws, stream);
  return (int)(e != cudaSuccess ? e : e2);
}

}  // namespace vb

using namespace vb;

extern "C" int vbatched_dgetrf(const int* d_m, const int* d_n, double* const* dA_array,
                               const int* d_ldda, int* const* dipiv_array, int* d_info,
                               int batchCount, int max_m, int max_n, vb_stream_t stream) {
  if (batchCount < 0) return -7;
  if (max_m < 0) return -8;
  if (max_n < 0) return -9;
  if (batchCount == 0) return 0;
  return getrf_impl(d_m, d_n, dA_array, d_ldda, dipiv_array, d_info, batchCount, max_m, max_n,
                    (cudaStream_t)stream);
}
