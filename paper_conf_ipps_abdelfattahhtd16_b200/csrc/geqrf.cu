// geqrf.cu — vbatched Householder QR (DGEQRF): the QR extension the paper
// names as future work (§V; §III-E), built from the same
// vbatched kernels in the paper's separated style.
//
// LAPACK DGEQRF's blocked algorithm in two levels, so that the trailing matrix is streamed three
// times per 64 columns instead of per 16 (its updates are HBM-bound). Per 16-column step j of a
// 64-column block [j0, j0 + 64):
//   step kernel   per-matrix sub-problem sizes and pointers, on the GPU;
//   panel kernel  DGEQR2 on the panel with the rows in registers (one CTA per matrix): per
//                 column one block reduction gives ||x||^2 and the 15 dot products the
//                 reflector needs; then V (unit lower, explicit) goes to the block's V in the
//                 workspace and the triangular factor T of the panel's block reflector
//                 H_1..H_nb = I - V T V^T (DLARFT, forward, columnwise) next to it;
//   block update  A2 <- (I - V T V^T)^T A2 = A2 - V (T^T (V^T A2)) on the block's columns right
//                 of the panel, three calls of the library's vbatched DGEMM (DMMA).
// After the block: G = Vb^T Vb (vbatched DGEMM), the block's 64 x 64 T from G and tau (DLARFT,
// qr_larft_kernel), and the same three GEMMs with k = 64 on the trailing columns.
#include <algorithm>

#include "../../include/vbatched.h"
#include "common.cuh"
#include "internal.h"

namespace vb {
namespace {

constexpr int kQrNB = 16;
constexpr int kQrOB = 64;  // outer block width
constexpr int kQrThreads = 256;
constexpr int kQrMaxRPT = 4;  // panel rows in registers: m - j <= 1024

struct QrStep {
  int *pm, *pn, *rn, *vld, *sixteen, *sixtyfour;
  double **P, **A2, **V, **W1, **W2, **T;
  // after a block: kb reflectors, bm = m - j0 rows, bn trailing columns
  int *kb, *bm, *bn;
  double **Vb, **G, **Tb, **A2b;
};
// per-matrix workspace (doubles): V 64 m | W1 64 n | W2 64 n | T 16 x 16 | Tb 64 x 64 | G 64 x 64
VB_DEVINL size_t qr_ws_doubles(int m, int n) {
  return (size_t)kQrOB * m + 2 * (size_t)kQrOB * n + kQrNB * kQrNB + 2 * kQrOB * kQrOB;
}

// info: -1 m < 0, -2 n < 0, -4 ldda < max(1, m), -9 beyond max_m / max_n; workspace offsets
// (16 m + 32 n + 256 doubles per matrix) by an exclusive prefix sum in one CTA.
__global__ void __launch_bounds__(1024, 1)
    qr_prep_kernel(const int* __restrict__ d_m, const int* __restrict__ d_n,
                   const int* __restrict__ d_ld, int* __restrict__ d_info, int batch, int max_m,
                   int max_n, size_t* __restrict__ woff, int* __restrict__ sixteen,
                   int* __restrict__ sixtyfour) {
  __shared__ size_t wsum[32];
  __shared__ size_t carry;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) carry = 0;
  __syncthreads();
  for (int base = 0; base < batch; base += 1024) {
    const int i = base + tid;
    size_t sz = 0;
    if (i < batch) {
      const int m = d_m[i], n = d_n[i], ld = d_ld[i];
      int code = 0;
      if (m < 0) code = -1;
      else if (n < 0) code = -2;
      else if (ld < (m > 1 ? m : 1)) code = -4;
      else if (m > max_m || n > max_n) code = -9;
      d_info[i] = code;
      sixteen[i] = kQrNB;
      sixtyfour[i] = kQrOB;
      if (code == 0) sz = qr_ws_doubles(m, n);
    }
    size_t incl = sz;
    for (int o = 1; o < 32; o <<= 1) {
      const size_t v = __shfl_up_sync(kFull, incl, o);
      if (lane >= o) incl += v;
    }
    if (lane == 31) wsum[warp] = incl;
    __syncthreads();
    if (warp == 0) {
      const size_t v = wsum[lane];
      size_t w = v;
      for (int o = 1; o < 32; o <<= 1) {
        const size_t t = __shfl_up_sync(kFull, w, o);
        if (lane >= o) w += t;
      }
      wsum[lane] = w - v;
    }
    __syncthreads();
    if (i < batch) woff[i] = carry + wsum[warp] + incl - sz;
    __syncthreads();
    if (tid == 1023) carry += wsum[31] + incl;
    __syncthreads();
  }
}

__global__ void qr_step_kernel(const int* __restrict__ d_m, const int* __restrict__ d_n,
                               double* const* __restrict__ dA, const int* __restrict__ d_ld,
                               const int* __restrict__ d_info, const size_t* __restrict__ woff,
                               double* __restrict__ wbase, int batch, int j, int j0, QrStep st) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < batch; i += gridDim.x * blockDim.x) {
    const int m = d_m[i], n = d_n[i], ld = d_ld[i];
    const int kmax = m < n ? m : n;
    const bool act = d_info[i] >= 0 && j < kmax;
    const int nb = act ? min(kQrNB, kmax - j) : 0;
    const int cend = min(j0 + kQrOB, n);  // the block's columns only
    st.pm[i] = act ? m - j : 0;
    st.pn[i] = nb;
    st.rn[i] = act ? max(0, cend - j - nb) : 0;
    st.vld[i] = act ? m - j0 : 1;
    double* A = dA[i];
    double* w = wbase + woff[i];
    const size_t mm = (size_t)max(m, 0), nn = (size_t)max(n, 0);
    st.P[i] = act ? A + (size_t)j * ld + j : A;
    st.A2[i] = act ? A + (size_t)(j + nb) * ld + j : A;
    // the block's V (ld m - j0): this panel's columns start at (j - j0, j - j0)
    st.V[i] = act ? w + (size_t)(j - j0) * (m - j0) + (j - j0) : w;
    st.W1[i] = w + kQrOB * mm;
    st.W2[i] = st.W1[i] + kQrOB * nn;
    st.T[i] = st.W2[i] + kQrOB * nn;  // 16 x 16
  }
}

// After the block [j0, j0 + 64): pointers and sizes of G = Vb^T Vb, the block T and the trailing
// update (rows j0.., columns j0 + 64..).
__global__ void qr_block_step_kernel(const int* __restrict__ d_m, const int* __restrict__ d_n,
                                     double* const* __restrict__ dA, const int* __restrict__ d_ld,
                                     const int* __restrict__ d_info, const size_t* __restrict__ woff,
                                     double* __restrict__ wbase, int batch, int j0, QrStep st) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < batch; i += gridDim.x * blockDim.x) {
    const int m = d_m[i], n = d_n[i], ld = d_ld[i];
    const int kmax = m < n ? m : n;
    const int e = j0 + kQrOB;
    const bool act = d_info[i] >= 0 && j0 < kmax && e < n;
    double* A = dA[i];
    double* w = wbase + woff[i];
    const size_t mm = (size_t)max(m, 0), nn = (size_t)max(n, 0);
    st.kb[i] = act ? min(kQrOB, kmax - j0) : 0;
    st.bm[i] = act ? m - j0 : 0;
    st.bn[i] = act ? n - e : 0;
    st.vld[i] = act ? m - j0 : 1;
    st.Vb[i] = w;
    st.W1[i] = w + kQrOB * mm;
    st.W2[i] = st.W1[i] + kQrOB * nn;
    st.Tb[i] = st.W2[i] + kQrOB * nn + kQrNB * kQrNB;
    st.G[i] = st.Tb[i] + kQrOB * kQrOB;
    st.A2b[i] = act ? A + (size_t)e * ld + j0 : A;
  }
}

// The block reflector's T (kb x kb, ld 64) from G = Vb^T Vb and tau (LAPACK DLARFT, forward,
// columnwise): T(c, c) = tau_c, T(0:c, c) = -tau_c T(0:c, 0:c) G(0:c, c). One CTA per matrix,
// thread r owns row r; one barrier per column.
__global__ void __launch_bounds__(64)
    qr_larft_kernel(QrStep st, double* const* __restrict__ d_tau, int batch, int j0) {
  __shared__ double T[kQrOB][kQrOB + 1];  // T[col][row]
  const int r = threadIdx.x;
  for (int i = blockIdx.x; i < batch; i += gridDim.x) {
    const int kb = st.kb[i];
    if (kb <= 0) continue;
    const double* G = st.G[i];
    const double* tau = d_tau[i] + j0;
    for (int c = 0; c < kb; ++c) {
      double v = 0.0;
      if (r < c) {
        double sacc = 0.0;
        for (int q = r; q < c; ++q) sacc = fma(T[q][r], G[(size_t)c * kQrOB + q], sacc);
        v = -tau[c] * sacc;
      } else if (r == c) {
        v = tau[c];
      }
      T[c][r] = v;
      __syncthreads();
    }
    double* Tg = st.Tb[i];
    for (int c = 0; c < kb; ++c) Tg[(size_t)c * kQrOB + r] = r < kb ? T[c][r] : 0.0;
    __syncthreads();
  }
}

// Block-wide sums of 16 per-thread partials (all threads get them in `out`). Within a warp by
// recursive halving: at each of the exchange levels 16, 8, 4, 2 a lane keeps one half of its
// values and adds the partner's copy of that half (8 + 4 + 2 + 1 shuffles instead of 16 x 5),
// after which lane l holds value 8 b4 + 4 b3 + 2 b2 + b1 (b_i = bit i of l) summed over the warp
// (lanes l and l ^ 1 alike). Across the 8 warps: 128 threads, one per (value, warp), 3 shuffles.
VB_DEVINL void block_sum16(double (&p)[kQrNB], double (*red)[kQrNB], double* out, int tid) {
  static_assert(kQrNB == 16 && kQrThreads == 256, "shapes");
  const int lane = tid & 31, warp = tid >> 5;
  double v8[8], v4[4], v2[2];
  bool hi = lane & 16;
#pragma unroll
  for (int k = 0; k < 8; ++k) {
    const double send = hi ? p[k] : p[k + 8], keep = hi ? p[k + 8] : p[k];
    v8[k] = keep + __shfl_xor_sync(kFull, send, 16);
  }
  hi = lane & 8;
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    const double send = hi ? v8[k] : v8[k + 4], keep = hi ? v8[k + 4] : v8[k];
    v4[k] = keep + __shfl_xor_sync(kFull, send, 8);
  }
  hi = lane & 4;
#pragma unroll
  for (int k = 0; k < 2; ++k) {
    const double send = hi ? v4[k] : v4[k + 2], keep = hi ? v4[k + 2] : v4[k];
    v2[k] = keep + __shfl_xor_sync(kFull, send, 4);
  }
  hi = lane & 2;
  double v1 = (hi ? v2[1] : v2[0]) + __shfl_xor_sync(kFull, hi ? v2[0] : v2[1], 2);
  v1 += __shfl_xor_sync(kFull, v1, 1);
  const int idx = ((lane >> 4) & 1) * 8 + ((lane >> 3) & 1) * 4 + ((lane >> 2) & 1) * 2 + ((lane >> 1) & 1);
  if ((lane & 1) == 0) red[warp][idx] = v1;
  __syncthreads();
  if (tid < 128) {
    double x = red[tid & 7][tid >> 3];
    x += __shfl_xor_sync(kFull, x, 1);
    x += __shfl_xor_sync(kFull, x, 2);
    x += __shfl_xor_sync(kFull, x, 4);
    if ((tid & 7) == 0) out[tid >> 3] = x;
  }
  __syncthreads();
}

template <int RPT>
__global__ void __launch_bounds__(kQrThreads, RPT == 1 ? 3 : RPT == 2 ? 2 : 1)
    qr_panel_kernel(QrStep st, const int* __restrict__ d_ld, double* const* __restrict__ d_tau,
                    int batch, int j, int j0) {
  __shared__ double red[kQrThreads / 32][kQrNB];
  __shared__ double sums[kQrNB], krow[kQrNB];
  __shared__ double s_tau[kQrNB], s_G[kQrNB][kQrNB + 1], s_T[kQrNB][kQrNB + 1];
  static_assert(kQrThreads == kQrNB * kQrNB, "one thread per entry of T");
  const int tid = threadIdx.x;
  for (int i = blockIdx.x; i < batch; i += gridDim.x) {
    const int pm = st.pm[i], pn = st.pn[i];
    if (pm <= 0 || pn <= 0) continue;
    const int ld = d_ld[i];
    double* P = st.P[i];
    double a[RPT][kQrNB];
#pragma unroll
    for (int s = 0; s < RPT; ++s) {
      const int r = tid + s * kQrThreads;
#pragma unroll
      for (int c = 0; c < kQrNB; ++c) a[s][c] = (r < pm && c < pn) ? P[(size_t)c * ld + r] : 0.0;
    }
#pragma unroll
    for (int k = 0; k < kQrNB; ++k) {
      if (k >= pn) break;
      // partial sums over rows r > k: x_r x_r (c = k) and x_r a_rc (c > k); row k published
      double p[kQrNB];
#pragma unroll
      for (int c = 0; c < kQrNB; ++c) p[c] = 0.0;
#pragma unroll
      for (int s = 0; s < RPT; ++s) {
        const int r = tid + s * kQrThreads;
        if (r > k && r < pm)
#pragma unroll
          for (int c = 0; c < kQrNB; ++c)
            if (c >= k) p[c] = fma(a[s][k], a[s][c], p[c]);
        if (r == k)
#pragma unroll
          for (int c = 0; c < kQrNB; ++c) krow[c] = a[s][c];
      }
      block_sum16(p, red, sums, tid);
      const double alpha = krow[k], xn2 = sums[k];
      double tau = 0.0, beta = alpha, rden = 0.0;
      if (xn2 != 0.0) {  // DLARFG
        const double rr = sqrt(fma(alpha, alpha, xn2));
        beta = alpha >= 0.0 ? -rr : rr;
        tau = (beta - alpha) / beta;
        rden = 1.0;  // marker: v_r = x_r / (alpha - beta)
      }
      const double den = alpha - beta;
      if (tid == 0) {
        s_tau[k] = tau;
        d_tau[i][j + k] = tau;
      }
#pragma unroll
      for (int s = 0; s < RPT; ++s) {
        const int r = tid + s * kQrThreads;
        if (rden != 0.0) {
          if (r > k && r < pm) {
            const double v = a[s][k] / den;
            a[s][k] = v;
#pragma unroll
            for (int c = 0; c < kQrNB; ++c)
              if (c > k) {
                const double w = krow[c] + sums[c] / den;  // v^T a_c with v_k = 1
                a[s][c] = fma(-tau * w, v, a[s][c]);
              }
          } else if (r == k) {
            a[s][k] = beta;
#pragma unroll
            for (int c = 0; c < kQrNB; ++c)
              if (c > k) a[s][c] -= tau * (krow[c] + sums[c] / den);
          }
        }
      }
      __syncthreads();  // krow / sums are rewritten by the next column
    }
    // panel back to global (R on/above the diagonal, v below); V (unit lower, explicit) to the
    // workspace; partial Gram sums V^T V for DLARFT
    double* V = st.V[i];
    const int vld = st.vld[i];
    {  // the block's rows above this panel are zero in its V columns
      const int top = j - j0;
      for (int e = tid; e < top * pn; e += kQrThreads)
        V[(size_t)(e / top) * vld - top + e % top] = 0.0;
    }
    double g[kQrNB];
#pragma unroll
    for (int c = 0; c < kQrNB; ++c) g[c] = 0.0;
    double (*G)[kQrNB + 1] = s_G;
#pragma unroll
    for (int b = 1; b < kQrNB; ++b) {  // column b of G: V[:, c]^T V[:, b], c < b
      if (b >= pn) break;
#pragma unroll
      for (int c = 0; c < kQrNB; ++c) g[c] = 0.0;
#pragma unroll
      for (int s = 0; s < RPT; ++s) {
        const int r = tid + s * kQrThreads;
        if (r < pm && r >= b) {
          const double vb = (r == b) ? 1.0 : a[s][b];
#pragma unroll
          for (int c = 0; c < kQrNB; ++c)
            if (c < b) g[c] = fma((r == c) ? 1.0 : a[s][c], vb, g[c]);
        }
      }
      block_sum16(g, red, sums, tid);
      if (tid < kQrNB) G[tid][b] = sums[tid];
    }
#pragma unroll
    for (int s = 0; s < RPT; ++s) {
      const int r = tid + s * kQrThreads;
      if (r < pm)
#pragma unroll
        for (int c = 0; c < kQrNB; ++c)
          if (c < pn) {
            P[(size_t)c * ld + r] = a[s][c];
            V[(size_t)c * vld + r] = (r == c) ? 1.0 : (r < c ? 0.0 : a[s][c]);
          }
    }
    __syncthreads();
    // DLARFT (forward, columnwise): T[0:c, c] = -tau_c T[0:c, 0:c] G[0:c, c], in shared memory,
    // thread r < 16 owning row r of T (it reads only its own row: no barrier between columns);
    // then the whole 16 x 16 T to the workspace. (A single thread doing this through global
    // memory was a chain of ~700 dependent L2 round trips, most of the panel kernel's time.)
    if (tid < kQrNB) {
      const int r = tid;
      for (int c = 0; c < kQrNB; ++c) {
        double v = 0.0;
        if (c < pn) {
          if (r < c) {
            double sacc = 0.0;
            for (int q = r; q < c; ++q) sacc += s_T[q][r] * G[q][c];
            v = -s_tau[c] * sacc;
          } else if (r == c) {
            v = s_tau[c];
          }
        }
        s_T[c][r] = v;
      }
    }
    __syncthreads();
    st.T[i][tid] = s_T[tid / kQrNB][tid % kQrNB];  // kQrThreads == 16 x 16
    __syncthreads();
  }
}

template <int RPT>
cudaError_t launch_qr_panel(int grid, QrStep st, const int* d_ld, double* const* d_tau, int batch,
                            int j, int j0, cudaStream_t stream) {
  qr_panel_kernel<RPT><<<grid, kQrThreads, 0, stream>>>(st, d_ld, d_tau, batch, j, j0);
  return cudaGetLastError();
}

}  // namespace

int geqrf_impl(const int* d_m, const int* d_n, double* const* dA, const int* d_ld,
               double* const* d_tau, int* d_info, int batch, int max_m, int max_n,
               cudaStream_t stream) {
  if (max_m > kQrThreads * kQrMaxRPT) return -8;
  int dev = 0, sms = 148;
  if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  // host-side upper bound of the per-matrix workspace (the device prefix sum fills it exactly)
  const size_t wdoubles = (size_t)batch * ((size_t)kQrOB * max_m + 2 * (size_t)kQrOB * max_n +
                                           kQrNB * kQrNB + 2 * kQrOB * kQrOB);
  const size_t ib = sizeof(int) * (size_t)batch, pb = sizeof(double*) * (size_t)batch;
  const size_t meta = 9 * ib + 10 * pb + sizeof(size_t) * (size_t)batch;
  void* ws = nullptr;
  cudaError_t e = ws_alloc(&ws, ((meta + 255) & ~(size_t)255) + 8 * wdoubles, stream);
  if (e != cudaSuccess) return (int)e;
  char* w = static_cast<char*>(ws);
  QrStep st;
  st.P = reinterpret_cast<double**>(w);
  st.A2 = st.P + batch;
  st.V = st.A2 + batch;
  st.W1 = st.V + batch;
  st.W2 = st.W1 + batch;
  st.T = st.W2 + batch;
  st.Vb = st.T + batch;
  st.G = st.Vb + batch;
  st.Tb = st.G + batch;
  st.A2b = st.Tb + batch;
  size_t* woff = reinterpret_cast<size_t*>(st.A2b + batch);
  st.pm = reinterpret_cast<int*>(woff + batch);
  st.pn = st.pm + batch;
  st.rn = st.pn + batch;
  st.vld = st.rn + batch;
  st.sixteen = st.vld + batch;
  st.sixtyfour = st.sixteen + batch;
  st.kb = st.sixtyfour + batch;
  st.bm = st.kb + batch;
  st.bn = st.bm + batch;
  double* wbase = reinterpret_cast<double*>(w + ((meta + 255) & ~(size_t)255));
  qr_prep_kernel<<<1, 1024, 0, stream>>>(d_m, d_n, d_ld, d_info, batch, max_m, max_n, woff,
                                         st.sixteen, st.sixtyfour);
  e = cudaGetLastError();
  const int eg = std::max(1, std::min((batch + 255) / 256, 4 * sms));
  const int pg = std::max(1, std::min(batch, 8 * sms));
  const int kmax = std::min(max_m, max_n);
  for (int j0 = 0; j0 < kmax && e == cudaSuccess; j0 += kQrOB) {
    for (int j = j0; j < std::min(j0 + kQrOB, kmax) && e == cudaSuccess; j += kQrNB) {
      qr_step_kernel<<<eg, 256, 0, stream>>>(d_m, d_n, dA, d_ld, d_info, woff, wbase, batch, j, j0, st);
      if ((e = cudaGetLastError()) != cudaSuccess) break;
      const int rows = max_m - j;
      if (rows <= kQrThreads) e = launch_qr_panel<1>(pg, st, d_ld, d_tau, batch, j, j0, stream);
      else if (rows <= 2 * kQrThreads) e = launch_qr_panel<2>(pg, st, d_ld, d_tau, batch, j, j0, stream);
      else e = launch_qr_panel<4>(pg, st, d_ld, d_tau, batch, j, j0, stream);
      if (e != cudaSuccess) break;
      // the block's columns right of the panel (a last panel narrower than 16 columns still has
      // the block's remaining columns on its right)
      if (j + 1 < std::min(j0 + kQrOB, max_n)) {
        int rc = gemm_launch('T', 'N', st.pn, st.rn, st.pm, 1.0, st.V, st.vld, st.A2, d_ld, 0.0,
                             st.W1, st.sixteen, batch, kQrNB, kQrOB, max_m, stream);
        if (rc == 0)
          rc = gemm_launch('T', 'N', st.pn, st.rn, st.pn, 1.0, st.T, st.sixteen, st.W1, st.sixteen,
                           0.0, st.W2, st.sixteen, batch, kQrNB, kQrOB, kQrNB, stream);
        if (rc == 0)
          rc = gemm_launch('N', 'N', st.pm, st.rn, st.pn, -1.0, st.V, st.vld, st.W2, st.sixteen, 1.0,
                           st.A2, d_ld, batch, max_m, kQrOB, kQrNB, stream);
        if (rc != 0) {
          e = rc > 0 ? (cudaError_t)rc : cudaErrorInvalidValue;
          break;
        }
      }
    }
    if (e == cudaSuccess && j0 + kQrOB < max_n) {  // the block reflector on the trailing columns
      qr_block_step_kernel<<<eg, 256, 0, stream>>>(d_m, d_n, dA, d_ld, d_info, woff, wbase, batch,
                                                   j0, st);
      if ((e = cudaGetLastError()) != cudaSuccess) break;
      int rc = gemm_launch('T', 'N', st.kb, st.kb, st.bm, 1.0, st.Vb, st.vld, st.Vb, st.vld, 0.0,
                           st.G, st.sixtyfour, batch, kQrOB, kQrOB, max_m, stream);
      if (rc == 0) {
        qr_larft_kernel<<<pg, 64, 0, stream>>>(st, d_tau, batch, j0);
        if ((e = cudaGetLastError()) != cudaSuccess) break;
        rc = gemm_launch('T', 'N', st.kb, st.bn, st.bm, 1.0, st.Vb, st.vld, st.A2b, d_ld, 0.0,
                         st.W1, st.sixtyfour, batch, kQrOB, max_n, max_m, stream);
      }
      if (rc == 0)
        rc = gemm_launch('T', 'N', st.kb, st.bn, st.kb, 1.0, st.Tb, st.sixtyfour, st.W1,
                         st.sixtyfour, 0.0, st.W2, st.sixtyfour, batch, kQrOB, max_n, kQrOB, stream);
      if (rc == 0)
        rc = gemm_launch('N', 'N', st.bm, st.bn, st.kb, -1.0, st.Vb, st.vld, st.W2, st.sixtyfour,
                         1.0, st.A2b, d_ld, batch, max_m, max_n, kQrOB, stream);
      if (rc != 0) e = rc > 0 ? (cudaError_t)rc : cudaErrorInvalidValue;
    }
  }
  cudaError_t e2 = ws_free(ws, stream);
  return (int)(e != cudaSuccess ? e : e2);
}

}  // namespace vb

using namespace vb;

extern "C" int vbatched_dgeqrf(const int* d_m, const int* d_n, double* const* dA_array,
                               const int* d_ldda, double* const* dtau_array, int* d_info,
                               int batchCount, int max_m, int max_n, vb_stream_t stream) {
  if (batchCount < 0) return -7;
  if (max_m < 0) return -8;
  if (max_n < 0) return -9;
  if (batchCount == 0) return 0;
  // The per-matrix workspace (64 m + 128 n + 8448 doubles at the bounds: 1.5 MB for 1024 x 1024)
  // is bounded to ~4 GiB per call by slicing the batch; matrices are independent, so a slice is
  // the same call on a sub-range of the arrays.
  const size_t per = ((size_t)kQrOB * max_m + 2 * (size_t)kQrOB * max_n + kQrNB * kQrNB +
                      2 * kQrOB * kQrOB) * sizeof(double) + 256;
  const int slice = (int)std::max<size_t>(1, std::min<size_t>(batchCount, (4ull << 30) / per));
  for (int b0 = 0; b0 < batchCount; b0 += slice) {
    const int cnt = std::min(slice, batchCount - b0);
    const int rc = geqrf_impl(d_m + b0, d_n + b0, dA_array + b0, d_ldda + b0, dtau_array + b0,
                              d_info + b0, cnt, max_m, max_n, (cudaStream_t)stream);
    if (rc != 0) return rc;
  }
  return 0;
}
