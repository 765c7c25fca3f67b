// geqrf.cu — vbatched Householder QR (DGEQRF): the QR extension the paper
// names as future work (§V; §III-E), built from the same
// vbatched kernels in the paper's separated style.
//
// Per panel of NB = 16 columns (LAPACK DGEQRF's blocked algorithm):
//   step kernel   per-matrix sub-problem sizes and pointers, on the GPU;
//   panel kernel  DGEQR2 on the panel with the rows in registers (one CTA per matrix): per
//                 column one block reduction gives ||x||^2 and the 15 dot products the
//                 reflector needs; then V (unit lower, explicit) and the triangular factor T of
//                 the block reflector H_1..H_nb = I - V T V^T (DLARFT, forward, columnwise) go to
//                 the workspace;
//   trailing      A2 <- (I - V T V^T)^T A2 = A2 - V (T^T (V^T A2)) as three calls of the
//                 library's vbatched DGEMM (DMMA): W1 = V^T A2, W2 = T^T W1, A2 -= V W2.
#include <algorithm>

#include "../../include/vbatched.h"
#include "common.cuh"
#include "internal.h"

namespace vb {
namespace {

constexpr int kQrNB = 16;
constexpr int kQrThreads = 256;
constexpr int kQrMaxRPT = 4;  // panel rows in registers: m - j <= 1024

struct QrStep {
  int *pm, *pn, *rn, *vld, *sixteen;
  double **P, **A2, **V, **W1, **W2, **T;
};

// info: -1 m < 0, -2 n < 0, -4 ldda < max(1, m), -9 beyond max_m / max_n; workspace offsets
// (16 m + 32 n + 256 doubles per matrix) by an exclusive prefix sum in one CTA.
__global__ void __launch_bounds__(1024, 1)
    qr_prep_kernel(const int* __restrict__ d_m, const int* __restrict__ d_n,
                   const int* __restrict__ d_ld, int* __restrict__ d_info, int batch, int max_m,
                   int max_n, size_t* __restrict__ woff, int* __restrict__ sixteen) {
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
      if (code == 0) sz = 16 * (size_t)m + 32 * (size_t)n + 256;
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
                               double* __restrict__ wbase, int batch, int j, QrStep st) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < batch; i += gridDim.x * blockDim.x) {
    const int m = d_m[i], n = d_n[i], ld = d_ld[i];
    const int kmax = m < n ? m : n;
    const bool act = d_info[i] >= 0 && j < kmax;
    const int nb = act ? min(kQrNB, kmax - j) : 0;
    st.pm[i] = act ? m - j : 0;
    st.pn[i] = nb;
    st.rn[i] = act ? n - j - nb : 0;
    st.vld[i] = act ? m - j : 1;
    double* A = dA[i];
    double* w = wbase + woff[i];
    st.P[i] = act ? A + (size_t)j * ld + j : A;
    st.A2[i] = act ? A + (size_t)(j + nb) * ld + j : A;
    st.V[i] = w;                                  // 16 m doubles (ld m - j this step)
    st.W1[i] = w + 16 * (size_t)max(m, 0);        // 16 n
    st.W2[i] = st.W1[i] + 16 * (size_t)max(n, 0); // 16 n
    st.T[i] = st.W2[i] + 16 * (size_t)max(n, 0);  // 16 x 16
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
__global__ void __launch_bounds__(kQrThreads, RPT == 1 ? 3 : 1)
    qr_panel_kernel(QrStep st, const int* __restrict__ d_ld, double* const* __restrict__ d_tau,
                    int batch, int j) {
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
            V[(size_t)c * pm + r] = (r == c) ? 1.0 : (r < c ? 0.0 : a[s][c]);
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
                            int j, cudaStream_t stream) {
  qr_panel_kernel<RPT><<<grid, kQrThreads, 0, stream>>>(st, d_ld, d_tau, batch, j);
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
  const size_t wdoubles = (size_t)batch * (16 * (size_t)max_m + 32 * (size_t)max_n + 256);
  const size_t ib = sizeof(int) * (size_t)batch, pb = sizeof(double*) * (size_t)batch;
  const size_t meta = 5 * ib + 6 * pb + sizeof(size_t) * (size_t)batch;
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
  size_t* woff = reinterpret_cast<size_t*>(st.T + batch);
  st.pm = reinterpret_cast<int*>(woff + batch);
  st.pn = st.pm + batch;
  st.rn = st.pn + batch;
  st.vld = st.rn + batch;
  st.sixteen = st.vld + batch;
  double* wbase = reinterpret_cast<double*>(w + ((meta + 255) & ~(size_t)255));
  qr_prep_kernel<<<1, 1024, 0, stream>>>(d_m, d_n, d_ld, d_info, batch, max_m, max_n, woff,
                                         st.sixteen);
  e = cudaGetLastError();
  const int eg = std::max(1, std::min((batch + 255) / 256, 4 * sms));
  const int pg = std::max(1, std::min(batch, 8 * sms));
  const int kmax = std::min(max_m, max_n);
  for (int j = 0; j < kmax && e == cudaSuccess; j += kQrNB) {
    qr_step_kernel<<<eg, 256, 0, stream>>>(d_m, d_n, dA, d_ld, d_info, woff, wbase, batch, j, st);
    if ((e = cudaGetLastError()) != cudaSuccess) break;
    const int rows = max_m - j;
    if (rows <= kQrThreads) e = launch_qr_panel<1>(pg, st, d_ld, d_tau, batch, j, stream);
    else if (rows <= 2 * kQrThreads) e = launch_qr_panel<2>(pg, st, d_ld, d_tau, batch, j, stream);
    else e = launch_qr_panel<4>(pg, st, d_ld, d_tau, batch, j, stream);
    if (e != cudaSuccess) break;
    if (j + kQrNB < max_n) {  // trailing update with the block reflector
      int rc = gemm_launch('T', 'N', st.pn, st.rn, st.pm, 1.0, st.V, st.vld, st.A2, d_ld, 0.0,
                           st.W1, st.sixteen, batch, kQrNB, max_n, max_m, stream);
      if (rc == 0)
        rc = gemm_launch('T', 'N', st.pn, st.rn, st.pn, 1.0, st.T, st.sixteen, st.W1, st.sixteen,
                         0.0, st.W2, st.sixteen, batch, kQrNB, max_n, kQrNB, stream);
      if (rc == 0)
        rc = gemm_launch('N', 'N', st.pm, st.rn, st.pn, -1.0, st.V, st.vld, st.W2, st.sixteen, 1.0,
                         st.A2, d_ld, batch, max_m, max_n, kQrNB, stream);
      if (rc != 0) {
        e = rc > 0 ? (cudaError_t)rc : cudaErrorInvalidValue;
        break;
      }
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
  return geqrf_impl(d_m, d_n, dA_array, d_ldda, dtau_array, d_info, batchCount, max_m, max_n,
                    (cudaStream_t)stream);
}
