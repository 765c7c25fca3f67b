// zpotrf.cu — vbatched complex Cholesky A_i = L_i L_i^H (ZPOTRF: complex<double> storage;
// CPOTRF: complex<float> storage, FP64 arithmetic inside, like vbatched_spotrf). SURVEY.md §8(f)
// NEXT-3: the paper's framework "supports complex precisions" (§IV-A).
//
// Same problem statement as vbatched_dpotrf with Hermitian
// matrices: l_jj = sqrt(Re a_jj - sum |l_jk|^2) (the diagonal's imaginary part is ignored and
// the factor's is stored as 0, as LAPACK ZPOTRF), l_ij = (a_ij - sum l_ik conj(l_jk)) / l_jj.
//
// One 4-warp CTA per matrix (persistent, matrices in the scan's LPT order), left-looking with
// NB = 16 panels (the paper's Algorithm 1):
//   warp 0   diagonal 16x16 block: panel update (complex DMMA), POTF2 in registers, L11^-1 by
//            substitution (lane = column), published through shared memory (named barrier);
//   warps 1-3 the 16-row strips below: panel update from L2 (complex DMMA), TRSM
//            X = C L11^-H (complex DMMA against the inverse), store.
// A complex product on the FP64 tensor cores is four real DMMA m8n8k4:
//   (Ar + i Ai)(Br - i Bi)^T:  re += Ar Br^T + Ai Bi^T,   im += Ai Br^T - Ar Bi^T.
#include <algorithm>

#include "../../include/vbatched.h"
#include "common.cuh"
#include "internal.h"

namespace vb {
namespace {

constexpr int kZNB = 16;
constexpr int kZLD = 17;  // complex leading dimension of the shared 16x16 blocks

template <typename E2>
struct Real;
template <>
struct Real<double2> {
  using T = double;
};
template <>
struct Real<float2> {
  using T = float;
};

struct ZSmem {
  double2 T[kZNB][kZLD];    // diagonal block T[c][r] = L(r, c) (lower)
  double2 inv[kZNB][kZLD];  // inv[k][c] = Linv(c, k): the TRSM's B operand (conjugated there)
  double2 col[kZNB];        // POTF2 column broadcast
  int item;
  int info[2];  // panel p's pivot status in info[p & 1]: read by every warp at the end of panel
                // p while warp 0 may already write panel p+1's
};

// L(r, c) (r >= c) of matrix storage A with uplo: 'L' keeps L, 'U' keeps U = L^H, so L(r, c) =
// conj(U(c, r)).
template <bool UP, typename E2>
VB_DEVINL double2 ld_l(const E2* __restrict__ A, int r, int c, int ld) {
  const E2 v = __ldcg(A + gix<UP>(r, c, ld));
  return make_double2((double)v.x, UP ? -(double)v.y : (double)v.y);
}
template <bool UP, typename E2>
VB_DEVINL void st_l(E2* __restrict__ A, int r, int c, int ld, double re, double im) {
  using T = typename Real<E2>::T;
  E2 v;
  v.x = (T)re;
  v.y = (T)(UP ? -im : im);
  A[gix<UP>(r, c, ld)] = v;
}

// acc (16 x 16 strip at rows r0.., cols c0..; re / im as DMMA C fragments) -=
//   L[r0.., kb:ke] L[c0.., kb:ke]^H, fragments from L2; DIAG: only tiles nt <= mt.
template <bool UP, typename E2, bool DIAG>
VB_DEVINL void zstrip_kloop(double (&ar)[2][2][2], double (&ai)[2][2][2], const E2* __restrict__ A,
                            int n, int ld, int r0, int c0, int kb, int ke, int lane) {
  const int g = lane >> 2, q = lane & 3;
  const bool rv0 = r0 + g < n, rv1 = r0 + 8 + g < n, cv0 = c0 + g < n, cv1 = c0 + 8 + g < n;
#pragma unroll 2
  for (int k0 = kb; k0 < ke; k0 += 4) {  // warp-uniform trip count (mma.sync.aligned)
    const int k = k0 + q;
    double2 a0 = rv0 ? ld_l<UP>(A, r0 + g, k, ld) : make_double2(0.0, 0.0);
    double2 a1 = rv1 ? ld_l<UP>(A, r0 + 8 + g, k, ld) : make_double2(0.0, 0.0);
    double2 b0 = cv0 ? ld_l<UP>(A, c0 + g, k, ld) : make_double2(0.0, 0.0);
    double2 b1 = cv1 ? ld_l<UP>(A, c0 + 8 + g, k, ld) : make_double2(0.0, 0.0);
    const double2 fa[2] = {a0, a1}, fb[2] = {b0, b1};
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
#pragma unroll
      for (int nt = 0; nt < 2; ++nt) {
        if (DIAG && nt > mt) continue;
        // acc -= a conj(b): re -= ar br + ai bi, im -= ai br - ar bi
        dmma(ar[mt][nt], -fa[mt].x, fb[nt].x);
        dmma(ar[mt][nt], -fa[mt].y, fb[nt].y);
        dmma(ai[mt][nt], -fa[mt].y, fb[nt].x);
        dmma(ai[mt][nt], fa[mt].x, fb[nt].y);
      }
  }
}

template <bool UP, typename E2>
VB_DEVINL void zstrip_init(double (&ar)[2][2][2], double (&ai)[2][2][2], const E2* __restrict__ A,
                           int n, int ld, int r0, int c0, int ncols, bool diag, int lane) {
  const int g = lane >> 2, q = lane & 3;
#pragma unroll
  for (int mt = 0; mt < 2; ++mt)
#pragma unroll
    for (int nt = 0; nt < 2; ++nt)
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int r = r0 + mt * 8 + g, c = c0 + nt * 8 + 2 * q + h;
        const bool v = r < n && c < c0 + ncols && (!diag || r >= c);
        const double2 x = v ? ld_l<UP>(A, r, c, ld) : make_double2(0.0, 0.0);
        ar[mt][nt][h] = x.x;
        ai[mt][nt][h] = (r == c) ? 0.0 : x.y;
      }
}

// X = C Linv^H for a 16-row strip (C in acc, Linv in s.inv[k][c] = Linv(c, k)), stored to rows
// < n of column block c0.
template <bool UP, typename E2>
VB_DEVINL void zstrip_trsm_store(ZSmem& s, double (&ar)[2][2][2], double (&ai)[2][2][2],
                                 E2* __restrict__ A, int n, int ld, int r0, int c0, int lane) {
  const int g = lane >> 2, q = lane & 3;
  double xr[2][2][2] = {}, xi[2][2][2] = {};
#pragma unroll
  for (int ks = 0; ks < 4; ++ks) {
    double fr[2], fi[2];
#pragma unroll
    for (int mt = 0; mt < 2; ++mt) {
      fr[mt] = cfrag_to_afrag(ar[mt][ks >> 1][0], ar[mt][ks >> 1][1], ks & 1, lane);
      fi[mt] = cfrag_to_afrag(ai[mt][ks >> 1][0], ai[mt][ks >> 1][1], ks & 1, lane);
    }
#pragma unroll
    for (int nt = 0; nt < 2; ++nt) {
      if (4 * ks > 8 * nt + 7) continue;  // Linv(c, k) = 0 for k > c
      const double2 b = s.inv[ks * 4 + q][nt * 8 + g];
#pragma unroll
      for (int mt = 0; mt < 2; ++mt) {
        // x += c conj(b)
        dmma(xr[mt][nt], fr[mt], b.x);
        dmma(xr[mt][nt], fi[mt], b.y);
        dmma(xi[mt][nt], fi[mt], b.x);
        dmma(xi[mt][nt], -fr[mt], b.y);
      }
    }
  }
#pragma unroll
  for (int mt = 0; mt < 2; ++mt)
#pragma unroll
    for (int nt = 0; nt < 2; ++nt)
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int r = r0 + mt * 8 + g, c = nt * 8 + 2 * q + h;
        if (r < n) st_l<UP>(A, r, c0 + c, ld, xr[mt][nt][h], xi[mt][nt][h]);
      }
}

// Complex POTF2 of the nb x nb (nb <= 16) block in s.T by one warp (lane r = row r, r < 16),
// right-looking, IEEE sqrt and division; stores L to s.T and global. Returns info (in-block).
template <bool UP, typename E2>
VB_DEVINL int zpotf2_warp(ZSmem& s, int nb, E2* __restrict__ Ad, int ld, int lane) {
  const int r = lane & 15;
  double2 a[kZNB];
#pragma unroll
  for (int c = 0; c < kZNB; ++c) a[c] = (c <= r && r < nb) ? s.T[c][r] : make_double2(0.0, 0.0);
  __syncwarp();  // lanes 16..31 mirror rows 0..15: their reads precede lanes 0..15's writes below
  int info = 0, ncol = nb;
#pragma unroll
  for (int j = 0; j < kZNB; ++j) {
    if (j >= nb) break;
    const double d = __shfl_sync(kFull, a[j].x, j);
    if (!(d > 0.0)) {
      info = j + 1;
      ncol = j;
      if (lane == j) a[j] = make_double2(d, 0.0);
      break;
    }
    const double ljj = sqrt(d);
    if (r == j) a[j] = make_double2(ljj, 0.0);
    else if (r > j) a[j] = make_double2(a[j].x / ljj, a[j].y / ljj);
    if (lane < 16) s.col[r] = a[j];
    __syncwarp();
    if (r > j && r < nb) {
#pragma unroll
      for (int c = j + 1; c < kZNB; ++c) {
        if (c > r) break;
        const double2 lc = s.col[c];
        // a_rc -= l_rj conj(l_cj)
        a[c].x -= a[j].x * lc.x + a[j].y * lc.y;
        a[c].y -= a[j].y * lc.x - a[j].x * lc.y;
      }
    }
    __syncwarp();
  }
  const int nstore = info ? info : nb;  // columns < info hold L; column info-1 keeps the pivot
#pragma unroll
  for (int c = 0; c < kZNB; ++c)
    if (lane < 16 && c < nstore && c <= r && r < nb) {
      if (c < ncol || r == c) {
        s.T[c][r] = a[c];
        st_l<UP>(Ad, r, c, ld, a[c].x, (r == c) ? 0.0 : a[c].y);
      }
    }
  __syncwarp();
  return info;
}

// Linv = L11^-1 (lower, real diagonal) by one warp: lane c < nb computes column c by forward
// substitution; s.inv[k][c] = Linv(c, k) (zero for k > c).
VB_DEVINL void ztrtri_warp(ZSmem& s, int nb, int lane) {
  const int c = lane & 15;
  double2 x[kZNB];
#pragma unroll
  for (int i = 0; i < kZNB; ++i) {
    double sr = 0.0, si = 0.0;
#pragma unroll
    for (int k = 0; k < i; ++k) {
      const double2 l = s.T[k][i];  // L(i, k)
      sr += l.x * x[k].x - l.y * x[k].y;
      si += l.x * x[k].y + l.y * x[k].x;
    }
    const double lii = s.T[i][i].x;
    if (i < c || i >= nb) x[i] = make_double2(0.0, 0.0);
    else if (i == c) x[i] = make_double2(1.0 / lii, 0.0);
    else x[i] = make_double2(-sr / lii, -si / lii);
  }
  __syncwarp();
  if (lane < 16)
#pragma unroll
    for (int i = 0; i < kZNB; ++i) s.inv[c][i] = (c < nb) ? x[i] : make_double2(0.0, 0.0);  // Linv(i, c) at [k=c][i]
  __syncwarp();
}

template <bool UP, typename E2>
VB_DEVINL void zpotrf_matrix(ZSmem& s, E2* __restrict__ A, int n, int ld, int* info_out, int warp,
                             int lane) {
  const int npan = (n + kZNB - 1) / kZNB;
  const int nstrip = npan;
  for (int p = 0; p < npan; ++p) {
    const int j0 = kZNB * p, nb = min(kZNB, n - j0);
    const bool below = p + 1 < npan;
    if (warp == 0) {
      double ar[2][2][2], ai[2][2][2];
      zstrip_init<UP, E2>(ar, ai, A, n, ld, j0, j0, nb, true, lane);
      zstrip_kloop<UP, E2, true>(ar, ai, A, n, ld, j0, j0, 0, j0, lane);
      const int g = lane >> 2, q = lane & 3;
#pragma unroll
      for (int mt = 0; mt < 2; ++mt)
#pragma unroll
        for (int nt = 0; nt < 2; ++nt)
#pragma unroll
          for (int h = 0; h < 2; ++h)
            s.T[nt * 8 + 2 * q + h][mt * 8 + g] = make_double2(ar[mt][nt][h], ai[mt][nt][h]);
      __syncwarp();
      const int info = zpotf2_warp<UP, E2>(s, nb, A + (size_t)j0 * ld + j0, ld, lane);
      if (!info && below) ztrtri_warp(s, nb, lane);
      if (lane == 0) {
        s.info[p & 1] = info;
        if (info) *info_out = j0 + info;
      }
      __syncwarp();  // the named barrier is entered by the whole, converged warp
      if (below) bar_group_arrive(1, 128);
    } else if (below) {
      // the first strip's update overlaps warp 0's POTF2; every warp then meets the barrier at
      // the same instruction (synccheck), and the remaining strips follow
      const int first = p + warp;
      double ar[2][2][2], ai[2][2][2];
      if (first < nstrip) {
        zstrip_init<UP, E2>(ar, ai, A, n, ld, kZNB * first, j0, kZNB, false, lane);
        zstrip_kloop<UP, E2, false>(ar, ai, A, n, ld, kZNB * first, j0, 0, j0, lane);
      }
      __syncwarp();
      bar_group(1, 128);
      if (!s.info[p & 1]) {
        for (int st = first; st < nstrip; st += 3) {
          const int r0 = kZNB * st;
          if (st != first) {
            zstrip_init<UP, E2>(ar, ai, A, n, ld, r0, j0, kZNB, false, lane);
            zstrip_kloop<UP, E2, false>(ar, ai, A, n, ld, r0, j0, 0, j0, lane);
          }
          zstrip_trsm_store<UP, E2>(s, ar, ai, A, n, ld, r0, j0, lane);
        }
      }
    }
    __syncthreads();  // the panel's L is stored before the next panel reads it; info settled
    if (s.info[p & 1]) return;
  }
}

template <bool UP, typename E2>
__global__ void __launch_bounds__(128, 4)
    zpotrf_kernel(const int* __restrict__ d_n, E2* const* __restrict__ dA,
                  const int* __restrict__ d_ldda, int* __restrict__ d_info,
                  const Ctrl* __restrict__ ctrl_c, const int* __restrict__ order) {
  __shared__ ZSmem s;
  Ctrl* ctrl = const_cast<Ctrl*>(ctrl_c);
  pdl_wait();
  const int total = *(volatile const int*)&ctrl->count[0] + *(volatile const int*)&ctrl->count[1] +
                    *(volatile const int*)&ctrl->count[2];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (;;) {
    if (threadIdx.x == 0) s.item = atomicAdd(&ctrl->head[0], 1);
    __syncthreads();
    const int it = s.item;
    __syncthreads();
    if (it >= total) break;
    const int m = order[it];  // the three ranges are contiguous: order[] is LPT over all n
    zpotrf_matrix<UP, E2>(s, dA[m], d_n[m], d_ldda[m], d_info + m, warp, lane);
    __syncthreads();
  }
}

template <typename E2>
int zpotrf_impl(char uplo, const int* d_n, E2* const* dA, const int* d_ldda, int* d_info,
                int batch, int max_n, cudaStream_t stream) {
  if (!(uplo == 'L' || uplo == 'l' || uplo == 'U' || uplo == 'u')) return -1;
  const bool up = (uplo == 'U' || uplo == 'u');
  if (batch < 0) return -6;
  if (max_n < 0) return -7;
  if (batch == 0) return 0;
  void* ws = nullptr;
  cudaError_t e = ws_alloc(&ws, sizeof(Ctrl) + sizeof(int) * (size_t)batch, stream);
  if (e != cudaSuccess) return (int)e;
  Ctrl* ctrl = static_cast<Ctrl*>(ws);
  int* order = reinterpret_cast<int*>(ctrl + 1);
  e = launch_scan_bin(d_n, d_ldda, d_info, batch, max_n, true, ctrl, order, stream);
  if (e == cudaSuccess && max_n > 0) {
    int dev = 0, sms = 148;
    if (cudaGetDevice(&dev) == cudaSuccess)
      cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaLaunchConfig_t cfg = {};
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    cfg.stream = stream;
    cfg.blockDim = dim3(128);
    cfg.gridDim = dim3(std::max(1, std::min(batch, 4 * sms)));
    e = cudaLaunchKernelEx(&cfg, up ? zpotrf_kernel<true, E2> : zpotrf_kernel<false, E2>, d_n, dA,
                           d_ldda, d_info, (const Ctrl*)ctrl, (const int*)order);
  }
  cudaError_t e2 = ws_free(ws, stream);
  return (int)(e != cudaSuccess ? e : e2);
}

}  // namespace
}  // namespace vb

using namespace vb;

extern "C" int vbatched_zpotrf(char uplo, const int* d_n, void* const* dA_array, const int* d_ldda,
                               int* d_info, int batchCount, int max_n, vb_stream_t stream) {
  return zpotrf_impl<double2>(uplo, d_n, reinterpret_cast<double2* const*>(dA_array), d_ldda,
                              d_info, batchCount, max_n, (cudaStream_t)stream);
}

extern "C" int vbatched_cpotrf(char uplo, const int* d_n, void* const* dA_array, const int* d_ldda,
                               int* d_info, int batchCount, int max_n, vb_stream_t stream) {
  return zpotrf_impl<float2>(uplo, d_n, reinterpret_cast<float2* const*>(dA_array), d_ldda,
                             d_info, batchCount, max_n, (cudaStream_t)stream);
}
