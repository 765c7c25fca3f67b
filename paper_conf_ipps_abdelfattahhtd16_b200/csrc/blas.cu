// blas.cu — standalone vbatched DGEMM / DSYRK / DTRSM (§III-E.2-3) on the
// FP64 tensor cores (DMMA m8n8k4), exposed through include/vbatched.h.
//
// Work distribution (replaces the paper's max-size grid with early-exit thread blocks,
// PAPER.md:633-674, which is Kepler prior art): a one-CTA device scan turns the per-matrix
// dimensions into a prefix sum of tile counts; persistent CTAs then pop global tile ids from
// an atomic counter and locate their matrix by binary search. Only real tiles are visited —
// for SYRK only the tiles of the referenced triangle ("decision layer").
#include <algorithm>
#include <mutex>

#include "common.cuh"
#include "internal.h"

namespace vb {
namespace {

constexpr int kBT = 64;      // C tile edge
constexpr int kBK = 16;      // k chunk
constexpr int kGThreads = 128;
constexpr int kLD = kBT + 4;

enum Mode { kGemm = 0, kSyrkLower = 1, kSyrkUpper = 2, kTrsm = 3 };

struct BlasArgs {
  int mode;
  bool ta, tb;  // operand transposed
  const int* m;
  const int* n;
  const int* k;
  double alpha, beta;
  const double* const* A;
  const int* lda;
  const double* const* B;
  const int* ldb;
  double* const* C;
  const int* ldc;
  int batch;
  // trsm
  bool tlower, unit, upper_in_A;
  bool bt;  // trsm side 'L': the kernel solves the side-'R' problem on the transposed view of B
};

__device__ __forceinline__ int cdiv(int a, int b) { return (a + b - 1) / b; }

__device__ __forceinline__ int tiles_of(const BlasArgs& a, int i) {
  if (a.mode == kGemm) {
    const int m = a.m[i], n = a.n[i];
    return (m > 0 && n > 0) ? cdiv(m, kBT) * cdiv(n, kBT) : 0;
  }
  if (a.mode == kTrsm) {
    const int m = a.m[i], n = a.n[i];
    return (m > 0 && n > 0) ? cdiv(m, kBT) : 0;
  }
  const int n = a.n[i];
  const int t = n > 0 ? cdiv(n, kBT) : 0;
  return t * (t + 1) / 2;
}

// Prefix sum of tile counts (one CTA of 1024 threads, carry across 1024-wide chunks).
__global__ void __launch_bounds__(1024, 1) tile_scan_kernel(BlasArgs a, int* off, int* counter) {
  pdl_launch_dependents();
  __shared__ int wsum[32];
  __shared__ int carry;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) carry = 0;
  __syncthreads();
  for (int base = 0; base < a.batch; base += 1024) {
    const int i = base + tid;
    const int v = i < a.batch ? tiles_of(a, i) : 0;
    int incl = v;
    for (int o = 1; o < 32; o <<= 1) {
      const int t = __shfl_up_sync(kFull, incl, o);
      if (lane >= o) incl += t;
    }
    if (lane == 31) wsum[warp] = incl;
    __syncthreads();
    if (warp == 0) {
      const int w = wsum[lane];
      int x = w;
      for (int o = 1; o < 32; o <<= 1) {
        const int t = __shfl_up_sync(kFull, x, o);
        if (lane >= o) x += t;
      }
      wsum[lane] = x - w;
    }
    __syncthreads();
    const int c = carry;
    if (i < a.batch) off[i] = c + wsum[warp] + incl - v;
    __syncthreads();
    if (tid == 1023) carry = c + wsum[warp] + incl;
    __syncthreads();
  }
  if (tid == 0) {
    off[a.batch] = carry;
    *counter = 0;
  }
}

// Tile -> matrix lookup (the matrix of tile t is the largest i with off[i] <= t; it has tiles,
// since off[i+1] > t). A binary search over off[] in global memory is a chain of ~log2(batch)
// dependent L2 round trips per tile (12 for 3000 matrices, several microseconds), which
// dominated the tiny rank-16 tiles of GETRF/GEQRF's trailing updates. Instead every CTA samples
// off[] once (coarse[c] = off[c S], S a multiple of 32 with at most kCoarse samples), and a tile
// is located by a binary search in shared memory plus one round of S / 32 independent
// coalesced warp loads of off[] and a ballot.
constexpr int kCoarse = 512;
struct TileIndex {
  int coarse[kCoarse];
  int S, nc;
};

__device__ __forceinline__ void tile_index_init(TileIndex& x, const int* off, int batch) {
  const int S = max(32, cdiv(cdiv(batch, kCoarse), 32) * 32);
  const int nc = cdiv(batch, S);
  for (int c = threadIdx.x; c < nc; c += blockDim.x) x.coarse[c] = off[c * S];
  if (threadIdx.x == 0) {
    x.S = S;
    x.nc = nc;
  }
  __syncthreads();
}

// One warp (all lanes get the result).
__device__ __forceinline__ int tile_locate(const TileIndex& x, const int* off, int batch, int t,
                                           int lane) {
  int lo = 0, hi = x.nc;
  while (hi - lo > 1) {
    const int mid = (lo + hi) >> 1;
    if (x.coarse[mid] <= t) lo = mid;
    else hi = mid;
  }
  const int base = lo * x.S;
  int cnt = 0;
  for (int u = 0; u < x.S; u += 32) {
    const int i = base + u + lane;
    cnt += __popc(__ballot_sync(kFull, i < batch && off[i] <= t));
  }
  return base + cnt - 1;
}

// ---------------------------------------------------------------------------------------
// GEMM / SYRK tile: C[r0:r0+64, c0:c0+64] = alpha op(A) op(B) + beta C (masked for SYRK).
constexpr int kGStages = 3;  // cp.async ring depth: one CTA barrier per k chunk
struct GemmSmem {
  double a[kGStages][kBK][kLD];  // [k][row]
  double b[kGStages][kBK][kLD];  // [k][col]
};

__device__ __forceinline__ void gemm_stage(GemmSmem& s, int st, const double* A, int lda, bool ta,
                                           const double* B, int ldb, bool tb, int m, int n, int K,
                                           int r0, int c0, int k0) {
  const int tid = threadIdx.x;
#pragma unroll
  for (int e = 0; e < (kBT * kBK) / kGThreads; ++e) {
    const int idx = tid + e * kGThreads;
    int i, k;
    if (!ta) { i = idx % kBT; k = idx / kBT; }
    else { k = idx % kBK; i = idx / kBK; }
    const bool p = (r0 + i < m) && (k0 + k < K);
    const size_t o = !ta ? (size_t)(k0 + k) * lda + (r0 + i) : (size_t)(r0 + i) * lda + (k0 + k);
    cp_async8(&s.a[st][k][i], A + (p ? o : 0), p);
  }
#pragma unroll
  for (int e = 0; e < (kBT * kBK) / kGThreads; ++e) {
    const int idx = tid + e * kGThreads;
    int j, k;
    if (!tb) { k = idx % kBK; j = idx / kBK; }
    else { j = idx % kBT; k = idx / kBT; }
    const bool p = (c0 + j < n) && (k0 + k < K);
    const size_t o = !tb ? (size_t)(c0 + j) * ldb + (k0 + k) : (size_t)(k0 + k) * ldb + (c0 + j);
    cp_async8(&s.b[st][k][j], B + (p ? o : 0), p);
  }
}

__global__ void __launch_bounds__(kGThreads, 4) gemm_syrk_kernel(BlasArgs a, const int* off,
                                                                 int* counter) {
  extern __shared__ __align__(16) unsigned char gsm_raw[];
  GemmSmem& s = *reinterpret_cast<GemmSmem*>(gsm_raw);
  __shared__ int s_t, s_mi;
  __shared__ TileIndex tix;
  pdl_wait();
  const int total = off[a.batch];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int g = lane >> 2, q = lane & 3;
  const int wr = (warp >> 1) * 32, wc = (warp & 1) * 32;
  tile_index_init(tix, off, a.batch);
  // the next tile id is popped while the current tile runs (thread 0 stores it at the loop top)
  int nxt = 0;
  if (tid == 0) nxt = atomicAdd(counter, 1);
  for (;;) {
    if (tid == 0) s_t = nxt;
    __syncthreads();
    if (warp == 0) {
      const int tt = s_t;
      const int mm = tt < total ? tile_locate(tix, off, a.batch, tt, lane) : 0;
      if (lane == 0) s_mi = mm;
    }
    __syncthreads();
    const int t = s_t;
    if (t >= total) break;
    if (tid == 0) nxt = atomicAdd(counter, 1);
    const int mi = s_mi;
    int lt = t - off[mi];
    const int n = a.n[mi];
    const int m = (a.mode == kGemm) ? a.m[mi] : n;
    const int K = a.k[mi];
    int ti, tj;
    if (a.mode == kGemm) {
      const int tm = cdiv(m, kBT);
      ti = lt % tm;
      tj = lt / tm;
    } else {
      const int T = cdiv(n, kBT);
      // enumerate the triangle column by column
      int col = 0;
      while (true) {
        const int len = (a.mode == kSyrkLower) ? T - col : col + 1;
        if (lt < len) break;
        lt -= len;
        ++col;
      }
      tj = col;
      ti = (a.mode == kSyrkLower) ? col + lt : lt;
    }
    const int r0 = ti * kBT, c0 = tj * kBT;
    const double* A = a.A[mi];
    const double* B = (a.mode == kGemm) ? a.B[mi] : a.A[mi];
    const int lda = a.lda[mi];
    const int ldb = (a.mode == kGemm) ? a.ldb[mi] : lda;
    double acc[4][4][2];
#pragma unroll
    for (int x = 0; x < 4; ++x)
#pragma unroll
      for (int y = 0; y < 4; ++y) acc[x][y][0] = acc[x][y][1] = 0.0;
    const int nk = cdiv(K, kBK);
    double* C = a.C[mi];
    const int ldc = a.ldc[mi];
    // One k chunk (K <= 16: the rank-16 trailing updates of GETRF/GEQRF): the C tile is fetched
    // into the idle ring stages 1-2 together with the chunk, so its load latency overlaps the
    // chunk's instead of following the products (columns 0..31 in a[1..2], 32..63 in b[1..2]).
    const bool cpre = nk == 1 && a.beta != 0.0;
    auto cs = [&](int c, int r) -> double* {
      return (c < 32 ? &s.a[1][0][0] : &s.b[1][0][0]) + (c & 31) * kLD + r;
    };
    if (nk > 0) gemm_stage(s, 0, A, lda, a.ta, B, ldb, a.tb, m, n, K, r0, c0, 0);
    cp_async_commit();
    if (nk > 1) gemm_stage(s, 1, A, lda, a.ta, B, ldb, a.tb, m, n, K, r0, c0, kBK);
    if (cpre) {
#pragma unroll 4
      for (int e = tid; e < kBT * kBT; e += kGThreads) {
        const int r = e % kBT, c = e / kBT;
        const bool p = r0 + r < m && c0 + c < n;
        cp_async8(cs(c, r), C + (p ? (size_t)(c0 + c) * ldc + (r0 + r) : 0), p);
      }
    }
    cp_async_commit();
    for (int kc = 0; kc < nk; ++kc) {
      cp_async_wait<1>();  // chunk kc has landed (only chunk kc+1 may still be in flight)
      __syncthreads();     // ... for every thread; and every warp is done with chunk kc-1
      if (kc + 2 < nk)
        gemm_stage(s, (kc + 2) % kGStages, A, lda, a.ta, B, ldb, a.tb, m, n, K, r0, c0,
                   (kc + 2) * kBK);
      cp_async_commit();
      const int st = kc % kGStages;
#pragma unroll
      for (int kk = 0; kk < kBK / 4; ++kk) {
        double fa[4], fb[4];
#pragma unroll
        for (int x = 0; x < 4; ++x) fa[x] = s.a[st][kk * 4 + q][wr + x * 8 + g];
#pragma unroll
        for (int y = 0; y < 4; ++y) fb[y] = s.b[st][kk * 4 + q][wc + y * 8 + g];
#pragma unroll
        for (int x = 0; x < 4; ++x)
#pragma unroll
          for (int y = 0; y < 4; ++y) dmma(acc[x][y], fa[x], fb[y]);
      }
    }
    cp_async_wait<0>();
    __syncthreads();  // the C tile has landed (cpre); the next tile's prologue refills stages 0-1
                      // only after the loop-top barriers, when every thread has read it
    // Epilogue in two passes: every load of C first (all in flight together), then every store.
    // As one read-modify-write per element the loads serialise behind the stores (the compiler
    // cannot move a load of C past a store to C): one memory round trip per element, most of a
    // tile's time for small k (the rank-16 trailing updates of GETRF/GEQRF).
    if (a.beta != 0.0) {
#pragma unroll
      for (int x = 0; x < 4; ++x)
#pragma unroll
        for (int y = 0; y < 4; ++y)
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            const int r = r0 + wr + x * 8 + g, c = c0 + wc + y * 8 + 2 * q + h;
            const bool p = r < m && c < n && !(a.mode == kSyrkLower && r < c) &&
                           !(a.mode == kSyrkUpper && r > c);
            const double cv = !p ? 0.0 : cpre ? *cs(c - c0, r - r0) : C[(size_t)c * ldc + r];
            acc[x][y][h] = a.alpha * acc[x][y][h] + (p ? a.beta * cv : 0.0);
          }
    } else {
#pragma unroll
      for (int x = 0; x < 4; ++x)
#pragma unroll
        for (int y = 0; y < 4; ++y)
#pragma unroll
          for (int h = 0; h < 2; ++h) acc[x][y][h] *= a.alpha;
    }
#pragma unroll
    for (int x = 0; x < 4; ++x)
#pragma unroll
      for (int y = 0; y < 4; ++y)
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const int r = r0 + wr + x * 8 + g, c = c0 + wc + y * 8 + 2 * q + h;
          if (r >= m || c >= n) continue;
          if (a.mode == kSyrkLower && r < c) continue;
          if (a.mode == kSyrkUpper && r > c) continue;
          C[(size_t)c * ldc + r] = acc[x][y][h];
        }
  }
}

// ---------------------------------------------------------------------------------------
// TRSM side 'R': X T = alpha B, T = op(A) (n x n triangular), one CTA per 64-row block of B.
// Column blocks of 32 are solved in dependency order (ascending for upper T, descending for
// lower T): R = alpha B_J - sum_K X_K T_{K,J} (DMMA), X_J = R inv(T_JJ) (TRTRI in smem + DMMA).
constexpr int kTW = 32;
constexpr int kTC = 16;      // k chunk of the solved-block accumulation
constexpr int kTStages = 3;  // its cp.async ring depth
struct TrsmSmem {
  union {
    struct {  // accumulation ring: X chunk [k][row] and T chunk [k][col]
      double xa[kTStages][kTC][kLD];
      double tb[kTStages][kTC][kTW + 4];
    } ring;
    struct {
      double x[kTW][kLD];      // R = alpha B_J - sum, [k=col][row]
      double t[kTW][kTW + 4];  // scratch for the transposed inverse
    } e;
  } u;
  double d[kTW][kTW + 1];  // diagonal block T_JJ as the lower factor L of TRTRI: d[c][r] = L[r][c]
  double inv[kTW][kTW + 4];  // inv(T_JJ) [k][col]
  double S[16 * LDS_T];      // TRTRI scratch
  double tv[kTW];            // 1 / L[c][c]
};

__device__ __forceinline__ double t_elem(const BlasArgs& a, const double* A, int lda, int i, int j) {
  // T(i,j) = op(A)(i,j) restricted to A's triangle; unit diagonal if requested.
  if (i == j && a.unit) return 1.0;
  const int ai = a.ta ? j : i, aj = a.ta ? i : j;
  const bool in_tri = a.upper_in_A ? (ai <= aj) : (ai >= aj);
  return in_tri ? A[(size_t)aj * lda + ai] : 0.0;
}

// Element (r, c) of the right-hand side the kernel works on: B itself (side 'R') or B^T (side
// 'L': op(A) X = alpha B  <=>  X^T op(A)^T = alpha B^T).
__device__ __forceinline__ size_t bix(bool bt, int r, int c, int ldb) {
  return bt ? (size_t)r * ldb + c : (size_t)c * ldb + r;
}

// One k chunk of the accumulation sum_K X_K T_{K,J}: X[r0:r0+64, k0:k0+16] (already solved
// columns of the right-hand side, B's storage view) and T[k0:k0+16, c0:c0+32] (op(A), an
// off-diagonal block: no triangle mask, no unit diagonal), 8-byte cp.async, zero-filled
// outside [k0, kend) and the matrix.
__device__ __forceinline__ void trsm_stage(TrsmSmem& s, int st, const BlasArgs& a, const double* A,
                                           int lda, const double* B, int ldb, int m, int r0,
                                           int c0, int w, int k0, int kend) {
  const int tid = threadIdx.x;
#pragma unroll
  for (int e = 0; e < (kTC * kBT) / kGThreads; ++e) {
    const int idx = tid + e * kGThreads;
    // contiguous direction of the storage view first: rows for B, k for B^T (side 'L')
    const int k = a.bt ? idx % kTC : idx / kBT, i = a.bt ? idx / kTC : idx % kBT;
    const bool p = (k0 + k < kend) && (r0 + i < m);
    cp_async8(&s.u.ring.xa[st][k][i], B + (p ? bix(a.bt, r0 + i, k0 + k, ldb) : 0), p);
  }
#pragma unroll
  for (int e = 0; e < (kTC * kTW) / kGThreads; ++e) {
    const int idx = tid + e * kGThreads;
    const int j = idx / kTC, k = idx % kTC;
    const bool p = (k0 + k < kend) && (j < w);
    const size_t o = a.ta ? (size_t)(k0 + k) * lda + (c0 + j) : (size_t)(c0 + j) * lda + (k0 + k);
    cp_async8(&s.u.ring.tb[st][k][j], A + (p ? o : 0), p);
  }
}

__global__ void __launch_bounds__(kGThreads) trsm_kernel(BlasArgs a, const int* off, int* counter) {
  extern __shared__ __align__(16) unsigned char tsm_raw[];
  TrsmSmem& s = *reinterpret_cast<TrsmSmem*>(tsm_raw);
  __shared__ int s_t, s_mi;
  __shared__ TileIndex tix;
  pdl_wait();
  const int total = off[a.batch];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int g = lane >> 2, q = lane & 3;
  const int wr = (warp >> 1) * 32, wc = (warp & 1) * 16;
  tile_index_init(tix, off, a.batch);
  int nxt = 0;  // the next tile id, popped while the current one runs (see gemm_syrk_kernel)
  if (tid == 0) nxt = atomicAdd(counter, 1);
  for (;;) {
    if (tid == 0) s_t = nxt;
    __syncthreads();
    if (warp == 0) {
      const int tt = s_t;
      const int mm = tt < total ? tile_locate(tix, off, a.batch, tt, lane) : 0;
      if (lane == 0) s_mi = mm;
    }
    __syncthreads();
    const int t = s_t;
    if (t >= total) break;
    if (tid == 0) nxt = atomicAdd(counter, 1);
    const int mi = s_mi;
    const int r0 = (t - off[mi]) * kBT;
    const int m = a.m[mi], n = a.n[mi];
    const double* A = a.A[mi];
    const int lda = a.lda[mi];
    double* B = a.C[mi];
    const int ldb = a.ldc[mi];
    const int nbk = cdiv(n, kTW);
    for (int step = 0; step < nbk; ++step) {
      const int J = a.tlower ? nbk - 1 - step : step;
      const int c0 = J * kTW, w = min(kTW, n - c0);
      // B_J and T_JJ are read into registers before the accumulation loop (neither is written
      // before this step's end), so these 24 loads per thread overlap it instead of running as
      // dependent round trips after it. Index order: the storage view's contiguous direction
      // across the lanes (rows of B; for B^T the columns of B_J).
      constexpr int kBE = (kTW * kBT) / kGThreads, kTE = (kTW * kTW) / kGThreads;
      double bv[kBE], tjj[kTE];
#pragma unroll
      for (int e = 0; e < kBE; ++e) {
        const int idx = tid + e * kGThreads;
        const int k = a.bt ? idx % kTW : idx / kBT, i = a.bt ? idx / kTW : idx % kBT;
        bv[e] = (k < w && r0 + i < m) ? B[bix(a.bt, r0 + i, c0 + k, ldb)] : 0.0;
      }
#pragma unroll
      for (int e = 0; e < kTE; ++e) {
        const int idx = tid + e * kGThreads;
        const int j = a.ta ? idx % kTW : idx / kTW, i = a.ta ? idx / kTW : idx % kTW;
        tjj[e] = (i < w && j < w) ? t_elem(a, A, lda, c0 + i, c0 + j) : (i == j ? 1.0 : 0.0);
      }
      double acc[4][2][2];
#pragma unroll
      for (int x = 0; x < 4; ++x)
#pragma unroll
        for (int y = 0; y < 2; ++y) acc[x][y][0] = acc[x][y][1] = 0.0;
      // sum over the solved blocks K of X_K T_{K,J} = X[:, kb:ke] T[kb:ke, J] as one pipelined
      // k loop (columns before J for an upper T, after J for a lower T)
      const int kb = a.tlower ? c0 + kTW : 0, ke = a.tlower ? n : c0;
      const int nkc = ke > kb ? cdiv(ke - kb, kTC) : 0;
      if (nkc > 0) trsm_stage(s, 0, a, A, lda, B, ldb, m, r0, c0, w, kb, ke);
      cp_async_commit();
      if (nkc > 1) trsm_stage(s, 1, a, A, lda, B, ldb, m, r0, c0, w, kb + kTC, ke);
      cp_async_commit();
      for (int kc = 0; kc < nkc; ++kc) {
        cp_async_wait<1>();
        __syncthreads();
        if (kc + 2 < nkc)
          trsm_stage(s, (kc + 2) % kTStages, a, A, lda, B, ldb, m, r0, c0, w, kb + (kc + 2) * kTC,
                     ke);
        cp_async_commit();
        const int st = kc % kTStages;
#pragma unroll
        for (int k4 = 0; k4 < kTC / 4; ++k4) {
          double fa[4], fb[2];
#pragma unroll
          for (int x = 0; x < 4; ++x) fa[x] = s.u.ring.xa[st][k4 * 4 + q][wr + x * 8 + g];
#pragma unroll
          for (int y = 0; y < 2; ++y) fb[y] = s.u.ring.tb[st][k4 * 4 + q][wc + y * 8 + g];
#pragma unroll
          for (int x = 0; x < 4; ++x)
#pragma unroll
            for (int y = 0; y < 2; ++y) dmma(acc[x][y], fa[x], fb[y]);
        }
      }
      cp_async_wait<0>();
      __syncthreads();  // the ring is dead: s.u.e aliases it from here on
      // R = alpha B_J - acc, into s.x as [k=col][row]; diagonal block into s.d
#pragma unroll
      for (int x = 0; x < 4; ++x)
#pragma unroll
        for (int y = 0; y < 2; ++y)
#pragma unroll
          for (int h = 0; h < 2; ++h) s.u.e.x[wc + y * 8 + 2 * q + h][wr + x * 8 + g] = -acc[x][y][h];
      // TRTRI input L (lower, L[r][c] at d[c][r]): L = T_JJ when T is lower, L = T_JJ^T when
      // it is upper (then inv(L)^T = inv(T_JJ) comes out of TRTRI directly)
#pragma unroll
      for (int e = 0; e < kTE; ++e) {
        const int idx = tid + e * kGThreads;
        const int j = a.ta ? idx % kTW : idx / kTW, i = a.ta ? idx / kTW : idx % kTW;
        if (a.tlower) s.d[j][i] = tjj[e];
        else s.d[i][j] = tjj[e];
      }
      __syncthreads();
#pragma unroll
      for (int e = 0; e < kBE; ++e) {
        const int idx = tid + e * kGThreads;
        const int k = a.bt ? idx % kTW : idx / kBT, i = a.bt ? idx / kTW : idx % kBT;
        s.u.e.x[k][i] = fma(a.alpha, bv[e], s.u.e.x[k][i]);
      }
      // inv(T_JJ) by warp 0: 8x8 substitution + recursive doubling on DMMA (trtri32_dmma_warp)
      // into the B-operand layout INV[k][n] = inv(L)[n][k]; for a lower T that is inv(T)^T,
      // transposed once through s.t
      if (warp == 0) {
        s.tv[lane] = 1.0 / s.d[lane][lane];
        __syncwarp();
        double* out = a.tlower ? &s.u.e.t[0][0] : &s.inv[0][0];
        trtri32_dmma_warp(&s.d[0][0], kTW + 1, s.tv, out, kTW + 4, s.S, LDS_T, lane);
        if (a.tlower) {
#pragma unroll 4
          for (int k = 0; k < kTW; ++k) s.inv[k][lane] = s.u.e.t[lane][k];
        }
      }
      __syncthreads();
      double xo[4][2][2];
#pragma unroll
      for (int x = 0; x < 4; ++x)
#pragma unroll
        for (int y = 0; y < 2; ++y) xo[x][y][0] = xo[x][y][1] = 0.0;
#pragma unroll
      for (int k4 = 0; k4 < kTW / 4; ++k4) {
        double fa[4], fb[2];
#pragma unroll
        for (int x = 0; x < 4; ++x) fa[x] = s.u.e.x[k4 * 4 + q][wr + x * 8 + g];
#pragma unroll
        for (int y = 0; y < 2; ++y) fb[y] = s.inv[k4 * 4 + q][wc + y * 8 + g];
#pragma unroll
        for (int x = 0; x < 4; ++x)
#pragma unroll
          for (int y = 0; y < 2; ++y) dmma(xo[x][y], fa[x], fb[y]);
      }
#pragma unroll
      for (int x = 0; x < 4; ++x)
#pragma unroll
        for (int y = 0; y < 2; ++y)
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            const int r = r0 + wr + x * 8 + g, c = wc + y * 8 + 2 * q + h;
            if (r < m && c < w) B[bix(a.bt, r, c0 + c, ldb)] = xo[x][y][h];
          }
      __syncthreads();  // X_J visible to the CTA before the next block reads it
    }
  }
}

int g_sms = 0;

int launch_blas(const BlasArgs& a, cudaStream_t stream) {
  {  // per-device kernel attribute (dynamic shared memory), once per device ordinal
    static unsigned long long ready = 0;
    static std::mutex mu;
    int dev = 0;
    cudaGetDevice(&dev);
    const unsigned long long bit = dev < 64 ? 1ull << dev : 0ull;
    if (!(g_sms && (ready & bit))) {
      std::lock_guard<std::mutex> lock(mu);
      cudaDeviceGetAttribute(&g_sms, cudaDevAttrMultiProcessorCount, dev);
      cudaError_t ea = cudaFuncSetAttribute(gemm_syrk_kernel,
                                            cudaFuncAttributeMaxDynamicSharedMemorySize,
                                            (int)sizeof(GemmSmem));
      if (ea != cudaSuccess) return (int)ea;
      ea = cudaFuncSetAttribute(trsm_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)sizeof(TrsmSmem));
      if (ea != cudaSuccess) return (int)ea;
      ready |= bit;
    }
  }
  void* ws = nullptr;
  cudaError_t e = ws_alloc(&ws, sizeof(int) * ((size_t)a.batch + 2), stream);
  if (e != cudaSuccess) return (int)e;
  int* off = static_cast<int*>(ws);
  int* counter = off + a.batch + 1;
  tile_scan_kernel<<<1, 1024, 0, stream>>>(a, off, counter);
  e = cudaGetLastError();
  if (e == cudaSuccess) {
    cudaLaunchConfig_t cfg = {};
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    cfg.stream = stream;
    cfg.blockDim = dim3(kGThreads);
    cfg.gridDim = dim3(g_sms * 8);
    if (a.mode == kTrsm) {
      cfg.gridDim = dim3(g_sms * 3);  // 3 CTAs per SM (61 KB smem each)
      cfg.dynamicSmemBytes = sizeof(TrsmSmem);
      e = cudaLaunchKernelEx(&cfg, trsm_kernel, a, (const int*)off, counter);
    } else {
      cfg.gridDim = dim3(g_sms * 4);  // 4 CTAs per SM (registers, 52 KB smem each)
      cfg.dynamicSmemBytes = sizeof(GemmSmem);
      e = cudaLaunchKernelEx(&cfg, gemm_syrk_kernel, a, (const int*)off, counter);
    }
  }
  cudaError_t e2 = ws_free(ws, stream);
  return (int)(e != cudaSuccess ? e : e2);
}

bool is_t(char c) { return c == 'T' || c == 't' || c == 'C' || c == 'c'; }

}  // namespace

int gemm_launch(char ta, char tb, const int* d_m, const int* d_n, const int* d_k, double alpha,
                const double* const* dA, const int* d_lda, const double* const* dB,
                const int* d_ldb, double beta, double* const* dC, const int* d_ldc, int batch,
                int, int, int, cudaStream_t stream) {
  BlasArgs a = {};
  a.mode = kGemm;
  a.ta = is_t(ta);
  a.tb = is_t(tb);
  a.m = d_m; a.n = d_n; a.k = d_k;
  a.alpha = alpha; a.beta = beta;
  a.A = dA; a.lda = d_lda; a.B = dB; a.ldb = d_ldb; a.C = dC; a.ldc = d_ldc;
  a.batch = batch;
  return launch_blas(a, stream);
}

int syrk_launch(char uplo, char trans, const int* d_n, const int* d_k, double alpha,
                const double* const* dA, const int* d_lda, double beta, double* const* dC,
                const int* d_ldc, int batch, int, int, cudaStream_t stream) {
  BlasArgs a = {};
  a.mode = (uplo == 'L' || uplo == 'l') ? kSyrkLower : kSyrkUpper;
  a.ta = is_t(trans);   // op(A) = A (N) or A^T (T)
  a.tb = !a.ta;         // second operand op(A)^T
  a.m = d_n; a.n = d_n; a.k = d_k;
  a.alpha = alpha; a.beta = beta;
  a.A = dA; a.lda = d_lda; a.B = dA; a.ldb = d_lda; a.C = dC; a.ldc = d_ldc;
  a.batch = batch;
  return launch_blas(a, stream);
}

int trsm_launch(char side, char uplo, char ta, char diag, const int* d_m, const int* d_n,
                double alpha, const double* const* dA, const int* d_lda, double* const* dB,
                const int* d_ldb, int batch, int, int, cudaStream_t stream) {
  BlasArgs a = {};
  a.mode = kTrsm;
  // side 'L' = side 'R' on B^T with T = op(A)^T: flip the transposition, swap m and n
  a.bt = (side == 'L' || side == 'l');
  a.ta = is_t(ta) ^ a.bt;
  a.upper_in_A = (uplo == 'U' || uplo == 'u');
  a.tlower = (!a.upper_in_A) ^ a.ta;  // T = op(A) is lower iff (A lower) xor transposed
  a.unit = (diag == 'U' || diag == 'u');
  if (a.bt) {
    a.m = d_n; a.n = d_m; a.k = d_m;
  } else {
    a.m = d_m; a.n = d_n; a.k = d_n;
  }
  a.alpha = alpha; a.beta = 0.0;
  a.A = dA; a.lda = d_lda; a.C = dB; a.ldc = d_ldb;
  a.batch = batch;
  return launch_blas(a, stream);
}

}  // namespace vb
