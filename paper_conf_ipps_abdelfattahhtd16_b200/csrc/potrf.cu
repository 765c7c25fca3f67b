// potrf.cu — the factorisation kernels of vbatched_dpotrf (steps a2-a7 of SURVEY.md §8(a)).
//
// Three persistent kernels drain the three ranges of the work list written by scan_bin
// (matrices sorted by n descending = flops descending: longest-processing-time first):
//
//  * potrf_blocked3_kernel, n > ts (128): one CTA (4 consumer warps + 1 TMA producer warp,
//    3 CTAs per SM) per matrix, the left-looking blocked Cholesky of PAPER.md Algorithm 1
//     with panel width NB = 64:
//      for each panel j0 (columns j0..j0+63), for each block of MB = 64 rows r0 >= j0:
//        panel update    C = A[r0:, j0:j0+64] - L[r0:, 0:j0] L[j0:j0+64, 0:j0]^T
//                        ("customized syrk" with B a part of A, Fig. 2) on
//                        the FP64 tensor cores (DMMA m8n8k4), operands staged by TMA bulk
//                        copies into an mbarrier ring fed by the producer warp (the paper's
//                        double buffering); the accumulators start from A's
//                        panel values;
//        tile factorize  L11 = chol(C1) for the first row block (r0 == j0): the 64x64 block as
//                        POTF2(32) / TRSM / SYRK / POTF2(32), each POTF2(32) = POTF2(16) in
//                        registers (LDL^T-form right-looking update, short pivot chain) + DMMA
//                        SYRK + POTF2(16);
//        panel factorize C2 <- C2 L11^-T: TRTRI of the 32x32 diagonal blocks (8x8 substitution +
//                        recursive doubling on DMMA), then DMMA against the triangular
//                        inverses from registers — the trtri + gemm TRSM of PAPER.md:760-772.
//    Every element of L is written once; earlier columns are re-read once per panel (HBM
//    re-read traffic ~ 8 n^3 / (6 NB) bytes per matrix).
//  * potrf_small_kernel, 32 < n <= ts: one (diagonal warp, off-diagonal warp) pair per matrix,
//    two pairs per 4-warp CTA, 4 CTAs per SM, NB = 32 left-looking with look-ahead,
//    panel-update fragments straight from L2.
//  * potrf_warp_kernel, n <= 32: one warp per matrix, whole matrix in registers
//    (the fused on-chip POTF2 of PAPER.md:551-560; one HBM read, one HBM write).
// The kernels are chained with programmatic dependent launch: each releases its dependent
// grid as soon as it starts, so the next range's CTAs take the SMs the previous kernel's
// CTAs free at its tail (the smaller matrices come later in LPT order anyway); every chained
// grid waits (griddepcontrol.wait) for its upstream grid before it exits, so completion is
// transitive and stream order holds for whatever the caller enqueues next.
// Failed matrices (pivot <= 0 or NaN) stop at the failing column and report the LAPACK info
// (SURVEY.md §8(c) readings #2-#3); nothing of them is touched again (a7).
#include <algorithm>
#include <cstdlib>
#include <atomic>
#include <mutex>

#include "common.cuh"
#include "internal.h"

namespace vb {

// Every other row block of a panel walks the k chunks backwards (produce_matrix3); 0 disables.
// Small-kernel CTAs per SM (launch bounds and grid).
#ifndef VB_SMALL_CPS
#define VB_SMALL_CPS 4
#endif
// L2 prefetch distance of the blocked kernel's A chunks (0: none).
#ifndef VB_PF
#define VB_PF 0
#endif
// 1: the blocked kernel's ring always uses the cp.async gather path (development A/B).
#ifndef VB_NOBULK
#define VB_NOBULK 0
#endif
#ifndef VB_KREV
#define VB_KREV 1
#endif
// SPOTRF's panel update on the FP32 FFMA pipe (k_loop_ffma) instead of FP64 DMMA: a measured
// experiment, off in the product (C5 FP32 174 ms vs 152 ms with DMMA); build with
// -DVB_SPOTRF_FFMA=1 to reproduce.
#ifndef VB_SPOTRF_FFMA
#define VB_SPOTRF_FFMA 0
#endif

// Optional phase timers (debug builds with -DVB_PHASE_PROF): warp 0 lane 0 of each CTA of the
// v2 kernel accumulates clock64() cycles per phase; read with vbatched_debug_phases().
#ifdef VB_PHASE_PROF
__device__ unsigned long long g_phase[8];
#define VB_T0(v) long long v = clock64();
#define VB_ADDW(i, v) \
  if ((threadIdx.x & 31) == 0) atomicAdd(&g_phase[i], (unsigned long long)(clock64() - (v)));
#define VB_ADD(i, v) \
  if (threadIdx.x == 0) atomicAdd(&g_phase[i], (unsigned long long)(clock64() - (v)));
#else
#define VB_T0(v)
#define VB_ADD(i, v)
#define VB_ADDW(i, v)
#endif
// Diagonal-block step timers (tools/diag_bench.cu built with -DVB_DIAG_PROF): thread 0
// accumulates clock64() deltas between consecutive marks into g_dprof[i].
#ifdef VB_DIAG_PROF
__device__ unsigned long long g_dprof[16];
#define DP_START long long dp_t = clock64();
#define DP_MARK(i)                                                  \
  if (threadIdx.x == 0) {                                           \
    const long long dp_n = clock64();                               \
    atomicAdd(&g_dprof[i], (unsigned long long)(dp_n - dp_t));      \
    dp_t = dp_n;                                                    \
  }
#else
#define DP_START
#define DP_MARK(i)
#endif

// Optional per-matrix timeline (debug builds with -DVB_TIMELINE): the owning CTA/warp writes
// (start ns, end ns, SM id, kernel) of each matrix to g_tl[4 m ..]; see tools/timeline.py.
#ifdef VB_TIMELINE
__device__ unsigned long long* g_tl;
VB_DEVINL unsigned long long tl_now() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#define TL_BEGIN(v) const unsigned long long v = tl_now();
#define TL_END(pred, v, m, kind)                               \
  if ((pred) && g_tl) {                                        \
    unsigned sm_;                                              \
    asm volatile("mov.u32 %0, %%smid;" : "=r"(sm_));           \
    g_tl[4 * (size_t)(m)] = v;                                 \
    g_tl[4 * (size_t)(m) + 1] = tl_now();                      \
    g_tl[4 * (size_t)(m) + 2] = sm_;                           \
    g_tl[4 * (size_t)(m) + 3] = kind;                          \
  }
#else
#define TL_BEGIN(v)
#define TL_END(pred, v, m, kind)
#endif


// Optional ring-latency records (debug builds with -DVB_CHUNK_LAT, tools/chunk_lat.py): for CTAs
// b < 64 and ring positions gi < 4096 of the blocked kernel, SM clock64() at: producer before its
// empty-slot wait (0), after it (1), after issuing the copies (2); consumer warp 0 before its
// full-barrier wait (3), after it (4). Same SM, so one clock domain per record.
#ifdef VB_CHUNK_LAT
__device__ unsigned long long* g_lat;
#define LAT_REC(gi, slot)                                                                  \
  if (g_lat && blockIdx.x < 64 && (gi) < 4096 && (threadIdx.x & 31) == 0)                   \
    g_lat[((size_t)blockIdx.x * 4096 + (gi)) * 8 + (slot)] = clock64();
#else
#define LAT_REC(gi, slot) {}
#endif

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
// 1/d for the LDL^T multipliers: hardware approximation + two Newton steps (within 1 ulp of
// the IEEE quotient; exact for powers of two). Shorter than the IEEE division sequence on the
// column-to-column chain. l_jj itself is still the IEEE correctly rounded sqrt.
VB_DEVINL double rcp_nr(double d) {
  double r;
  asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(d));
  double e = fma(-d, r, 1.0);
  r = fma(r, e, r);
  e = fma(-d, r, 1.0);
  return fma(r, e, r);
}

template <int NM>
VB_DEVINL int potf2_regs_warp(double (&a)[NM], int nb, int lane, double* ws_, double* sv,
                              double* tv) {
  double* ws = static_cast<double*>(__builtin_assume_aligned(ws_, 16));
  // Branch-free over all NM columns: the caller pads rows/columns >= nb with the identity, so
  // the padded pivots are 1 and leave the leading nb x nb factor untouched (no runtime branch
  // around the shuffles, so a[] stays in registers). The first failing pivot (j < nb) is
  // recorded and the (garbage) work after it continues; only columns before it are scaled
  // and stored, and lane j's a[j] (the failing pivot) is never modified after its column, so
  // LAPACK's convention of leaving the pivot at (j,j) holds.
  int info = 0;
  double myd = 1.0;
  double dn = a[0];  // candidate next pivot (meaningful in lane j+1)
#pragma unroll
  for (int j = 0; j < NM; ++j) {
    const double d = __shfl_sync(kFull, dn, j);
    if (!(d > 0.0) && info == 0 && j < nb) info = j + 1;
    if (lane == j) myd = d;
    const double rd = rcp_nr(d);
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
  const double isq = rcp_nr(sq);
  if (lane < ncols) {
    sv[lane] = sq;
    tv[lane] = isq;
  }
  __syncwarp();
  // selects through opaque selp: written as `if (c == lane) a[c] = sq` the compiler turns the
  // unrolled loop into one dynamically indexed store a[lane] = sq, which demotes a[] to local
  // memory for the whole factorisation
#pragma unroll
  for (int c = 0; c < NM; ++c) {
    const double v = selp(c < lane, a[c] * tv[c], sq);
    a[c] = selp(c < ncols && c <= lane, v, a[c]);
  }
  return info;
}

// ---------------------------------------------------------------------------------------
// One warp: POTF2 of the nb x nb (nb <= 32) lower block at T (T[c*ldt + r]), written back
// to T and to global (Ag, lda) — lower part, on failure up to the failing column (incl. the
// pivot). Blocked 16 + 16: POTF2 of columns 0..15 with all 32 rows in registers (which also
// produces L21), the trailing 16x16 update C22 -= L21 L21^T on DMMA, POTF2 of C22.
// sv/tv (>= 32 doubles) receive l_cc and 1/l_cc. Returns info.
template <bool UP, typename E = double>
VB_DEVINL int potf2_block32(double* T, int ldt, int nb, int lane, E* Ag, int lda,
                            double* ws, double* sv, double* tv) {
  const int nb1 = min(nb, 16), nb2 = nb - nb1;
  int info;
  {
    double a[16];  // rows/columns outside the block: identity (potf2_regs_warp is branch-free)
#pragma unroll
    for (int c = 0; c < 16; ++c)
      a[c] = (c < nb1 && lane < nb) ? T[c * ldt + lane] : selp(c == lane, 1.0, 0.0);
    info = potf2_regs_warp<16>(a, nb1, lane, ws, sv, tv);
    const int ncol = info ? info : nb1;
#pragma unroll
    for (int c = 0; c < 16; ++c)
      if (c < ncol && lane >= c && lane < nb) {
        T[c * ldt + lane] = a[c];
        Ag[gix<UP>(lane, c, lda)] = a[c];
      }
  }
  __syncwarp();
  if (info || nb2 <= 0) return info;
  {  // C22 -= L21 L21^T (rows/cols 16..31; lower tiles only)
    const int g = lane >> 2, q = lane & 3;
    double acc[2][2][2];
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
#pragma unroll
      for (int nt = 0; nt < 2; ++nt)
#pragma unroll
        for (int h = 0; h < 2; ++h)
          acc[mt][nt][h] = T[(16 + nt * 8 + 2 * q + h) * ldt + 16 + mt * 8 + g];
#pragma unroll
    for (int ks = 0; ks < 4; ++ks) {
      double fa[2], fb[2];
#pragma unroll
      for (int t = 0; t < 2; ++t) {
        fa[t] = -T[(ks * 4 + q) * ldt + 16 + t * 8 + g];
        fb[t] = T[(ks * 4 + q) * ldt + 16 + t * 8 + g];
      }
#pragma unroll
      for (int mt = 0; mt < 2; ++mt)
#pragma unroll
        for (int nt = 0; nt < 2; ++nt)
          if (nt <= mt) dmma(acc[mt][nt], fa[mt], fb[nt]);
    }
    __syncwarp();
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
#pragma unroll
      for (int nt = 0; nt < 2; ++nt)
#pragma unroll
        for (int h = 0; h < 2; ++h)
          if (nt <= mt) T[(16 + nt * 8 + 2 * q + h) * ldt + 16 + mt * 8 + g] = acc[mt][nt][h];
  }
  __syncwarp();
  {  // POTF2 of C22: lanes 0..15 own its rows (lanes 16..31 mirror them, results unused)
    const int r = lane & 15;
    double* T22 = T + 16 * ldt + 16;
    double a[16];
#pragma unroll
    for (int c = 0; c < 16; ++c) a[c] = (c < nb2 && r < nb2) ? T22[c * ldt + r] : selp(c == r, 1.0, 0.0);
    const int info2 = potf2_regs_warp<16>(a, nb2, lane, ws, sv + 16, tv + 16);
    const int ncol = info2 ? info2 : nb2;
    E* A22 = Ag + (size_t)16 * lda + 16;
#pragma unroll
    for (int c = 0; c < 16; ++c)
      if (lane < 16 && c < ncol && r >= c && r < nb2) {
        T22[c * ldt + r] = a[c];
        A22[gix<UP>(r, c, lda)] = a[c];
      }
    info = info2 ? 16 + info2 : 0;
  }
  __syncwarp();
  return info;
}

// 32x32x32 DMMA products on a 4-warp group (wg = warp index 0..3): each warp owns a 16x16
// quarter (2x2 tiles). acc[m][n] += sum_k fa(m,k) fb(k,n) over k = 0..31.
template <class FA, class FB>
VB_DEVINL void mm32_quarter(double (&acc)[2][2][2], int wg, int lane, FA fa, FB fb) {
  const int g = lane >> 2, q = lane & 3;
  const int m0 = (wg >> 1) * 16, n0 = (wg & 1) * 16;
#pragma unroll
  for (int ks = 0; ks < 8; ++ks) {
    double a[2], b[2];
#pragma unroll
    for (int mt = 0; mt < 2; ++mt) a[mt] = fa(m0 + mt * 8 + g, ks * 4 + q);
#pragma unroll
    for (int nt = 0; nt < 2; ++nt) b[nt] = fb(ks * 4 + q, n0 + nt * 8 + g);
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
#pragma unroll
      for (int nt = 0; nt < 2; ++nt) dmma(acc[mt][nt], a[mt], b[nt]);
  }
}


// =======================================================================================
// Blocked kernel (n > ts) building blocks: warp w owns 16 full rows of each MB-row block, so
// the TRSM runs from registers and stores straight to global; the TMA stage ring is not
// aliased with anything, so the producer keeps prefetching across row blocks and panels.
// E: the matrices' storage type (double for DPOTRF, float for SPOTRF); the ring stages hold E,
// everything from the fragments on is FP64 (DMMA). Ring leading dims padded so that the
// DMMA fragment loads are bank-conflict free (+4 doubles / +8 floats); with VB_SPOTRF_FFMA the
// FP32 stages are read only by the FFMA k-loop, whose lanes all read the same k row (no padding).
template <int NB_, int KC_, int STAGES_, int MINB_, int WARPS_ = 8, typename E_ = double>
struct Cfg2 {
  using E = E_;
  static constexpr int NB = NB_, KC = KC_, STAGES = STAGES_, MINB = MINB_;
  static constexpr int WARPS = WARPS_;       // compute warps (16 rows each)
  static constexpr int THREADS = 32 * WARPS, MB = 16 * WARPS, NT = NB / 8;
  static constexpr int PAD = sizeof(E_) == 8 ? 4 : (VB_SPOTRF_FFMA ? 0 : 8);
  static constexpr int LDA = MB + PAD, LDB = NB + PAD, LDT = NB + 4;
  static constexpr int G = 16 / (int)sizeof(E_);  // elements per 16 bytes (bulk-copy granule)
};
// 3 CTAs/SM: 4 compute warps (MB = NB) + 1 producer; ring of 2 x 16-column chunks (measured
// against 3 x 8 and 4 x 8: C5 154.4 / 160.5 vs 152.3 ms, the per-chunk barrier cost dominates)
using Cfg64d = Cfg2<64, 16, 2, 3, 4>;
// FP32 storage (SPOTRF). With the FFMA k-loop the unpadded 16-column FP32 chunks leave room for a
// third ring stage.
using Cfg64s = Cfg2<64, 16, VB_SPOTRF_FFMA ? 3 : 2, 3, 4, float>;

template <class C>
struct Smem2 {
  alignas(16) typename C::E a[C::STAGES][C::KC][C::LDA];  // A chunk: [k][row]
  alignas(16) typename C::E b[C::STAGES][C::KC][C::LDB];  // B chunk: [k][panel row]
  // Diagonal block T[c][r]. After diag_block64v2: T11 slot = inv(L22) as B operand,
  // T12 slot (cols 32..63, rows 0..31) = inv(L11) as B operand, T21 = L21, T22 = L22.
  double T[C::NB][C::LDT];
  double S[16 * LDS_T];  // TRTRI scratch
  double wbuf[64];
  double sv[C::NB];
  double tv[C::NB];
  // VB_SPOTRF_FFMA only: per-warp staging of the FFMA k-loop's FP32 partial sums (one 16 x 32
  // half of the warp's 16 x 64 tile at a time) on their way into the FP64 fragment layout
  alignas(16) float xs[(VB_SPOTRF_FFMA && sizeof(typename C::E) == 4) ? C::WARPS : 1][16][40];
  uint64_t full[C::STAGES];
  uint64_t empty[C::STAGES];
  uint64_t panel_done;  // v3: one phase per panel (8 consumer-warp arrivals)
  uint32_t chunks;  // chunks issued so far (ring position)
  int item;
  int info;
};

static_assert(sizeof(Smem2<Cfg64d>) + 1024 <= 228 * 1024 / 3, "3 CTAs/SM");
static_assert(sizeof(Smem2<Cfg64s>) + 1024 <= 228 * 1024 / 3, "3 CTAs/SM");

// Diagonal 64x64 block by warps 0..3 (named barrier 1): L11 = potf2(C11), inv(L11) -> T12,
// L21 = C21 inv(L11)^T -> T21, C22 -= L21 L21^T, L22 = potf2(C22), inv(L22) -> T11.
// Stores L11, L21, L22 (rows < nb) to global (Ad, ld). Sets s.info (1-based, in-block).
template <class CC, bool UP>
__device__ __noinline__ void diag_block64v2(Smem2<CC>& s, int nb, int wg, int lane,
                                            typename CC::E* Ad,
                                            int ld, bool below) {
  constexpr int LDT = CC::LDT;
  double* T = &s.T[0][0];
  double* INV11 = T + 32 * LDT;  // T12 slot: INV11[k*LDT + n]
  double* INV22 = T;             // T11 slot (after L11 is dead)
  const int g = lane >> 2, q = lane & 3;
  const int m0 = (wg >> 1) * 16, n0 = (wg & 1) * 16;
  const int nb1 = min(nb, 32), nb2 = nb - nb1;
  DP_START
  if (wg == 0) {
    const int info = potf2_block32<UP>(T, LDT, nb1, lane, Ad, ld, s.wbuf, s.sv, s.tv);
    DP_MARK(0)
    if (!info && nb2 > 0) trtri32_dmma_warp(T, LDT, s.tv, INV11, LDT, s.S, LDS_T, lane);
    DP_MARK(1)
    if (lane == 0) s.info = info;
  }
  bar_group(1, 128);
  DP_MARK(2)
  if (s.info || nb2 == 0) return;
  {  // L21 = C21 inv(L11)^T
    double acc[2][2][2] = {};
    mm32_quarter(acc, wg, lane, [&](int m, int k) { return T[k * LDT + 32 + m]; },
                 [&](int k, int n) { return INV11[k * LDT + n]; });
    bar_group(1, 128);
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
#pragma unroll
      for (int nt = 0; nt < 2; ++nt)
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const int r = 32 + m0 + mt * 8 + g, c = n0 + nt * 8 + 2 * q + h;
          T[c * LDT + r] = acc[mt][nt][h];
          if (r < nb) Ad[gix<UP>(r, c, ld)] = acc[mt][nt][h];
        }
  }
  bar_group(1, 128);
  DP_MARK(3)
  {  // C22 -= L21 L21^T
    double acc[2][2][2];
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
#pragma unroll
      for (int nt = 0; nt < 2; ++nt)
#pragma unroll
        for (int h = 0; h < 2; ++h)
          acc[mt][nt][h] = T[(32 + n0 + nt * 8 + 2 * q + h) * LDT + 32 + m0 + mt * 8 + g];
    mm32_quarter(acc, wg, lane, [&](int m, int k) { return -T[k * LDT + 32 + m]; },
                 [&](int k, int n) { return T[k * LDT + 32 + n]; });
    bar_group(1, 128);
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
#pragma unroll
      for (int nt = 0; nt < 2; ++nt)
#pragma unroll
        for (int h = 0; h < 2; ++h)
          T[(32 + n0 + nt * 8 + 2 * q + h) * LDT + 32 + m0 + mt * 8 + g] = acc[mt][nt][h];
  }
  bar_group(1, 128);
  DP_MARK(4)
  if (wg == 0) {
    double* T22 = T + 32 * LDT + 32;
    const int info = potf2_block32<UP>(T22, LDT, nb2, lane, Ad + (size_t)32 * ld + 32, ld, s.wbuf,
                                   s.sv + 32, s.tv + 32);
    DP_MARK(5)
    if (!info && below) trtri32_dmma_warp(T22, LDT, s.tv + 32, INV22, LDT, s.S, LDS_T, lane);
    DP_MARK(6)
    if (lane == 0) s.info = info ? 32 + info : 0;
  }
  bar_group(1, 128);
  DP_MARK(7)
}

// Producer (warp 0): chunk kc of the row block at r0 into ring slot gi % STAGES.
template <class C, bool UP>
VB_DEVINL void issue_chunk2(Smem2<C>& s, uint32_t gi, int kc, const typename C::E* A, int n,
                            int ld, int r0, int j0, int lane, bool bulk, int mrows = C::MB) {
  using E = typename C::E;
  constexpr int G = C::G;
  const int st = gi % C::STAGES;
  const uint32_t u = gi / C::STAGES;
  const int k0 = kc * C::KC;
  LAT_REC(gi, 0)
  if (lane == 0 && u > 0) mbar_wait(&s.empty[st], (u - 1) & 1);
  __syncwarp();
  LAT_REC(gi, 1)
  if (bulk) {
    // segments rounded up to 16 bytes: the extra rows lie inside ldda (ldda is a multiple of
    // G here) and only ever feed output rows/columns that are never stored
    const int ra = (min(mrows, n - r0) + G - 1) / G * G;
    const int rb = (min(C::NB, n - j0) + G - 1) / G * G;
    // the full barrier expects 32 arrivals per phase (one per producer lane on the gather path
    // below); here lane 0 posts the transaction bytes and the 32 arrivals itself
    if (lane == 0) {  // the phase's transaction bytes, then all 32 expected arrivals at once
      mbar_expect_tx(&s.full[st], (uint32_t)(C::KC * (ra + rb) * (int)sizeof(E)));
      mbar_arrive_cnt(&s.full[st], 32);
    }
    __syncwarp();
    if (lane < C::KC) {
      // A rows stream (re-read only a panel later): evict first; the panel rows are re-read
      // for every row block of the panel: evict last (C5 DRAM traffic and time)
      bulk_g2s_hint(&s.a[st][lane][0], A + (size_t)(k0 + lane) * ld + r0, ra * sizeof(E),
                    &s.full[st], policy_evict_first());
    } else if (lane >= 16 && lane < 16 + C::KC) {
      const int c = lane - 16;
      bulk_g2s_hint(&s.b[st][c][0], A + (size_t)(k0 + c) * ld + j0, rb * sizeof(E), &s.full[st],
                    policy_evict_last());
    }
  } else {
    // Odd ldda / unaligned base ('L'), or uplo 'U': the chunk is gathered with 8-byte cp.async
    // (LDGSTS, no register staging; rows >= n are zero-filled). 'L': lanes run down a column;
    // 'U': L's rows are contiguous in storage (16 k-values of one row = 128 B), 16 lanes per
    // row. Each lane's arrival on the full barrier is its cp.async.mbarrier.arrive.noinc,
    // triggered when all of that lane's copies have landed (32 expected arrivals per phase).
    static_assert((C::KC == 8 || C::KC == 16) && C::MB % 32 == 0 && C::NB % 32 == 0, "copy shapes");
    if (UP) {
      constexpr int RS = 32 / C::KC;  // rows per pass (KC lanes per row)
      const int c = lane % C::KC;
#pragma unroll 4
      for (int r = lane / C::KC; r < C::MB; r += RS) {
        const bool p = r < mrows && r0 + r < n;
        cp_async_e<E>(&s.a[st][c][r], A + (p ? (size_t)(r0 + r) * ld + k0 + c : 0), p);
      }
#pragma unroll 4
      for (int r = lane / C::KC; r < C::NB; r += RS) {
        const bool p = j0 + r < n;
        cp_async_e<E>(&s.b[st][c][r], A + (p ? (size_t)(j0 + r) * ld + k0 + c : 0), p);
      }
    } else {
#pragma unroll 4
      for (int c = 0; c < C::KC; ++c) {
        const E* col = A + (size_t)(k0 + c) * ld;
#pragma unroll
        for (int r = lane; r < C::MB; r += 32) {
          const bool p = r < mrows && r0 + r < n;
          cp_async_e<E>(&s.a[st][c][r], p ? col + r0 + r : A, p);
        }
#pragma unroll
        for (int r = lane; r < C::NB; r += 32) {
          const bool p = j0 + r < n;
          cp_async_e<E>(&s.b[st][c][r], p ? col + j0 + r : A, p);
        }
      }
    }
    cp_async_mbar_arrive_noinc(&s.full[st]);
  }
  LAT_REC(gi, 2)
}

// TRSM of this warp's 16 rows, in registers: X = C inv(L)^T (NB = 64: two 32-column steps
// with inv(L11), L21, inv(L22)). Operands as B fragments: inv11[k*ldo + n] = inv(L11)[n][k],
// l21[k*ldo + n] = L21[n][k], inv22[k*ldo + n] = inv(L22)[n][k]. Result overwrites acc.
VB_DEVINL void trsm_regs64_ops(const double* inv11, const double* l21, const double* inv22, int ldo,
                               double (&acc)[2][8][2], int lane) {
  const int g = lane >> 2, q = lane & 3;
  double x[2][4][2];
  // X1 = C1 inv(L11)^T
#pragma unroll
  for (int mt = 0; mt < 2; ++mt)
#pragma unroll
    for (int nt = 0; nt < 4; ++nt) x[mt][nt][0] = x[mt][nt][1] = 0.0;
#pragma unroll
  for (int ks = 0; ks < 8; ++ks) {
    double fa[2], fb[4];
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
      fa[mt] = cfrag_to_afrag(acc[mt][ks >> 1][0], acc[mt][ks >> 1][1], ks & 1, lane);
#pragma unroll
    for (int nt = 0; nt < 4; ++nt) fb[nt] = inv11[(ks * 4 + q) * ldo + nt * 8 + g];
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
#pragma unroll
      for (int nt = 0; nt < 4; ++nt)
        if (4 * ks <= 8 * nt + 7) dmma(x[mt][nt], fa[mt], fb[nt]);  // inv(L11)^T is upper
  }
  // C2 -= X1 L21^T
#pragma unroll
  for (int ks = 0; ks < 8; ++ks) {
    double fa[2], fb[4];
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
      fa[mt] = -cfrag_to_afrag(x[mt][ks >> 1][0], x[mt][ks >> 1][1], ks & 1, lane);
#pragma unroll
    for (int nt = 0; nt < 4; ++nt) fb[nt] = l21[(ks * 4 + q) * ldo + nt * 8 + g];
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
#pragma unroll
      for (int nt = 0; nt < 4; ++nt) dmma(acc[mt][4 + nt], fa[mt], fb[nt]);
  }
#pragma unroll
  for (int mt = 0; mt < 2; ++mt)
#pragma unroll
    for (int nt = 0; nt < 4; ++nt) {
      acc[mt][nt][0] = x[mt][nt][0];
      acc[mt][nt][1] = x[mt][nt][1];
      x[mt][nt][0] = x[mt][nt][1] = 0.0;
    }
  // X2 = C2 inv(L22)^T
#pragma unroll
  for (int ks = 0; ks < 8; ++ks) {
    double fa[2], fb[4];
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
      fa[mt] = cfrag_to_afrag(acc[mt][4 + (ks >> 1)][0], acc[mt][4 + (ks >> 1)][1], ks & 1, lane);
#pragma unroll
    for (int nt = 0; nt < 4; ++nt) fb[nt] = inv22[(ks * 4 + q) * ldo + nt * 8 + g];
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
#pragma unroll
      for (int nt = 0; nt < 4; ++nt)
        if (4 * ks <= 8 * nt + 7) dmma(x[mt][nt], fa[mt], fb[nt]);  // inv(L22)^T is upper
  }
#pragma unroll
  for (int mt = 0; mt < 2; ++mt)
#pragma unroll
    for (int nt = 0; nt < 4; ++nt) {
      acc[mt][4 + nt][0] = x[mt][nt][0];
      acc[mt][4 + nt][1] = x[mt][nt][1];
    }
}

// The same with the operands in the diagonal tile s.T after diag_block64v2: T12 slot = inv(L11),
// T21 = L21, T11 slot = inv(L22).
template <class CC>
VB_DEVINL void trsm_regs64(Smem2<CC>& s, double (&acc)[2][8][2], int lane) {
  constexpr int LDT = CC::LDT;
  const double* T = &s.T[0][0];
  trsm_regs64_ops(T + 32 * LDT, T + 32, T, LDT, acc, lane);
}

// =======================================================================================
// v3 blocked kernel (large n): v2 plus a dedicated TMA producer warp (warp 8). Measured in
// tools/kloop_bench.cu: when a compute warp also produces, the k-loop stalls on the
// producer/consumer handshake (16.6 TF/s at one CTA per SM); a producer warp that never
// computes lifts it to 29 (one CTA) / 31.8 TF/s (two CTAs per SM). The producer walks the
// same chunk sequence as the consumers; before the chunks of panel p it waits on the
// panel_done mbarrier for panel p-1 (the consumers arrive after storing and fencing that
// panel's L), so TMA never reads a column before it is final.

template <class C, bool UP>
VB_DEVINL void produce_matrix3(Smem2<C>& s, const typename C::E* A, int n, int ld, int lane,
                               uint32_t& gchunk, uint32_t& gpanel) {
  constexpr int NB = C::NB, MB = C::MB, KC = C::KC;
  using E = typename C::E;
  constexpr int G = C::G;
  const bool bulk = !VB_NOBULK && !UP && ((reinterpret_cast<uintptr_t>(A) & 15) == 0) && (ld % G == 0);
  const int npan = (n + NB - 1) / NB;
  int done = npan;  // panels the consumers will complete for this matrix
  fence_proxy_async();
  for (int p = 1; p < npan; ++p) {
    const int j0 = p * NB, nk = j0 / KC;
    // The first row block's chunks that read only columns < j0 - NB (final since before
    // panel p-1 started) are issued before waiting for panel p-1: the ring does not drain
    // at the panel boundary. Everything after them reads panel p-1's columns.
    const int nk_free = (j0 - NB) / KC;
    if (bulk && lane < min(NB, n - j0)) {
      const int rn = (min(MB, n - j0) + G - 1) / G * G;
      bulk_prefetch_l2(A + (size_t)(j0 + lane) * ld + j0, rn * (int)sizeof(E));
    }
    // L2 prefetch of the A chunk VB_PF chunks ahead of the one being issued (the ring holds one)
    auto pf = [&](int r0, int kcp, int lim) {
      if (VB_PF > 0 && bulk && kcp >= 0 && kcp < lim && lane < KC) {
        const int ra = (min(MB, n - r0) + G - 1) / G * G;
        bulk_prefetch_l2(A + (size_t)(kcp * KC + lane) * ld + r0, ra * (int)sizeof(E));
      }
    };
    for (int kc = 0; kc < nk_free; ++kc) {
      pf(j0, kc + VB_PF, nk_free);
      issue_chunk2<C, UP>(s, gchunk++, kc, A, n, ld, j0, j0, lane, bulk);
    }
    if (lane == 0) mbar_wait(&s.panel_done, (gpanel + p - 1) & 1);  // panel p-1 is stored
    __syncwarp();
    if (s.info) {  // the consumers failed in panel p-1 and stop there (they also drain the
      done = p;    // nk_free chunks issued above, see consume_matrix3)
      break;
    }
    for (int r0 = j0; r0 < n; r0 += MB) {
      if (r0 > j0 && bulk && lane < min(NB, n - j0)) {  // warm L2 with this block's panel values
        const int rn = (min(MB, n - r0) + G - 1) / G * G;
        bulk_prefetch_l2(A + (size_t)(j0 + lane) * ld + r0, rn * (int)sizeof(E));
      }
      // Every other row block walks the k chunks backwards, so the panel rows' chunks it reads
      // first are the ones the previous block read last (still in L2)
      const bool rev = VB_KREV && (((r0 - j0) / MB) & 1);
      for (int i = (r0 == j0 ? nk_free : 0); i < nk; ++i) {
        pf(r0, rev ? nk - 1 - (i + VB_PF) : i + VB_PF, nk);
        issue_chunk2<C, UP>(s, gchunk++, rev ? nk - 1 - i : i, A, n, ld, r0, j0, lane, bulk);
      }
    }
  }
  gpanel += done;
}

// Consumer k-loop over nk chunks of the ring for this warp's 16 rows and the first NTL
// 8-column tiles (NTL = 0: consume without computing — rows beyond n).
template <class C, int NTL>
VB_DEVINL void k_loop3(Smem2<C>& s, double (&acc)[2][C::NT][2], uint32_t& gchunk, int nk, int wrow,
                       int lane) {
  const int g = lane >> 2, q = lane & 3;
  for (int kc = 0; kc < nk; ++kc) {
    const uint32_t gi = gchunk++;
    const int st = gi % C::STAGES;
    if (threadIdx.x < 32) { LAT_REC(gi, 3) }
    mbar_wait(&s.full[st], (gi / C::STAGES) & 1);
    if (threadIdx.x < 32) { LAT_REC(gi, 4) }
    if constexpr (NTL > 0) {
#pragma unroll
      for (int kk = 0; kk < C::KC / 4; ++kk) {
        double fa[2], fb[NTL];
#pragma unroll
        for (int mt = 0; mt < 2; ++mt) fa[mt] = -(double)s.a[st][kk * 4 + q][wrow + mt * 8 + g];
#pragma unroll
        for (int nt = 0; nt < NTL; ++nt) fb[nt] = (double)s.b[st][kk * 4 + q][nt * 8 + g];
#pragma unroll
        for (int mt = 0; mt < 2; ++mt)
#pragma unroll
          for (int nt = 0; nt < NTL; ++nt) dmma(acc[mt][nt], fa[mt], fb[nt]);
      }
      // Release of the slot to the TMA producer. The slot was read by generic-proxy LDS and is
      // refilled through the async proxy: without this fence ptxas issues the arrive while the
      // last LDS of the chunk are still in flight (their DMMAs are scheduled after it) and the
      // refill can overtake them (a measured 1-in-10 run-to-run difference at C3).
      fence_proxy_async();
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&s.empty[st]);
  }
}

// VB_SPOTRF_FFMA (FP32 storage): the panel update -= L[r0:, 0:j0] L[j0:j0+64, 0:j0]^T on the FP32
// FFMA pipe instead of DMMA. Register tile 4 rows x 8 columns per lane
// (rows wrow + 4 rg .. +3, columns 4 cg .. +3 and 32 + 4 cg .. +3; rg = lane / 8, cg = lane % 8):
// per k one LDS.128 of A (broadcast) and two LDS.128 of B feed 32 FFMAs. HALF: the columns
// 32..63 are skipped (a panel's first row block, warps whose rows are all < 32). The FP32 sums
// join A's values in FP64 in ffma_to_acc; everything after the update stays FP64.
template <class C, bool HALF>
VB_DEVINL void k_loop_ffma(Smem2<C>& s, float (&c)[4][8], uint32_t& gchunk, int nk, int wrow,
                           int lane) {
  const int rg = lane >> 3, cg = lane & 7;
  for (int kc = 0; kc < nk; ++kc) {
    const uint32_t gi = gchunk++;
    const int st = gi % C::STAGES;
    mbar_wait(&s.full[st], (gi / C::STAGES) & 1);
#pragma unroll
    for (int k = 0; k < C::KC; ++k) {
      const float4 a = *reinterpret_cast<const float4*>(&s.a[st][k][wrow + rg * 4]);
      const float4 b0 = *reinterpret_cast<const float4*>(&s.b[st][k][cg * 4]);
      const float av[4] = {a.x, a.y, a.z, a.w};
      float bv[8] = {b0.x, b0.y, b0.z, b0.w, 0.f, 0.f, 0.f, 0.f};
      if (!HALF) {
        const float4 b1 = *reinterpret_cast<const float4*>(&s.b[st][k][32 + cg * 4]);
        bv[4] = b1.x;
        bv[5] = b1.y;
        bv[6] = b1.z;
        bv[7] = b1.w;
      }
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < (HALF ? 4 : 8); ++j) c[i][j] = fmaf(-av[i], bv[j], c[i][j]);
    }
    fence_proxy_async();  // see k_loop3
    __syncwarp();
    if (lane == 0) mbar_arrive(&s.empty[st]);
  }
}

// acc (FP64 fragment layout) = A's values a0 + the FFMA tile c, through the warp's xs staging in
// two 32-column halves (STS.128 per lane row, LDS.64 in the fragment layout; row stride 40 floats
// keeps each half-warp on 32 distinct banks).
template <class C>
VB_DEVINL void ffma_to_acc(Smem2<C>& s, const float (&c)[4][8], const float (&a0)[2][C::NT][2],
                           double (&acc)[2][C::NT][2], int warp, int lane) {
  const int rg = lane >> 3, cg = lane & 7, g = lane >> 2, q = lane & 3;
  float(*x)[40] = s.xs[warp];
#pragma unroll
  for (int h = 0; h < 2; ++h) {
#pragma unroll
    for (int i = 0; i < 4; ++i)
      *reinterpret_cast<float4*>(&x[rg * 4 + i][cg * 4]) =
          make_float4(c[i][4 * h], c[i][4 * h + 1], c[i][4 * h + 2], c[i][4 * h + 3]);
    __syncwarp();
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
#pragma unroll
      for (int nt = 0; nt < 4; ++nt) {
        const float2 v = *reinterpret_cast<const float2*>(&x[mt * 8 + g][nt * 8 + 2 * q]);
        acc[mt][4 * h + nt][0] = (double)a0[mt][4 * h + nt][0] + (double)v.x;
        acc[mt][4 * h + nt][1] = (double)a0[mt][4 * h + nt][1] + (double)v.y;
      }
    __syncwarp();
  }
}

template <class C, bool UP>
VB_DEVINL void consume_matrix3(Smem2<C>& s, typename C::E* __restrict__ A, int n, int ld,
                               int* info_out, uint32_t& gchunk, uint32_t& gpanel) {
  constexpr int NB = C::NB, MB = C::MB, KC = C::KC, STAGES = C::STAGES, NT = C::NT;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int g = lane >> 2, q = lane & 3;
  const int wrow = warp * 16;
  constexpr int CT = 32 * C::WARPS;  // consumer threads (named barriers)
  int npan_done = 0;
  for (int j0 = 0; j0 < n; j0 += NB) {
    const int nb = min(NB, n - j0);
    const int nk = j0 / KC;
    bool failed = false;
    for (int r0 = j0; r0 < n; r0 += MB) {
      const bool first = (r0 == j0);
      const bool active = (r0 + wrow) < n;
      if (failed) {  // drain this panel's remaining chunks (already issued by the producer)
        for (int kc = 0; kc < nk; ++kc) {
          const uint32_t gi = gchunk++;
          mbar_wait(&s.full[gi % STAGES], (gi / STAGES) & 1);
          __syncwarp();
          if (lane == 0) mbar_arrive(&s.empty[gi % STAGES]);
        }
        continue;
      }
      // A's panel values in the storage type (FP32 for SPOTRF), entries outside the panel's
      // lower part 0
      using E = typename C::E;
      constexpr bool kFfma = VB_SPOTRF_FFMA && sizeof(E) == 4;
      E a0[2][NT][2];
#pragma unroll
      for (int mt = 0; mt < 2; ++mt)
#pragma unroll
        for (int nt = 0; nt < NT; ++nt)
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            const int row = r0 + wrow + mt * 8 + g, col = j0 + nt * 8 + 2 * q + h;
            const bool v = row < n && col < j0 + nb && row >= col;
            a0[mt][nt][h] = v ? __ldcg(A + gix<UP>(row, col, ld)) : E(0);
          }
      double acc[2][NT][2];
      if constexpr (!kFfma) {
#pragma unroll
        for (int mt = 0; mt < 2; ++mt)
#pragma unroll
          for (int nt = 0; nt < NT; ++nt)
#pragma unroll
            for (int h = 0; h < 2; ++h) acc[mt][nt][h] = a0[mt][nt][h];
      }
      VB_T0(t_k)
      // In a panel's first row block the diagonal-block warps only need the column tiles on
      // or below their rows (SYRK): compile-time variants skip the strictly upper tiles.
      const int ntl = (first && wrow < NB) ? (wrow + 16) / 8 : NT;
      if (!active) {
        k_loop3<C, 0>(s, acc, gchunk, nk, wrow, lane);
        if constexpr (kFfma) {
#pragma unroll
          for (int mt = 0; mt < 2; ++mt)
#pragma unroll
            for (int nt = 0; nt < NT; ++nt)
#pragma unroll
              for (int h = 0; h < 2; ++h) acc[mt][nt][h] = a0[mt][nt][h];
        }
      } else if constexpr (kFfma) {
        float c[4][8];
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
          for (int j = 0; j < 8; ++j) c[i][j] = 0.f;
        if (ntl <= 4)
          k_loop_ffma<C, true>(s, c, gchunk, nk, wrow, lane);
        else
          k_loop_ffma<C, false>(s, c, gchunk, nk, wrow, lane);
        // entries outside the panel's lower part (stale ring rows/columns included) are dropped
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
          for (int j = 0; j < 8; ++j) {
            const int row = r0 + wrow + (lane >> 3) * 4 + i;
            const int col = j0 + (j < 4 ? 0 : 32) + (lane & 7) * 4 + (j & 3);
            c[i][j] = (row < n && col < j0 + nb && row >= col) ? c[i][j] : 0.f;
          }
        ffma_to_acc<C>(s, c, a0, acc, warp, lane);
      } else if (ntl == 2) {
        k_loop3<C, 2>(s, acc, gchunk, nk, wrow, lane);
      } else if (ntl == 4) {
        k_loop3<C, 4>(s, acc, gchunk, nk, wrow, lane);
      } else if (ntl == 6) {
        k_loop3<C, 6>(s, acc, gchunk, nk, wrow, lane);
      } else {
        k_loop3<C, NT>(s, acc, gchunk, nk, wrow, lane);
      }
      VB_ADD(0, t_k)
      VB_T0(t_d)
      if (first) {
        const bool below = r0 + nb < n;
        const bool diag_warp = warp < NB / 16;
        if (diag_warp) {
#pragma unroll
          for (int mt = 0; mt < 2; ++mt)
#pragma unroll
            for (int nt = 0; nt < NT; ++nt) {
              s.T[nt * 8 + 2 * q][wrow + mt * 8 + g] = acc[mt][nt][0];
              s.T[nt * 8 + 2 * q + 1][wrow + mt * 8 + g] = acc[mt][nt][1];
            }
          bar_group(2, CT);
          diag_block64v2<C, UP>(s, nb, warp, lane, A + (size_t)j0 * ld + j0, ld, below);
          bar_group(3, CT);
          failed = s.info != 0;
        } else {
          bar_group(2, CT);
          bar_group(3, CT);
          failed = s.info != 0;
          if (!failed && below && active) {
            trsm_regs64(s, acc, lane);
#pragma unroll
            for (int mt = 0; mt < 2; ++mt)
#pragma unroll
              for (int nt = 0; nt < NT; ++nt)
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                  const int row = r0 + wrow + mt * 8 + g, col = nt * 8 + 2 * q + h;
                  if (row < n && row >= j0 + nb && col < nb)
                    A[gix<UP>(row, j0 + col, ld)] = acc[mt][nt][h];
                }
          }
        }
        VB_ADD(1, t_d)
        if (failed && tid == 0) *info_out = j0 + s.info;
        continue;
      }
      VB_T0(t_t)
      if (active) {
        trsm_regs64(s, acc, lane);
#pragma unroll
        for (int mt = 0; mt < 2; ++mt)
#pragma unroll
          for (int nt = 0; nt < NT; ++nt)
#pragma unroll
            for (int h = 0; h < 2; ++h) {
              const int row = r0 + wrow + mt * 8 + g, col = nt * 8 + 2 * q + h;
              if (row < n && col < nb) A[gix<UP>(row, j0 + col, ld)] = acc[mt][nt][h];
            }
      }
      VB_ADD(2, t_t)
    }
    // panel end: this warp's L stores are fenced for the async proxy, then released to the
    // producer (which waits before issuing the next panel's reads of them)
    fence_proxy_async_global();
    __syncwarp();
    if (lane == 0) mbar_arrive(&s.panel_done);
    ++npan_done;
    if (failed) {
      // the producer issued the next panel's first nk (= j0 / KC) independent chunks before
      // it learnt of the failure: consume them too, so the ring stays consistent
      if (j0 + NB < n) {
        for (int kc = 0; kc < nk; ++kc) {
          const uint32_t gi = gchunk++;
          mbar_wait(&s.full[gi % STAGES], (gi / STAGES) & 1);
          __syncwarp();
          if (lane == 0) mbar_arrive(&s.empty[gi % STAGES]);
        }
      }
      break;
    }
  }
  gpanel += npan_done;
}

template <class C, bool UP>
__global__ void __launch_bounds__(32 * (C::WARPS + 1), C::MINB)
    potrf_blocked3_kernel(const int* __restrict__ d_n, typename C::E* const* __restrict__ dA,
                          const int* __restrict__ d_ldda, int* __restrict__ d_info,
                          const Ctrl* __restrict__ ctrl_c, const int* __restrict__ order,
                          int range, int wait_upstream) {
  constexpr int kV3Consumers = C::WARPS;
  extern __shared__ __align__(128) unsigned char smem_raw3[];
  Smem2<C>& s = *reinterpret_cast<Smem2<C>*>(smem_raw3);
  Ctrl* ctrl = const_cast<Ctrl*>(ctrl_c);
  if (threadIdx.x == 0) {
    for (int i = 0; i < C::STAGES; ++i) {
      mbar_init(&s.full[i], 32);  // 32 arrivals per phase (see issue_chunk2)
      mbar_init(&s.empty[i], kV3Consumers);
    }
    mbar_init(&s.panel_done, kV3Consumers);
    s.info = 0;
    fence_proxy_async();
  }
  __syncthreads();
  if (wait_upstream) pdl_wait();
  pdl_launch_dependents();
  const int count = *(volatile const int*)&ctrl->count[range];
  const int start = *(volatile const int*)&ctrl->start[range];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  uint32_t gchunk = 0, gpanel = 0;
  for (;;) {
    if (tid == 0) s.item = atomicAdd(&ctrl->head[range], 1);
    __syncthreads();
    const int it = s.item;
    __syncthreads();
    if (it >= count) break;
    const int m = order[start + it];
    TL_BEGIN(t_tl)
    if (warp == kV3Consumers) {
      produce_matrix3<C, UP>(s, dA[m], d_n[m], d_ldda[m], lane, gchunk, gpanel);
    } else {
      VB_T0(t_m)
      consume_matrix3<C, UP>(s, dA[m], d_n[m], d_ldda[m], d_info + m, gchunk, gpanel);
      VB_ADD(4, t_m)
    }
    TL_END(tid == 0, t_tl, m, 30)
  }
  // Chained without waiting (wait_upstream == 0): hold this grid's completion until the
  // upstream grid has completed, so that completion stays transitive along the PDL chain and
  // stream successors (workspace free, caller kernels) see every earlier grid finished. One
  // thread of CTA 0 is enough (a grid completes when its last CTA exits); the other CTAs leave
  // at once and free their SM slots for the next grid.
  if (!wait_upstream && blockIdx.x == 0 && threadIdx.x == 0) pdl_wait();
}

// =======================================================================================
// Small-matrix kernel (32 < n <= ts): one CTA of 2 warps per matrix, ~10 CTAs per SM, so
// ~20 small matrices are in flight per SM (the regime is HBM/latency bound: C2). Left-
// looking with NB = 32; within a panel the 32-row blocks alternate between the two warps
// (block 0 = the diagonal block, always warp 0). Panel-update fragments are loaded straight
// from L2 (__ldcg) into DMMA registers; the owning warp factors the diagonal block (POTF2 +
// TRTRI in shared memory) and releases it to the other warp with a named barrier; TRSM runs
// from registers and stores directly. One __syncthreads per panel.
struct SmallSmem {
  double T[32][36];    // diagonal block, T[c][r]
  double inv[32][36];  // inv(L11) as TRSM B operand: inv[k][n] = X[n][k]
  double S[16 * LDS_T];
  double wbuf[64];
  double sv[32];
  double tv[32];
  int item;
  int info;
};

// acc (32 x 32 block at rows r0.., cols j0..) = A (its lower part when diag)
template <bool UP, typename E = double>
VB_DEVINL void small_acc_init(double (&acc)[4][4][2], const E* __restrict__ A, int n, int ld,
                              int r0, int j0, int nb, bool diag, int lane) {
  const int g = lane >> 2, q = lane & 3;
#pragma unroll
  for (int mt = 0; mt < 4; ++mt)
#pragma unroll
    for (int nt = 0; nt < 4; ++nt)
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int row = r0 + mt * 8 + g, col = j0 + nt * 8 + 2 * q + h;
        const bool v = row < n && col < j0 + nb && (!diag || row >= col);
        acc[mt][nt][h] = v ? __ldcg(A + gix<UP>(row, col, ld)) : 0.0;
      }
}

// Number of 8-row (8-column) DMMA tiles of a 32-wide block starting at r0 that hold rows < n
// (warp-uniform). Tiles entirely outside the matrix are skipped: no loads, no DMMAs.
VB_DEVINL int tiles8(int n, int r0) { return max(0, min(4, (n - r0 + 7) >> 3)); }

// acc -= L[r0:r0+32, kb:ke] L[j0:j0+32, kb:ke]^T, fragments straight from L2 (k ascending),
// for the first MT row tiles and NT column tiles (DIAG: only the tiles on or below the
// diagonal, nt <= mt). Compile-time tile counts: no predicates inside the unrolled loop.
template <bool UP, typename E, int MT, int NT, bool DIAG>
VB_DEVINL void small_kloop_t(double (&acc)[4][4][2], const E* __restrict__ A, int n, int ld,
                             int r0, int j0, int kb, int ke, int lane) {
  const int g = lane >> 2, q = lane & 3;
  const E* pa[MT];
  const E* pb[NT];
  bool rv[MT], cv[NT];
#pragma unroll
  for (int t = 0; t < MT; ++t) {
    rv[t] = r0 + t * 8 + g < n;
    pa[t] = A + gix<UP>(rv[t] ? r0 + t * 8 + g : 0, 0, ld);
  }
#pragma unroll
  for (int t = 0; t < NT; ++t) {
    cv[t] = j0 + t * 8 + g < n;
    pb[t] = A + gix<UP>(cv[t] ? j0 + t * 8 + g : 0, 0, ld);
  }
  const size_t kstride = UP ? 1 : (size_t)ld;
#pragma unroll 2
  for (int k0 = kb; k0 < ke; k0 += 4) {  // warp-uniform trip count (mma.sync.aligned)
    const int k = k0 + q;
    double fa[MT], fb[NT];
#pragma unroll
    for (int t = 0; t < MT; ++t) fa[t] = rv[t] ? -(double)__ldcg(pa[t] + k * kstride) : 0.0;
#pragma unroll
    for (int t = 0; t < NT; ++t) fb[t] = cv[t] ? (double)__ldcg(pb[t] + k * kstride) : 0.0;
#pragma unroll
    for (int mt = 0; mt < MT; ++mt)
#pragma unroll
      for (int nt = 0; nt < NT; ++nt)
        if (!DIAG || nt <= mt) dmma(acc[mt][nt], fa[mt], fb[nt]);
  }
}

// Dispatch on the number of 8x8 tiles holding rows/columns < n (warp-uniform): tiles entirely
// outside the matrix cost no loads and no DMMAs (C2: 1.95x -> ~1.2x the useful flops).
template <bool UP, typename E = double>
VB_DEVINL void small_kloop(double (&acc)[4][4][2], const E* __restrict__ A, int n, int ld,
                           int r0, int j0, int kb, int ke, int lane) {
  const int mtv = tiles8(n, r0);
  if (r0 == j0) {
    switch (mtv) {
      case 1: small_kloop_t<UP, E, 1, 1, true>(acc, A, n, ld, r0, j0, kb, ke, lane); break;
      case 2: small_kloop_t<UP, E, 2, 2, true>(acc, A, n, ld, r0, j0, kb, ke, lane); break;
      case 3: small_kloop_t<UP, E, 3, 3, true>(acc, A, n, ld, r0, j0, kb, ke, lane); break;
      case 4: small_kloop_t<UP, E, 4, 4, true>(acc, A, n, ld, r0, j0, kb, ke, lane); break;
      default: break;
    }
  } else {
    switch (mtv) {
      case 1: small_kloop_t<UP, E, 1, 4, false>(acc, A, n, ld, r0, j0, kb, ke, lane); break;
      case 2: small_kloop_t<UP, E, 2, 4, false>(acc, A, n, ld, r0, j0, kb, ke, lane); break;
      case 3: small_kloop_t<UP, E, 3, 4, false>(acc, A, n, ld, r0, j0, kb, ke, lane); break;
      case 4: small_kloop_t<UP, E, 4, 4, false>(acc, A, n, ld, r0, j0, kb, ke, lane); break;
      default: break;
    }
  }
}

// acc (32 x 32 block at rows r0.., cols j0..) = A - L[r0:, 0:j0] L[j0:j0+32, 0:j0]^T
template <bool UP, typename E = double>
VB_DEVINL void small_panel_update(double (&acc)[4][4][2], const E* __restrict__ A, int n,
                                  int ld, int r0, int j0, int nb, bool diag, int lane) {
  small_acc_init<UP, E>(acc, A, n, ld, r0, j0, nb, diag, lane);
  small_kloop<UP, E>(acc, A, n, ld, r0, j0, 0, j0, lane);
}

// The TRSM below for the first MT row tiles (compile-time count).
template <bool UP, typename E, int MT>
VB_DEVINL void small_trsm_store_t(SmallSmem& s, double (&acc)[4][4][2], E* __restrict__ A,
                                  int n, int ld, int r0, int j0, int lane, double (*xs)[36]) {
  const int g = lane >> 2, q = lane & 3;
  double x[MT][4][2];
#pragma unroll
  for (int mt = 0; mt < MT; ++mt)
#pragma unroll
    for (int nt = 0; nt < 4; ++nt) x[mt][nt][0] = x[mt][nt][1] = 0.0;
#pragma unroll
  for (int ks = 0; ks < 8; ++ks) {
    double fa[MT], fb[4];
#pragma unroll
    for (int mt = 0; mt < MT; ++mt)
      fa[mt] = cfrag_to_afrag(acc[mt][ks >> 1][0], acc[mt][ks >> 1][1], ks & 1, lane);
#pragma unroll
    for (int nt = 0; nt < 4; ++nt) fb[nt] = s.inv[ks * 4 + q][nt * 8 + g];
#pragma unroll
    for (int mt = 0; mt < MT; ++mt)
#pragma unroll
      for (int nt = 0; nt < 4; ++nt)
        if (4 * ks <= 8 * nt + 7) dmma(x[mt][nt], fa[mt], fb[nt]);
  }
#pragma unroll
  for (int mt = 0; mt < MT; ++mt)
#pragma unroll
    for (int nt = 0; nt < 4; ++nt)
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int row = r0 + mt * 8 + g, col = nt * 8 + 2 * q + h;
        if (row < n) A[gix<UP>(row, j0 + col, ld)] = x[mt][nt][h];
        // optional copy for the next diagonal update, as stored (rounded to E), [col][row]
        if (xs) xs[col][mt * 8 + g] = row < n ? (double)(E)x[mt][nt][h] : 0.0;
      }
}

// X = C inv(L11)^T for a 32 x 32 block in registers (inv[k][n] upper in k,n: zero blocks
// skipped; row tiles entirely below n skipped), then direct stores of rows < n (and, if xs,
// a copy of the stored block in shared memory for the next diagonal update).
template <bool UP, typename E = double>
VB_DEVINL void small_trsm_store(SmallSmem& s, double (&acc)[4][4][2], E* __restrict__ A,
                                int n, int ld, int r0, int j0, int lane,
                                double (*xs)[36] = nullptr) {
  switch (tiles8(n, r0)) {
    case 1: small_trsm_store_t<UP, E, 1>(s, acc, A, n, ld, r0, j0, lane, xs); break;
    case 2: small_trsm_store_t<UP, E, 2>(s, acc, A, n, ld, r0, j0, lane, xs); break;
    case 3: small_trsm_store_t<UP, E, 3>(s, acc, A, n, ld, r0, j0, lane, xs); break;
    case 4: small_trsm_store_t<UP, E, 4>(s, acc, A, n, ld, r0, j0, lane, xs); break;
    default: break;
  }
}

// Variant with the roles split by instruction mix (VB_SMALL=5): the diagonal warp runs only the
// pivot chain (POTF2 + TRTRI of the tile in s.T); the off-diagonal warp does every DMMA update,
// including the next diagonal tile: right after the TRSM of block 1 of panel p (the rows of the
// next diagonal block) it leaves that block in s.T, adds the update by all older columns from
// L2 and by block 1 itself from smem, and hands the tile over. Barriers (64 threads):
// bar0 = inv ready (D -> O), bar0+1 = tile ready (O -> D), bar0+2 = inverse free (O -> D).
template <bool UP, typename E>
VB_DEVINL void la_matrix_v2(SmallSmem& s, int role, int lane, E* __restrict__ A, int n, int ld,
                            int* info_out, int bar0, int bar_lb) {
  const int g = lane >> 2, q = lane & 3;
  const int npan = (n + 31) / 32;
  if (role == 0) {
    bool pending_free = false;
    for (int p = 0; p < npan; ++p) {
      const int j0 = 32 * p, nb = min(32, n - j0);
      const bool below = p + 1 < npan;
      bar_group(bar0 + 1, 64);  // tile of panel p in s.T
      const int info = potf2_block32<UP>(&s.T[0][0], 36, nb, lane, A + (size_t)j0 * ld + j0, ld,
                                         s.wbuf, s.sv, s.tv);
      if (pending_free) {
        bar_group(bar0 + 2, 64);
        pending_free = false;
      }
      if (info) {
        if (lane == 0) {
          s.info = info;
          *info_out = j0 + info;
        }
        if (below) bar_group_arrive(bar0, 64);
        break;
      }
      if (!below) break;
      trtri32_dmma_warp(&s.T[0][0], 36, s.tv, &s.inv[0][0], 36, s.S, LDS_T, lane);
      if (lane == 0) s.info = 0;
      bar_group_arrive(bar0, 64);  // inv(L11) of panel p is ready (s.T is free again)
      pending_free = true;
      // The off-diagonal warp carried every other update and was the pair's bottleneck (ncu: the
      // diagonal warp waited ~37 % of its time for the next tile); the diagonal warp now takes
      // the panel's blocks from the second one below the diagonal on (every block but block 1,
      // whose rows form the next tile), while it would wait anyway: C2 121 -> 117 us with the
      // last block only, -> 113 us with all of them (tools/ab_time.py).
      const int nblk = (n - j0 + 31) / 32;
      if (nblk >= 3) {
        const int b0 = nblk >= 4 ? nblk - 2 : nblk - 1;
        for (int b = b0; b < nblk; ++b) {
          double acc[4][4][2];
          const int r0 = j0 + 32 * b;
          small_panel_update<UP>(acc, A, n, ld, r0, j0, 32, false, lane);
          small_trsm_store<UP>(s, acc, A, n, ld, r0, j0, lane);
        }
        __syncwarp();
        bar_group_arrive(bar_lb, 64);  // last block(s) of panel p stored
      }
    }
  } else {
    {  // tile of panel 0: A's diagonal block as it is
      double acc[4][4][2];
      small_acc_init<UP, E>(acc, A, n, ld, 0, 0, min(32, n), true, lane);
#pragma unroll
      for (int mt = 0; mt < 4; ++mt)
#pragma unroll
        for (int nt = 0; nt < 4; ++nt) {
          s.T[nt * 8 + 2 * q][mt * 8 + g] = acc[mt][nt][0];
          s.T[nt * 8 + 2 * q + 1][mt * 8 + g] = acc[mt][nt][1];
        }
      __syncwarp();
      bar_group_arrive(bar0 + 1, 64);
    }
    for (int p = 0; p + 1 < npan; ++p) {  // panels with blocks below the diagonal
      const int j0 = 32 * p;
      const int nblk = (n - j0 + 31) / 32;
      double acc[4][4][2];
      // panel p-1's last block was the diagonal warp's: its stores precede any read of them here
      if (p > 0 && nblk + 1 >= 3) bar_group(bar_lb, 64);
      small_panel_update<UP>(acc, A, n, ld, j0 + 32, j0, 32, false, lane);
      bar_group(bar0, 64);  // inv(L11) of panel p (or the failure)
      if (s.info) break;
      // block 1 -> global and, as stored, into s.T ([col][row]) for the next tile's update
      small_trsm_store<UP>(s, acc, A, n, ld, j0 + 32, j0, lane, s.T);
      __syncwarp();
      {  // the tile of panel p+1 (rows/cols j0+32..): A - L[., 0:j0] L[., 0:j0]^T - X1 X1^T
        const int j1 = j0 + 32, nb1 = min(32, n - j1);
        small_acc_init<UP, E>(acc, A, n, ld, j1, j1, nb1, true, lane);
        small_kloop<UP, E>(acc, A, n, ld, j1, j1, 0, j0, lane);
        const int mtv1 = tiles8(n, j1);
#pragma unroll
        for (int ks = 0; ks < 8; ++ks) {
          double fa[4], fb[4];
#pragma unroll
          for (int t = 0; t < 4; ++t) {
            fb[t] = s.T[ks * 4 + q][t * 8 + g];
            fa[t] = -fb[t];
          }
#pragma unroll
          for (int mt = 0; mt < 4; ++mt)
#pragma unroll
            for (int nt = 0; nt <= mt; ++nt)
              if (mt < mtv1) dmma(acc[mt][nt], fa[mt], fb[nt]);
        }
        __syncwarp();
#pragma unroll
        for (int mt = 0; mt < 4; ++mt)
#pragma unroll
          for (int nt = 0; nt < 4; ++nt) {
            s.T[nt * 8 + 2 * q][mt * 8 + g] = acc[mt][nt][0];
            s.T[nt * 8 + 2 * q + 1][mt * 8 + g] = acc[mt][nt][1];
          }
        __syncwarp();
        bar_group_arrive(bar0 + 1, 64);  // tile of panel p+1 ready
      }
      const int bend = nblk >= 4 ? nblk - 2 : (nblk >= 3 ? nblk - 1 : nblk);  // diagonal warp's
      for (int b = 2; b < bend; ++b) {
        small_panel_update<UP>(acc, A, n, ld, j0 + 32 * b, j0, 32, false, lane);
        small_trsm_store<UP>(s, acc, A, n, ld, j0 + 32 * b, j0, lane);
      }
      bar_group_arrive(bar0 + 2, 64);  // done with s.inv of panel p
    }
  }
}

// The same pairs packed two per 4-warp CTA with the roles on fixed sub-partitions: warps 0/1 are
// the diagonal warps of pair 0/1, warps 2/3 their off-diagonal warps (warp w runs on SMSP
// w % 4), so the pivot chains share their sub-partitions only with other pivot chains, not
// with the off-diagonal DMMA streams (tools/contention_bench.cu: a DMMA stream starves the
// FP64 chain on its sub-partition). Each pair fetches its own matrices.
template <bool UP, typename E = double>
__global__ void __launch_bounds__(128, VB_SMALL_CPS)
    potrf_small_kernel(const int* __restrict__ d_n, E* const* __restrict__ dA,
                           const int* __restrict__ d_ldda, int* __restrict__ d_info,
                           const Ctrl* __restrict__ ctrl_c, const int* __restrict__ order,
                           int range, int wait_upstream) {
  __shared__ SmallSmem ss[2];
  Ctrl* ctrl = const_cast<Ctrl*>(ctrl_c);
  if (wait_upstream) pdl_wait();
  pdl_launch_dependents();
  const int count = *(volatile const int*)&ctrl->count[range];
  const int start = *(volatile const int*)&ctrl->start[range];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int pair = warp & 1, role = warp >> 1;
  SmallSmem& s = ss[pair];
  const int bar0 = 1 + 4 * pair, tsync = 4 + 4 * pair;
  for (;;) {
    if (role == 0 && lane == 0) s.item = atomicAdd(&ctrl->head[range], 1);
    bar_group(tsync, 64);
    const int it = s.item;
    bar_group(tsync, 64);
    if (it >= count) break;
    const int m = order[start + it];
    TL_BEGIN(t_tl)
    la_matrix_v2<UP, E>(s, role, lane, dA[m], d_n[m], d_ldda[m], d_info + m, bar0, 9 + pair);
    bar_group(tsync, 64);
    if (role == 0 && lane == 0) s.info = 0;
    TL_END(role == 0 && lane == 0, t_tl, m, 22)
  }
  if (!wait_upstream && blockIdx.x == 0 && threadIdx.x == 0) pdl_wait();  // transitive completion (see blocked)
}

// ---------------------------------------------------------------------------------------
constexpr int kWarpsPerCta = 2;
struct WarpSmem {
  double w[kWarpsPerCta][64];
  double sv[kWarpsPerCta][32];
  double tv[kWarpsPerCta][32];
};

// One matrix (n <= NM) by one warp, rows in registers: one HBM read, one HBM write.
template <int NM, bool UP, typename E = double>
VB_DEVINL void potrf_warp_matrix(E* __restrict__ A, int n, int ld, int* info_out, int lane,
                                 double* ws, double* sv, double* tv) {
  double a[NM];
#pragma unroll
  for (int c = 0; c < NM; ++c)
    a[c] = (c < n && lane >= c && lane < n) ? A[gix<UP>(lane, c, ld)] : selp(c == lane, 1.0, 0.0);
  const int info = potf2_regs_warp<NM>(a, n, lane, ws, sv, tv);
  const int ncol = info ? info : n;
#pragma unroll
  for (int c = 0; c < NM; ++c)
    if (c < ncol && lane >= c && lane < n) A[gix<UP>(lane, c, ld)] = a[c];
  if (lane == 0 && info) *info_out = info;
  __syncwarp();
}

// Warp path: one matrix (n <= 32) per warp, whole matrix in registers.
// wait_upstream: 1 when launched directly after the scan (the only factorisation kernel),
// 0 when launched after a blocked kernel (whose CTAs passed the scan's completion before
// releasing this grid, so the scan's outputs are already visible).
template <bool UP, typename E = double>
__global__ void __launch_bounds__(32 * kWarpsPerCta)
    potrf_warp_kernel(const int* __restrict__ d_n, E* const* __restrict__ dA,
                      const int* __restrict__ d_ldda, int* __restrict__ d_info,
                      const Ctrl* __restrict__ ctrl_c, const int* __restrict__ order,
                      int wait_upstream) {
  __shared__ WarpSmem s;
  Ctrl* ctrl = const_cast<Ctrl*>(ctrl_c);
  if (wait_upstream) pdl_wait();
  const int start = *(volatile const int*)&ctrl->start[2];
  const int count = *(volatile const int*)&ctrl->count[2];
  const int lane = threadIdx.x & 31, wi = threadIdx.x >> 5;
  for (;;) {
    int w = 0;
    if (lane == 0) w = atomicAdd(&ctrl->head[2], 1);
    w = __shfl_sync(kFull, w, 0);
    if (w >= count) break;
    const int m = order[start + w];
    const int n = d_n[m], ld = d_ldda[m];
    TL_BEGIN(t_tl)
    if (n <= 8)
      potrf_warp_matrix<8, UP, E>(dA[m], n, ld, d_info + m, lane, s.w[wi], s.sv[wi], s.tv[wi]);
    else if (n <= 16)
      potrf_warp_matrix<16, UP, E>(dA[m], n, ld, d_info + m, lane, s.w[wi], s.sv[wi], s.tv[wi]);
    else
      potrf_warp_matrix<32, UP, E>(dA[m], n, ld, d_info + m, lane, s.w[wi], s.sv[wi], s.tv[wi]);
    TL_END(lane == 0, t_tl, m, 40)
  }
  if (!wait_upstream && blockIdx.x == 0 && threadIdx.x == 0) pdl_wait();  // transitive completion (see blocked)
}

// Direct warp path for batches whose max_n <= 32 (no scan, no sort: with every matrix this
// small there is nothing to balance): warp w validates (info -2/-4/-7, as the scan would) and
// factors matrices w, w + nwarps, ... One launch per call — the latency path for C1.
template <bool UP, typename E = double>
__global__ void __launch_bounds__(32 * kWarpsPerCta)
    potrf_warp_direct_kernel(const int* __restrict__ d_n, E* const* __restrict__ dA,
                             const int* __restrict__ d_ldda, int* __restrict__ d_info, int batch,
                             int max_n) {
  __shared__ WarpSmem s;
  const int lane = threadIdx.x & 31, wi = threadIdx.x >> 5;
  const int nw = gridDim.x * kWarpsPerCta;
  for (int m = blockIdx.x * kWarpsPerCta + wi; m < batch; m += nw) {
    const int n = d_n[m], ld = d_ldda[m];
    int code = 0;
    if (n < 0) code = -2;
    else if (ld < (n > 1 ? n : 1)) code = -4;
    else if (n > max_n) code = -7;
    if (lane == 0) d_info[m] = code;
    if (code != 0 || n == 0) continue;
    if (n <= 8)
      potrf_warp_matrix<8, UP, E>(dA[m], n, ld, d_info + m, lane, s.w[wi], s.sv[wi], s.tv[wi]);
    else if (n <= 16)
      potrf_warp_matrix<16, UP, E>(dA[m], n, ld, d_info + m, lane, s.w[wi], s.sv[wi], s.tv[wi]);
    else
      potrf_warp_matrix<32, UP, E>(dA[m], n, ld, d_info + m, lane, s.w[wi], s.sv[wi], s.tv[wi]);
  }
}

// ---------------------------------------------------------------------------------------
// Host-side state. The size threshold is read once per process (std::call_once); the kernel
// attributes (dynamic shared memory limits) are set once per device (bit per ordinal, under a
// mutex); occupancies and the SM count are those of the first device initialised (the pool's
// GPUs are identical B200s) and are published through atomics.
static std::atomic<int> g_num_sms{0};
static std::atomic<int> g_occ64{0}, g_occ64s{0};
static int g_ts = 128;
static std::once_flag g_ts_once;

// Size threshold: n > ts takes the blocked NB=64 kernel, 32 < n <= ts the small-matrix kernel
// (env VB_TS; default 128, measured: the blocked kernel beats the small kernel above 128 and
// loses below, tools/cfgtime.py sweeps in profiles/r01).
int potrf_ts() {
  std::call_once(g_ts_once, [] {
    const char* e = getenv("VB_TS");
    int t = e ? atoi(e) : 128;
    g_ts = t < kWarpMaxN ? kWarpMaxN : t;
  });
  return g_ts;
}

template <class C>
static cudaError_t setup_blocked(std::atomic<int>* occ_out) {
  cudaError_t e = cudaFuncSetAttribute(potrf_blocked3_kernel<C, false>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)sizeof(Smem2<C>));
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(potrf_blocked3_kernel<C, true>,
                           cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(Smem2<C>));
  if (e != cudaSuccess) return e;
  int occ = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, potrf_blocked3_kernel<C, false>,
                                                    32 * (C::WARPS + 1), sizeof(Smem2<C>));
  occ_out->store(occ < 1 ? 1 : occ);
  return e;
}

static unsigned long long g_dev_ready = 0;
static std::mutex g_init_mu;

static cudaError_t init_device_info() {
  int dev;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (dev < 0 || dev >= 64) return cudaErrorInvalidDevice;
  const unsigned long long bit = 1ull << dev;
  std::lock_guard<std::mutex> lock(g_init_mu);
  if (g_dev_ready & bit) return cudaSuccess;
  int sms = 0;
  e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (e != cudaSuccess) return e;
  if ((e = setup_blocked<Cfg64d>(&g_occ64)) != cudaSuccess) return e;
  if ((e = setup_blocked<Cfg64s>(&g_occ64s)) != cudaSuccess) return e;
  potrf_ts();
  g_num_sms.store(sms);
  g_dev_ready |= bit;
  return cudaSuccess;
}

template <typename E>
struct BlockedCfgOf;
template <>
struct BlockedCfgOf<double> {
  using C = Cfg64d;
};
template <>
struct BlockedCfgOf<float> {
  using C = Cfg64s;
};

// One persistent grid per non-empty size range, chained with programmatic dependent launch
// (each grid releases the next as soon as it starts, so the next range's CTAs take the SMs
// the previous kernel frees at its tail). E = storage type (double: DPOTRF, float: SPOTRF; the
// arithmetic is FP64 in both).
template <typename E>
static cudaError_t launch_paths(const int* d_n, E* const* dA, const int* d_ldda, int* d_info,
                                int batch, int max_n_hint, const Ctrl* ctrl, const int* order,
                                bool up, cudaStream_t stream) {
  using C = typename BlockedCfgOf<E>::C;
  cudaError_t e = init_device_info();
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg = {};
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  cfg.stream = stream;
  int wait = 1;  // the first factorisation kernel after the scan waits for it
  if (max_n_hint > potrf_ts()) {
    const int occ = sizeof(E) == 8 ? g_occ64.load() : g_occ64s.load();
    cfg.blockDim = dim3(32 * (C::WARPS + 1));
    cfg.gridDim = dim3(std::max(1, std::min(batch, g_num_sms.load() * occ)));
    cfg.dynamicSmemBytes = sizeof(Smem2<C>);
    e = cudaLaunchKernelEx(&cfg, up ? potrf_blocked3_kernel<C, true> : potrf_blocked3_kernel<C, false>,
                           d_n, dA, d_ldda, d_info, ctrl, order, 0, wait);
    if (e != cudaSuccess) return e;
    wait = 0;
  }
  const int sms = g_num_sms.load();
  if (max_n_hint > kWarpMaxN) {
    cfg.blockDim = dim3(128);
    cfg.gridDim = dim3(std::max(1, std::min((batch + 1) / 2, sms * VB_SMALL_CPS)));
    cfg.dynamicSmemBytes = 0;
    e = cudaLaunchKernelEx(&cfg, up ? potrf_small_kernel<true, E> : potrf_small_kernel<false, E>,
                           d_n, dA, d_ldda, d_info, ctrl, order, 1, wait);
    if (e != cudaSuccess) return e;
    wait = 0;
  }
  const int warps = std::max(1, batch);
  cfg.blockDim = dim3(32 * kWarpsPerCta);
  cfg.gridDim = dim3(std::max(1, std::min((warps + kWarpsPerCta - 1) / kWarpsPerCta, sms * 8)));
  cfg.dynamicSmemBytes = 0;
  return cudaLaunchKernelEx(&cfg, up ? potrf_warp_kernel<true, E> : potrf_warp_kernel<false, E>,
                            d_n, dA, d_ldda, d_info, ctrl, order, wait);
}

cudaError_t launch_potrf_paths(const int* d_n, double* const* dA, const int* d_ldda, int* d_info,
                               int batch, int max_n_hint, const Ctrl* ctrl, const int* order,
                               bool up, cudaStream_t stream) {
  return launch_paths<double>(d_n, dA, d_ldda, d_info, batch, max_n_hint, ctrl, order, up, stream);
}
cudaError_t launch_potrf_paths(const int* d_n, float* const* dA, const int* d_ldda, int* d_info,
                               int batch, int max_n_hint, const Ctrl* ctrl, const int* order,
                               bool up, cudaStream_t stream) {
  return launch_paths<float>(d_n, dA, d_ldda, d_info, batch, max_n_hint, ctrl, order, up, stream);
}

void potrf_occupancy(int* out4) {
  init_device_info();
  out4[0] = g_occ64.load();
  out4[1] = Cfg64d::WARPS;
  out4[2] = 0;  // (no separate NB=32 range)
  out4[3] = VB_SMALL_CPS;  // small kernel: CTAs (2 matrices each) per SM
}

int potrf_num_launches(int max_n_hint) {
  init_device_info();
  if (max_n_hint <= kWarpMaxN) return 1;  // direct warp kernel only
  return 3 + (max_n_hint > potrf_ts() ? 1 : 0);
}

const char* potrf_kernel_names(int max_n_hint) {
  if (max_n_hint <= 0) return "";
  if (max_n_hint <= kWarpMaxN) return "potrf_warp_direct_kernel";
  if (max_n_hint <= potrf_ts()) return "potrf_small_kernel + potrf_warp_kernel";
  return "potrf_blocked3_kernel + potrf_small_kernel + potrf_warp_kernel";
}

template <typename E>
static cudaError_t launch_direct(const int* d_n, E* const* dA, const int* d_ldda, int* d_info,
                                 int batch, int max_n, bool up, cudaStream_t stream) {
  cudaError_t e = init_device_info();
  if (e != cudaSuccess) return e;
  const int grid = std::max(1, std::min((batch + kWarpsPerCta - 1) / kWarpsPerCta, g_num_sms.load() * 16));
  if (up)
    potrf_warp_direct_kernel<true, E><<<grid, 32 * kWarpsPerCta, 0, stream>>>(d_n, dA, d_ldda,
                                                                             d_info, batch, max_n);
  else
    potrf_warp_direct_kernel<false, E><<<grid, 32 * kWarpsPerCta, 0, stream>>>(d_n, dA, d_ldda,
                                                                              d_info, batch, max_n);
  return cudaGetLastError();
}
cudaError_t launch_potrf_direct(const int* d_n, double* const* dA, const int* d_ldda, int* d_info,
                                int batch, int max_n, bool up, cudaStream_t stream) {
  return launch_direct<double>(d_n, dA, d_ldda, d_info, batch, max_n, up, stream);
}
cudaError_t launch_potrf_direct(const int* d_n, float* const* dA, const int* d_ldda, int* d_info,
                                int batch, int max_n, bool up, cudaStream_t stream) {
  return launch_direct<float>(d_n, dA, d_ldda, d_info, batch, max_n, up, stream);
}

}  // namespace vb

#ifdef VB_CHUNK_LAT
extern "C" int vbatched_debug_chunk_lat(unsigned long long* dptr) {
  return (int)cudaMemcpyToSymbol(vb::g_lat, &dptr, sizeof(dptr));
}
#endif

#ifdef VB_TIMELINE
extern "C" int vbatched_debug_timeline(unsigned long long* dptr) {
  return (int)cudaMemcpyToSymbol(vb::g_tl, &dptr, sizeof(dptr));
}
#endif

#ifdef VB_PHASE_PROF
extern "C" int vbatched_debug_phases(unsigned long long* out, int reset) {
  cudaError_t e = cudaMemcpyFromSymbol(out, vb::g_phase, sizeof(unsigned long long) * 8);
  if (reset) {
    unsigned long long z[8] = {};
    cudaMemcpyToSymbol(vb::g_phase, z, sizeof z);
  }
  return (int)e;
}
#endif
