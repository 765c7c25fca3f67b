// quad_experiment.cuh (tool, NOT product code): the "quad" small-matrix kernel measured and
// rejected in round 2 (one matrix per 4-warp CTA: a pivot-chain warp on SMSP 0 chosen from
// %warpid + three DMMA warps on 16-row strips). Correct (GPU parity green when it was the
// default), but slower than the paired kernel: C2 173-187 us vs 122 us — per-matrix latency
// stayed ~80 us at n = 128 (chain-bound: POTF2 17 K cycles in situ) while only 4 matrices per SM
// were in flight instead of 8. Kept for the benchmarks that reuse its strip k-loop.
// Include after paper_conf_ipps_abdelfattahhtd16_b200/csrc/potrf.cu.
#pragma once
namespace vb {
// =======================================================================================
// Quad small-matrix kernel (32 < n <= ts): one matrix per 4-warp CTA, 4 CTAs per SM.
//   warp 0 (sub-partition 0): the pivot chain only — POTF2 of the 32x32 diagonal tile and its
//     inverse (TRTRI). Every CTA's warp 0 sits on SMSP 0, so no DMMA stream shares its FP64
//     pipe (a DMMA-streaming warp on the same SMSP slows a DFMA chain ~50x, none elsewhere:
//     tools/pipe_share_bench.cu).
//   warps 1..3 (SMSPs 1..3): all DMMA work, on 16-row strips. Strip s = rows 16s..16s+15 is
//     owned by warp 1 + s % 3 for the whole factorisation, so a strip's own earlier columns are
//     always the owner's own stores.
// Left-looking, NB = 32 (the paper's fused kernel: panel update / factorize / trsm,
// PAPER.md:532-560). Panel p (columns j0 = 32p..j0+31) with rows below (j1 = j0 + 32 < n):
//   chain   : T(p) -> POTF2 -> L11 stored; TRTRI -> inv[p&1]; arrive INV(p).
//   strips  : s >= 2p+2: acc = A[rows, j0:j0+32] - L[rows, 0:j0] L[j0:j0+32, 0:j0]^T (k-loop:
//             columns < j0-32 from L2, overlapped with the chain; the newest 32 columns with the
//             B operand from xs[(p-1)&1] in shared memory), sync INV(p), TRSM X = acc inv^T,
//             store; the two block-1 strips (2p+2, 2p+3: the rows of the next diagonal tile) also
//             keep X in xs[p&1].
//   tile    : right after its block-1 strip, the owner of strip 2p+2 builds rows 0..15 of
//             T(p+1) (SYRK over its own rows only: columns < j0 from L2, panel p from xs), the
//             owner of strip 2p+3 rows 16..31 (after PAIR(p): strip 2p+2's xs rows are there);
//             both arrive TILE(p+1), which the chain syncs on.
// Named barriers: 1 INV (128: chain arrives, DMMA warps sync), 2 TILE (chain + the tile
// builders: 64 or 96), 3 PAIR (64), 4 matrix end (128). Panel p-2's inverse and block-1 rows
// are dead before panel p rewrites them (double buffers; ordering through INV(p-1) and
// TILE(p)). A failed pivot: the chain publishes info before INV(p); every DMMA warp checks it
// right after INV(p), before any other barrier of the panel, and all four meet at the end.
struct QuadSmem {
  double T[32][36];       // diagonal tile T[c][r]
  double inv[2][32][36];  // inv(L11) of panel p in inv[p&1]: inv[k][n] = X[n][k]
  double xs[2][32][36];   // block-1 rows of panel p (stored values) in xs[p&1]: xs[col][row]
  double S[16 * LDS_T];
  double wbuf[64];
  double sv[32];
  double tv[32];
  int item;
  int info;
};

// acc[mt][nt] (rows r0 + 8mt + g, cols c0 + 8nt + 2q + h) = A for rows < n, cols < c0 + ncols
// (lower part only when TRI), 0 elsewhere.
template <bool UP, typename E>
VB_DEVINL void strip_init(double (&acc)[2][4][2], const E* __restrict__ A, int n, int ld, int r0,
                          int c0, int ncols, bool tri, int lane) {
  const int g = lane >> 2, q = lane & 3;
#pragma unroll
  for (int mt = 0; mt < 2; ++mt)
#pragma unroll
    for (int nt = 0; nt < 4; ++nt)
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int row = r0 + mt * 8 + g, col = c0 + nt * 8 + 2 * q + h;
        const bool v = row < n && col < c0 + ncols && (!tri || row >= col);
        acc[mt][nt][h] = v ? (double)__ldcg(A + gix<UP>(row, col, ld)) : 0.0;
      }
}

// acc -= L[r0.., kb:ke] L[c0.., kb:ke]^T from L2 for the first MT row tiles, NT column tiles,
// and (DOFF >= 0) only tiles with nt <= mt + DOFF (the rest lie above the diagonal).
template <bool UP, typename E, int MT, int NT, int DOFF>
VB_DEVINL void strip_kloop_t(double (&acc)[2][4][2], const E* __restrict__ A, int n, int ld,
                             int r0, int c0, int kb, int ke, int lane) {
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
    cv[t] = c0 + t * 8 + g < n;
    pb[t] = A + gix<UP>(cv[t] ? c0 + t * 8 + g : 0, 0, ld);
  }
  const size_t ks = UP ? 1 : (size_t)ld;
#pragma unroll 4
  for (int k = kb + q; k < ke; k += 4) {
    double fa[MT], fb[NT];
#pragma unroll
    for (int t = 0; t < MT; ++t) fa[t] = rv[t] ? -(double)__ldcg(pa[t] + k * ks) : 0.0;
#pragma unroll
    for (int t = 0; t < NT; ++t) fb[t] = cv[t] ? (double)__ldcg(pb[t] + k * ks) : 0.0;
#pragma unroll
    for (int mt = 0; mt < MT; ++mt)
#pragma unroll
      for (int nt = 0; nt < NT; ++nt)
        if (DOFF < 0 || nt <= mt + DOFF) dmma(acc[mt][nt], fa[mt], fb[nt]);
  }
}

// The same for a 32-column k range whose B operand (rows c0.., these 32 columns) is in shared
// memory: bs[k][row] (row relative to the buffer), A operand from L2 (a_smem == nullptr) or
// from shared memory too (as[k][row]).
template <bool UP, typename E, int MT, int NT, int DOFF>
VB_DEVINL void strip_kloop_smem_t(double (&acc)[2][4][2], const E* __restrict__ A, int n, int ld,
                                  int r0, int kb, const double (*as)[36], int arow0,
                                  const double (*bs)[36], int brow0, int lane) {
  const int g = lane >> 2, q = lane & 3;
  const E* pa[MT];
  bool rv[MT];
#pragma unroll
  for (int t = 0; t < MT; ++t) {
    rv[t] = r0 + t * 8 + g < n;
    pa[t] = A + gix<UP>(rv[t] ? r0 + t * 8 + g : 0, 0, ld);
  }
  const size_t ks = UP ? 1 : (size_t)ld;
#pragma unroll
  for (int kk = 0; kk < 8; ++kk) {
    const int k = kk * 4 + q;
    double fa[MT], fb[NT];
#pragma unroll
    for (int t = 0; t < MT; ++t)
      fa[t] = as ? -as[k][arow0 + t * 8 + g]
                 : (rv[t] ? -(double)__ldcg(pa[t] + (kb + k) * ks) : 0.0);
#pragma unroll
    for (int t = 0; t < NT; ++t) fb[t] = bs[k][brow0 + t * 8 + g];
#pragma unroll
    for (int mt = 0; mt < MT; ++mt)
#pragma unroll
      for (int nt = 0; nt < NT; ++nt)
        if (DOFF < 0 || nt <= mt + DOFF) dmma(acc[mt][nt], fa[mt], fb[nt]);
  }
}

// X = acc inv^T (16 rows x 32 columns, inv upper in (k, n): zero 8x8 blocks skipped) for the
// first MT row tiles; rows < n stored to global at column block j0; if xs, the stored values
// also go to xs[col][xrow0 + row] (zeros for rows >= n).
template <bool UP, typename E, int MT>
VB_DEVINL void strip_trsm_store_t(const double (*inv)[36], double (&acc)[2][4][2],
                                  E* __restrict__ A, int n, int ld, int r0, int j0, int lane,
                                  double (*xs)[36], int xrow0) {
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
    for (int nt = 0; nt < 4; ++nt) fb[nt] = inv[ks * 4 + q][nt * 8 + g];
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
        if (row < n) A[gix<UP>(row, j0 + col, ld)] = (E)x[mt][nt][h];
        if (xs) xs[col][xrow0 + mt * 8 + g] = row < n ? (double)(E)x[mt][nt][h] : 0.0;
      }
  if (MT < 2 && xs) {  // the strip's second row tile lies beyond n: zeros for the tile builders
#pragma unroll
    for (int nt = 0; nt < 4; ++nt)
#pragma unroll
      for (int h = 0; h < 2; ++h) xs[nt * 8 + 2 * q + h][xrow0 + 8 + g] = 0.0;
  }
}

// Dispatchers on the number of 8-row tiles of the strip at r0 that hold rows < n (1 or 2).
VB_DEVINL int strip_tiles(int n, int r0) { return (n - r0) > 8 ? 2 : 1; }

template <bool UP, typename E>
VB_DEVINL void strip_kloop(double (&acc)[2][4][2], const E* __restrict__ A, int n, int ld, int r0,
                           int c0, int kb, int ke, int lane) {
  if (ke <= kb) return;
  if (strip_tiles(n, r0) == 2)
    strip_kloop_t<UP, E, 2, 4, -1>(acc, A, n, ld, r0, c0, kb, ke, lane);
  else
    strip_kloop_t<UP, E, 1, 4, -1>(acc, A, n, ld, r0, c0, kb, ke, lane);
}

template <bool UP, typename E>
VB_DEVINL void strip_trsm_store(const double (*inv)[36], double (&acc)[2][4][2], E* __restrict__ A,
                                int n, int ld, int r0, int j0, int lane, double (*xs)[36],
                                int xrow0) {
  if (strip_tiles(n, r0) == 2)
    strip_trsm_store_t<UP, E, 2>(inv, acc, A, n, ld, r0, j0, lane, xs, xrow0);
  else
    strip_trsm_store_t<UP, E, 1>(inv, acc, A, n, ld, r0, j0, lane, xs, xrow0);
}

// Write the computed tiles of a tile-builder's accumulator into T (rows trow0 + .., T[c][r]).
template <int MT, int NT, int DOFF>
VB_DEVINL void tile_put(double (*T)[36], const double (&acc)[2][4][2], int trow0, int lane) {
  const int g = lane >> 2, q = lane & 3;
#pragma unroll
  for (int mt = 0; mt < MT; ++mt)
#pragma unroll
    for (int nt = 0; nt < NT; ++nt)
      if (nt <= mt + DOFF) {
        T[nt * 8 + 2 * q][trow0 + mt * 8 + g] = acc[mt][nt][0];
        T[nt * 8 + 2 * q + 1][trow0 + mt * 8 + g] = acc[mt][nt][1];
      }
}

template <bool UP, typename E>
VB_DEVINL void quad_matrix(QuadSmem& s, int warp, int lane, E* __restrict__ A, int n, int ld,
                           int* info_out) {
  constexpr int kInv = 1, kTile = 2, kPair = 3;
  const int npan = (n + 31) / 32;
  const int nstrip = (n + 15) / 16;
  if (warp == 0) {  // ---------------- the pivot chain
    const int g = lane >> 2, q = lane & 3;
    for (int p = 0; p < npan; ++p) {
      const int j0 = 32 * p, nb = min(32, n - j0);
      const bool below = j0 + 32 < n;
      if (p == 0) {
#pragma unroll
        for (int mt = 0; mt < 4; ++mt)
#pragma unroll
          for (int nt = 0; nt < 4; ++nt)
#pragma unroll
            for (int h = 0; h < 2; ++h) {
              const int r = mt * 8 + g, c = nt * 8 + 2 * q + h;
              s.T[c][r] = (r < nb && c <= r) ? (double)__ldcg(A + gix<UP>(r, c, ld)) : 0.0;
            }
        __syncwarp();
      } else {
        const bool two = (j0 + 16 < n);  // tile p was built by two strips' owners
        VB_T0(t_w)
        bar_group(kTile, two ? 96 : 64);
        VB_ADDW(0, t_w)
      }
      VB_T0(t_p)
      const int info = potf2_block32<UP>(&s.T[0][0], 36, nb, lane, A + (size_t)j0 * ld + j0, ld,
                                         s.wbuf, s.sv, s.tv);
      VB_ADDW(1, t_p)
      if (info) {
        if (lane == 0) {
          s.info = info;
          *info_out = j0 + info;
        }
        if (below) bar_group_arrive(kInv, 128);
        break;
      }
      if (!below) break;
      VB_T0(t_i)
      trtri32_dmma_warp(&s.T[0][0], 36, s.tv, &s.inv[p & 1][0][0], 36, s.S, LDS_T, lane);
      VB_ADDW(2, t_i)
      bar_group_arrive(kInv, 128);  // inv(L11) of panel p is ready
    }
    return;
  }
  // ---------------- DMMA warps 1..3
  for (int p = 0; p + 1 < npan; ++p) {
    const int j0 = 32 * p, j1 = j0 + 32;
    const int sa = 2 * p + 2, sb = 2 * p + 3;   // the block-1 strips (rows of tile p+1)
    const bool has_b = sb < nstrip;
    const double(*inv)[36] = s.inv[p & 1];
    double(*xs)[36] = s.xs[p & 1];
    const double(*xprev)[36] = s.xs[(p + 1) & 1];  // block-1 rows of panel p-1 = L[j0.., j0-32:j0]
    int first = sa + ((warp - 1 - sa % 3) + 3) % 3;  // my first strip of this panel
    double acc[2][4][2];
    VB_T0(t_pre)
    if (first < nstrip) {  // pre-accumulate my first strip's old columns while the chain runs
      strip_init<UP, E>(acc, A, n, ld, 16 * first, j0, 32, false, lane);
      strip_kloop<UP, E>(acc, A, n, ld, 16 * first, j0, 0, j0 - 32, lane);
    }
    VB_ADDW(3, t_pre)
    VB_T0(t_inv)
    bar_group(kInv, 128);
    VB_ADDW(4, t_inv)
    if (s.info) return;
    for (int st = first; st < nstrip; st += 3) {
      VB_T0(t_st)
      const int r0 = 16 * st;
      if (st != first) {
        strip_init<UP, E>(acc, A, n, ld, r0, j0, 32, false, lane);
        strip_kloop<UP, E>(acc, A, n, ld, r0, j0, 0, j0 - 32, lane);
      }
      if (p > 0) {  // the newest 32 columns: B rows j0..j0+31 from xs of panel p-1
        if (strip_tiles(n, r0) == 2)
          strip_kloop_smem_t<UP, E, 2, 4, -1>(acc, A, n, ld, r0, j0 - 32, nullptr, 0, xprev, 0, lane);
        else
          strip_kloop_smem_t<UP, E, 1, 4, -1>(acc, A, n, ld, r0, j0 - 32, nullptr, 0, xprev, 0, lane);
      }
      const bool blk1 = (st == sa || st == sb);
      strip_trsm_store<UP, E>(inv, acc, A, n, ld, r0, j0, lane, blk1 ? xs : nullptr,
                              16 * (st - sa));
      __syncwarp();
      VB_ADDW(5, t_st)
      VB_T0(t_tb)
      if (st == sa) {  // rows 0..15 of tile p+1: own rows only
        if (has_b) bar_group_arrive(kPair, 64);
        double t[2][4][2];
        strip_init<UP, E>(t, A, n, ld, j1, j1, 16, true, lane);
        if (strip_tiles(n, j1) == 2) {
          strip_kloop_t<UP, E, 2, 2, 0>(t, A, n, ld, j1, j1, 0, j0, lane);
          strip_kloop_smem_t<UP, E, 2, 2, 0>(t, A, n, ld, j1, 0, xs, 0, xs, 0, lane);
          tile_put<2, 2, 0>(s.T, t, 0, lane);
        } else {
          strip_kloop_t<UP, E, 1, 1, 0>(t, A, n, ld, j1, j1, 0, j0, lane);
          strip_kloop_smem_t<UP, E, 1, 1, 0>(t, A, n, ld, j1, 0, xs, 0, xs, 0, lane);
          tile_put<1, 1, 0>(s.T, t, 0, lane);
        }
        __syncwarp();
        bar_group_arrive(kTile, has_b ? 96 : 64);
      } else if (st == sb) {  // rows 16..31 of tile p+1 (columns 0..31)
        double t[2][4][2];
        strip_init<UP, E>(t, A, n, ld, j1 + 16, j1, 32, true, lane);
        const int mt2 = strip_tiles(n, j1 + 16);
        if (mt2 == 2)
          strip_kloop_t<UP, E, 2, 4, 2>(t, A, n, ld, j1 + 16, j1, 0, j0, lane);
        else
          strip_kloop_t<UP, E, 1, 3, 2>(t, A, n, ld, j1 + 16, j1, 0, j0, lane);
        bar_group(kPair, 64);  // xs rows 0..15 (strip sa) written
        if (mt2 == 2) {
          strip_kloop_smem_t<UP, E, 2, 4, 2>(t, A, n, ld, j1 + 16, 0, xs, 16, xs, 0, lane);
          tile_put<2, 4, 2>(s.T, t, 16, lane);
        } else {
          strip_kloop_smem_t<UP, E, 1, 3, 2>(t, A, n, ld, j1 + 16, 0, xs, 16, xs, 0, lane);
          tile_put<1, 3, 2>(s.T, t, 16, lane);
        }
        __syncwarp();
        bar_group_arrive(kTile, 96);
      }
      VB_ADDW(6, t_tb)
    }
  }
}

template <bool UP, typename E = double>
__global__ void __launch_bounds__(128, 4)
    potrf_quad_kernel(const int* __restrict__ d_n, E* const* __restrict__ dA,
                      const int* __restrict__ d_ldda, int* __restrict__ d_info,
                      const Ctrl* __restrict__ ctrl_c, const int* __restrict__ order, int range,
                      int wait_upstream) {
  extern __shared__ __align__(16) unsigned char smem_quad[];  // QuadSmem (49.5 KB: dynamic)
  QuadSmem& s = *reinterpret_cast<QuadSmem*>(smem_quad);
  Ctrl* ctrl = const_cast<Ctrl*>(ctrl_c);
  if (wait_upstream) pdl_wait();
  pdl_launch_dependents();
  const int count = *(volatile const int*)&ctrl->count[range];
  const int start = *(volatile const int*)&ctrl->start[range];
  // Roles by sub-partition, not by warp index: the k-th CTA resident on an SM gets hardware warp
  // slots 4k + (w + k) % 4 (tools/warpid_probe.cu), so warp w runs on SMSP (w + k) % 4 and a
  // fixed warp index would put the chain warps of different CTAs on different SMSPs, beside
  // other CTAs' DMMA streams. The four warps of a CTA always occupy four distinct SMSPs; the one
  // on SMSP 0 takes the pivot chain (role 0), the others the DMMA roles 1..3 (their SMSP).
  unsigned wslot;
  asm volatile("mov.u32 %0, %%warpid;" : "=r"(wslot));
  const int lane = threadIdx.x & 31, warp = (int)(wslot & 3);
  if (threadIdx.x == 0) s.info = 0;
  for (;;) {
    if (threadIdx.x == 0) s.item = atomicAdd(&ctrl->head[range], 1);
    __syncthreads();
    const int it = s.item;
    __syncthreads();
    if (it >= count) break;
    const int m = order[start + it];
    TL_BEGIN(t_tl)
    VB_T0(t_mat)
    quad_matrix<UP, E>(s, warp, lane, dA[m], d_n[m], d_ldda[m], d_info + m);
    VB_ADDW(7, t_mat)
    __syncthreads();
    if (threadIdx.x == 0) s.info = 0;
    TL_END(threadIdx.x == 0, t_tl, m, 23)
  }
  if (!wait_upstream && threadIdx.x == 0) pdl_wait();  // transitive completion (see blocked)
}

}  // namespace vb
