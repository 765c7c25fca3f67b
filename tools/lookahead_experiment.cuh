// lookahead_experiment.cuh (tool, NOT product code): the look-ahead blocked kernel measured and
// rejected in round 2 — a dedicated diagonal warp factors panel p+1's 64x64 block while six
// consumer warps (96-row blocks) finish panel p, 2 CTAs per SM. Slower than the 3-CTA/SM
// potrf_blocked3_kernel (C3 2.53 vs 2.27 ms, C5 177 vs 154 ms) and it hung on one of the
// failure tests (protocol not finished). Kept as a record; include after csrc/potrf.cu.
#pragma once
namespace vb {
// =======================================================================================
// Look-ahead blocked kernel (n > ts): the diagonal factorisation of panel p+1 runs on a warp of
// its own while the consumer warps finish panel p (the "pipelined stages" of PAPER.md:583-589
// applied to the panel factorisation). 8 warps per CTA, 2 CTAs per SM:
//   warps 0-5  consumers: 96-row blocks x 64 columns (16 rows each), DMMA from the TMA ring;
//   warp 6     TMA producer (as in potrf_blocked3_kernel);
//   warp 7     diagonal warp D: POTF2 / TRTRI / L21 / SYRK / POTF2 / TRTRI of each 64x64 tile.
// Per panel p (columns j0 = 64p.., j1 = j0 + 64):
//   R1(p)     rows j1..j1+95: k-loop over columns < j0; wait INV(p); copy D's operands out of
//             the tile; TRSM; store; arrive R1_DONE(p).
//   TILE(p+1) rows / columns j1..j1+63 (warps 0-3): SYRK k-loop over columns < j1 (the newest
//             64 = R1(p) just stored); written to the tile; arrive TILE_READY: D factors it while
//   R2..(p)   the remaining 96-row blocks of panel p run (k-loop, TRSM, store); PANEL_DONE(p).
// D stores L of each diagonal block itself and never touches the consumers' operand copy.
// Failure: D publishes info with INV(t); the producer waits INV(p) before issuing anything past
// R1(p) and every consumer checks right after INV(p), so nobody issues or expects chunks beyond
// the failing panel (no drain).
template <class C>
struct SmemLA : Smem2<C> {
  double cinv11[32][36];  // operands of panel p's row-block TRSM (copied from T after INV(p))
  double cl21[32][36];
  double cinv22[32][36];
  uint64_t inv_ready;   // D -> all: tile t factored (1 arrival)
  uint64_t tile_ready;  // consumers 0-3 -> D: tile written (4 arrivals)
  uint64_t r1_done;     // consumers -> producer: R1(p) stored (6 arrivals)
  int info_la;          // D's failure (global 1-based column), 0 otherwise
};
using CfgLAd = Cfg2<64, 16, 2, 2, 6>;
using CfgLAs = Cfg2<64, 16, 2, 2, 6, float>;

// The whole 64x64 diagonal block by one warp (diag_block64v2's steps, sequential): L11 =
// potf2(C11) -> inv(L11) in the T12 slot -> L21 = C21 inv(L11)^T -> C22 -= L21 L21^T -> L22 =
// potf2(C22) -> inv(L22) in the T11 slot. L11 / L21 / L22 (rows < nb) stored to (Ad, ld).
template <class CC, bool UP>
__device__ __noinline__ int diag64_one_warp(Smem2<CC>& s, int nb, int lane, typename CC::E* Ad,
                                            int ld, bool below) {
  constexpr int LDT = CC::LDT;
  double* T = &s.T[0][0];
  double* INV11 = T + 32 * LDT;
  const int g = lane >> 2, q = lane & 3;
  const int nb1 = min(nb, 32), nb2 = nb - nb1;
  int info = potf2_block32<UP>(T, LDT, nb1, lane, Ad, ld, s.wbuf, s.sv, s.tv);
  if (info || nb2 == 0) return info;
  trtri32_dmma_warp(T, LDT, s.tv, INV11, LDT, s.S, LDS_T, lane);
  // L21 = C21 inv(L11)^T, one 16-row half at a time (both column quarters read the half's C21
  // rows before they are overwritten)
#pragma unroll 1
  for (int m0 = 0; m0 < 32; m0 += 16) {
    double acc[2][2][2][2] = {};
#pragma unroll
    for (int h = 0; h < 2; ++h)
      mm32_quarter(acc[h], (m0 >> 3) | h, lane, [&](int m, int k) { return T[k * LDT + 32 + m]; },
                   [&](int k, int n) { return INV11[k * LDT + n]; });
    __syncwarp();
#pragma unroll
    for (int h = 0; h < 2; ++h)
#pragma unroll
      for (int mt = 0; mt < 2; ++mt)
#pragma unroll
        for (int nt = 0; nt < 2; ++nt)
#pragma unroll
          for (int e = 0; e < 2; ++e) {
            const int r = 32 + m0 + mt * 8 + g, c = h * 16 + nt * 8 + 2 * q + e;
            T[c * LDT + r] = acc[h][mt][nt][e];
            if (r < nb) Ad[gix<UP>(r, c, ld)] = acc[h][mt][nt][e];
          }
    __syncwarp();
  }
  // C22 -= L21 L21^T: the three lower 16x16 quarters
#pragma unroll 1
  for (int wq = 0; wq < 4; ++wq) {
    if (wq == 1) continue;  // (rows 0..15, cols 16..31): above the diagonal
    const int m0 = (wq >> 1) * 16, n0 = (wq & 1) * 16;
    double acc[2][2][2];
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
#pragma unroll
      for (int nt = 0; nt < 2; ++nt)
#pragma unroll
        for (int e = 0; e < 2; ++e)
          acc[mt][nt][e] = T[(32 + n0 + nt * 8 + 2 * q + e) * LDT + 32 + m0 + mt * 8 + g];
    mm32_quarter(acc, wq, lane, [&](int m, int k) { return -T[k * LDT + 32 + m]; },
                 [&](int k, int n) { return T[k * LDT + 32 + n]; });
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
#pragma unroll
      for (int nt = 0; nt < 2; ++nt)
#pragma unroll
        for (int e = 0; e < 2; ++e)
          T[(32 + n0 + nt * 8 + 2 * q + e) * LDT + 32 + m0 + mt * 8 + g] = acc[mt][nt][e];
    __syncwarp();
  }
  double* T22 = T + 32 * LDT + 32;
  info = potf2_block32<UP>(T22, LDT, nb2, lane, Ad + (size_t)32 * ld + 32, ld, s.wbuf, s.sv + 32,
                           s.tv + 32);
  if (info) return 32 + info;
  if (below) trtri32_dmma_warp(T22, LDT, s.tv + 32, T, LDT, s.S, LDS_T, lane);
  return 0;
}

template <class C, bool UP>
VB_DEVINL void la_produce(SmemLA<C>& s, const typename C::E* A, int n, int ld, int lane,
                          uint32_t& gchunk, uint32_t& ph_panel, uint32_t& ph_inv, uint32_t& ph_r1) {
  constexpr int NB = C::NB, MB = C::MB, KC = C::KC;
  using E = typename C::E;
  const bool bulk = !UP && ((reinterpret_cast<uintptr_t>(A) & 15) == 0) && (ld % C::G == 0);
  const int npan = (n + NB - 1) / NB;
  fence_proxy_async();
  for (int p = 0; p < npan; ++p) {
    const int j0 = p * NB, j1 = j0 + NB, nk = j0 / KC;
    if (p > 0) {  // panel p-1 stored (all its row blocks)
      if (lane == 0) mbar_wait(&s.panel_done, ph_panel & 1);
      ++ph_panel;
      __syncwarp();
    }
    if (j1 < n)
      for (int kc = 0; kc < nk; ++kc) issue_chunk2<C, UP>(s, gchunk++, kc, A, n, ld, j1, j0, lane, bulk);
    if (lane == 0) mbar_wait(&s.inv_ready, ph_inv & 1);
    ++ph_inv;
    __syncwarp();
    if (s.info_la || j1 >= n) break;
    // TILE(p+1): rows / columns j1..j1+63 over columns < j1; the newest 64 columns after R1(p)
    const int nk1 = j1 / KC;
    for (int kc = 0; kc < nk1; ++kc) {
      if (kc == nk) {
        if (lane == 0) mbar_wait(&s.r1_done, ph_r1 & 1);
        ++ph_r1;
        __syncwarp();
      }
      issue_chunk2<C, UP>(s, gchunk++, kc, A, n, ld, j1, j1, lane, bulk, NB);
    }
    for (int r0 = j1 + MB; r0 < n; r0 += MB)
      for (int kc = 0; kc < nk; ++kc) issue_chunk2<C, UP>(s, gchunk++, kc, A, n, ld, r0, j0, lane, bulk);
  }
}

// acc (this warp's 16 rows of a block at r0, columns j0..j0+63) = A (lower part if tri)
template <class C, bool UP>
VB_DEVINL void la_acc_init(double (&acc)[2][C::NT][2], const typename C::E* A, int n, int ld,
                           int row0, int j0, bool tri, int lane) {
  const int g = lane >> 2, q = lane & 3;
#pragma unroll
  for (int mt = 0; mt < 2; ++mt)
#pragma unroll
    for (int nt = 0; nt < C::NT; ++nt)
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int row = row0 + mt * 8 + g, col = j0 + nt * 8 + 2 * q + h;
        const bool v = row < n && col < n && (!tri || row >= col);
        acc[mt][nt][h] = v ? (double)__ldcg(A + gix<UP>(row, col, ld)) : 0.0;
      }
}

template <class C, bool UP>
VB_DEVINL void la_kloop(SmemLA<C>& s, double (&acc)[2][C::NT][2], uint32_t& gchunk, int nk, int wrow,
                        int ntl, int lane) {
  if (ntl == 0) k_loop3<C, 0>(s, acc, gchunk, nk, wrow, lane);
  else if (ntl == 2) k_loop3<C, 2>(s, acc, gchunk, nk, wrow, lane);
  else if (ntl == 4) k_loop3<C, 4>(s, acc, gchunk, nk, wrow, lane);
  else if (ntl == 6) k_loop3<C, 6>(s, acc, gchunk, nk, wrow, lane);
  else k_loop3<C, C::NT>(s, acc, gchunk, nk, wrow, lane);
}

template <class C, bool UP>
VB_DEVINL void la_store(const double (&acc)[2][C::NT][2], typename C::E* A, int n, int ld, int row0,
                        int j0, int lane) {
  const int g = lane >> 2, q = lane & 3;
#pragma unroll
  for (int mt = 0; mt < 2; ++mt)
#pragma unroll
    for (int nt = 0; nt < C::NT; ++nt)
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int row = row0 + mt * 8 + g, col = nt * 8 + 2 * q + h;
        if (row < n) A[gix<UP>(row, j0 + col, ld)] = acc[mt][nt][h];
      }
}

template <class C, bool UP>
VB_DEVINL void la_consume(SmemLA<C>& s, typename C::E* __restrict__ A, int n, int ld, int warp,
                          int lane, uint32_t& gchunk, uint32_t& ph_inv) {
  constexpr int NB = C::NB, MB = C::MB, KC = C::KC, NT = C::NT, LDT = C::LDT;
  constexpr int CT = 32 * C::WARPS;  // consumer threads
  const int g = lane >> 2, q = lane & 3, wrow = warp * 16;
  const int npan = (n + NB - 1) / NB;
  double acc[2][NT][2];
  if (warp < 4) {  // tile 0 = A's leading 64x64 block (no update)
    la_acc_init<C, UP>(acc, A, n, ld, wrow, 0, true, lane);
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
#pragma unroll
      for (int nt = 0; nt < NT; ++nt) {
        s.T[nt * 8 + 2 * q][wrow + mt * 8 + g] = acc[mt][nt][0];
        s.T[nt * 8 + 2 * q + 1][wrow + mt * 8 + g] = acc[mt][nt][1];
      }
    __syncwarp();
    if (lane == 0) mbar_arrive(&s.tile_ready);
  }
  for (int p = 0; p < npan; ++p) {
    const int j0 = p * NB, j1 = j0 + NB, nk = j0 / KC;
    const bool r1 = j1 < n;
    bool act = r1 && j1 + wrow < n;
    if (r1) {
      la_acc_init<C, UP>(acc, A, n, ld, j1 + wrow, j0, false, lane);
      la_kloop<C, UP>(s, acc, gchunk, nk, wrow, act ? NT : 0, lane);
    }
    mbar_wait(&s.inv_ready, ph_inv & 1);  // tile p factored (or failed)
    ++ph_inv;
    if (s.info_la || !r1) break;
    // D's operands for this panel's TRSMs, out of the tile (which TILE(p+1) reuses below)
    for (int e = threadIdx.x; e < 32 * 32; e += CT) {
      const int k = e >> 5, c = e & 31;
      s.cinv11[k][c] = s.T[32 + k][c];
      s.cl21[k][c] = s.T[k][32 + c];
      s.cinv22[k][c] = s.T[k][c];
    }
    bar_group(1, CT);
    if (act) {
      trsm_regs64_ops(&s.cinv11[0][0], &s.cl21[0][0], &s.cinv22[0][0], 36, acc, lane);
      la_store<C, UP>(acc, A, n, ld, j1 + wrow, j0, lane);
    }
    fence_proxy_async_global();  // R1's L is read by TMA (TILE(p+1) chunks)
    __syncwarp();
    if (lane == 0) mbar_arrive(&s.r1_done);
    // TILE(p+1): SYRK of rows / columns j1..j1+63 over columns < j1 (warps 0-3 compute)
    const bool tw = warp < 4 && j1 + wrow < n;
    if (warp < 4) la_acc_init<C, UP>(acc, A, n, ld, j1 + wrow, j1, true, lane);
    la_kloop<C, UP>(s, acc, gchunk, j1 / KC, wrow, tw ? (wrow + 16) / 8 : 0, lane);
    if (warp < 4) {
#pragma unroll
      for (int mt = 0; mt < 2; ++mt)
#pragma unroll
        for (int nt = 0; nt < NT; ++nt) {
          s.T[nt * 8 + 2 * q][wrow + mt * 8 + g] = acc[mt][nt][0];
          s.T[nt * 8 + 2 * q + 1][wrow + mt * 8 + g] = acc[mt][nt][1];
        }
      __syncwarp();
      if (lane == 0) mbar_arrive(&s.tile_ready);
    }
    // the rest of panel p
    for (int r0 = j1 + MB; r0 < n; r0 += MB) {
      act = r0 + wrow < n;
      la_acc_init<C, UP>(acc, A, n, ld, r0 + wrow, j0, false, lane);
      la_kloop<C, UP>(s, acc, gchunk, nk, wrow, act ? NT : 0, lane);
      if (act) {
        trsm_regs64_ops(&s.cinv11[0][0], &s.cl21[0][0], &s.cinv22[0][0], 36, acc, lane);
        la_store<C, UP>(acc, A, n, ld, r0 + wrow, j0, lane);
      }
    }
    fence_proxy_async_global();
    __syncwarp();
    if (lane == 0) mbar_arrive(&s.panel_done);
    bar_group(1, CT);  // every consumer is done with the operand copy before the next panel's
  }
  (void)LDT;
}

template <class C, bool UP>
VB_DEVINL void la_diag(SmemLA<C>& s, typename C::E* A, int n, int ld, int* info_out, int lane,
                       uint32_t& ph_tile) {
  constexpr int NB = C::NB;
  const int npan = (n + NB - 1) / NB;
  for (int t = 0; t < npan; ++t) {
    const int j0 = t * NB, nb = min(NB, n - j0);
    mbar_wait(&s.tile_ready, ph_tile & 1);
    ++ph_tile;
    const int info = diag64_one_warp<C, UP>(s, nb, lane, A + (size_t)j0 * ld + j0, ld, j0 + nb < n);
    if (info && lane == 0) {
      s.info_la = j0 + info;
      *info_out = j0 + info;
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&s.inv_ready);
    if (info) break;
  }
}

template <class C, bool UP>
__global__ void __launch_bounds__(32 * (C::WARPS + 2), C::MINB)
    potrf_la_kernel(const int* __restrict__ d_n, typename C::E* const* __restrict__ dA,
                    const int* __restrict__ d_ldda, int* __restrict__ d_info,
                    const Ctrl* __restrict__ ctrl_c, const int* __restrict__ order, int range,
                    int wait_upstream) {
  constexpr int W = C::WARPS;
  extern __shared__ __align__(128) unsigned char smem_la[];
  SmemLA<C>& s = *reinterpret_cast<SmemLA<C>*>(smem_la);
  Ctrl* ctrl = const_cast<Ctrl*>(ctrl_c);
  if (threadIdx.x == 0) {
    for (int i = 0; i < C::STAGES; ++i) {
      mbar_init(&s.full[i], 32);  // one arrival per producer lane
      mbar_init(&s.empty[i], W);
    }
    mbar_init(&s.panel_done, W);
    mbar_init(&s.r1_done, W);
    mbar_init(&s.tile_ready, 4);
    mbar_init(&s.inv_ready, 1);
    s.info_la = 0;
    fence_proxy_async();
  }
  __syncthreads();
  if (wait_upstream) pdl_wait();
  pdl_launch_dependents();
  const int count = *(volatile const int*)&ctrl->count[range];
  const int start = *(volatile const int*)&ctrl->start[range];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  uint32_t gchunk = 0, ph_panel = 0, ph_inv = 0, ph_r1 = 0, ph_tile = 0;
  for (;;) {
    if (tid == 0) {
      s.item = atomicAdd(&ctrl->head[range], 1);
      s.info_la = 0;
    }
    __syncthreads();
    const int it = s.item;
    __syncthreads();
    if (it >= count) break;
    const int m = order[start + it];
    TL_BEGIN(t_tl)
    if (warp == W) {
      la_produce<C, UP>(s, dA[m], d_n[m], d_ldda[m], lane, gchunk, ph_panel, ph_inv, ph_r1);
    } else if (warp == W + 1) {
      la_diag<C, UP>(s, dA[m], d_n[m], d_ldda[m], d_info + m, lane, ph_tile);
    } else {
      la_consume<C, UP>(s, dA[m], d_n[m], d_ldda[m], warp, lane, gchunk, ph_inv);
    }
    TL_END(tid == 0, t_tl, m, 31)
  }
  if (!wait_upstream && threadIdx.x == 0) pdl_wait();  // transitive completion (see blocked)
}

}  // namespace vb
