// common.cuh — device helpers shared by the vbatched kernels (sm_100a only).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#if defined(__CUDA_ARCH__) && (__CUDA_ARCH__ != 1000)
#error "libvbatched is written for sm_100a only (compile with -gencode arch=compute_100a,code=sm_100a)"
#endif

#define VB_DEVINL __device__ __forceinline__

namespace vb {

constexpr unsigned kFull = 0xffffffffu;

// Control block written by the scan (one per call, in the stream-ordered workspace).
// The sorted work list order[] holds the valid matrices by n descending, split in three
// contiguous ranges, one per factorisation kernel:
//   range 0: n > ts           (blocked kernel, panel width 64)
//   range 1: 32 < n <= ts     (small-matrix kernel, 2 warps per matrix)
//   range 2: 1 <= n <= 32     (warp-per-matrix kernel)
constexpr int kRanges = 3;
struct Ctrl {
  int head[kRanges];   // atomic queue heads (per range)
  int count[kRanges];  // matrices per range
  int start[kRanges];  // first position of each range in order[]
  int max_n;           // max n over valid matrices (for the _nomax interface / logging)
  int pad[6];
};

constexpr int kWarpMaxN = 32;

// Offset of element (r, c) of the lower factor L (r >= c) in a matrix's storage: uplo 'L' keeps
// L in the lower triangle, column-major (r + c ld); uplo 'U' keeps U = L^T in the upper
// triangle, so L(r, c) = U(c, r) sits at c + r ld.
template <bool UP>
VB_DEVINL size_t gix(int r, int c, int ld) {
  return UP ? (size_t)r * ld + c : (size_t)c * ld + r;
}  // warp-per-matrix path for n <= 32

// FP64 tensor-core MMA: D(8x8) += A(8x4, row) * B(4x8, col). Native SASS: DMMA.8x8x4.
// Fragment layout (verified on B200 by tools/fp64_peaks.cu): lane l = 4g + q holds
//   A[g][q], B[q][g], and C[g][2q], C[g][2q+1].
VB_DEVINL void dmma(double (&d)[2], double a, double b) {
  asm("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
      : "+d"(d[0]), "+d"(d[1])
      : "d"(a), "d"(b));
}

// p ? x : y through an opaque PTX selp, so that the compiler cannot rewrite a per-element
// select over an unrolled register array into a dynamically indexed store.
VB_DEVINL double selp(bool p, double x, double y) {
  double r;
  asm("{\n .reg .pred q;\n setp.ne.s32 q, %3, 0;\n selp.f64 %0, %1, %2, q;\n}\n"
      : "=d"(r) : "d"(x), "d"(y), "r"((int)p));
  return r;
}

VB_DEVINL uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// cp.async 8 bytes with zero fill when !pred (src must still be a mapped address).
VB_DEVINL void cp_async8(void* sdst, const void* gsrc, bool pred) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(smem_u32(sdst)), "l"(gsrc),
               "r"(pred ? 8 : 0));
}
// cp.async 4 bytes with zero fill when !pred.
VB_DEVINL void cp_async4(void* sdst, const void* gsrc, bool pred) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;\n" ::"r"(smem_u32(sdst)), "l"(gsrc),
               "r"(pred ? 4 : 0));
}
// cp.async of one element of the storage type (double or float).
template <typename E>
VB_DEVINL void cp_async_e(E* sdst, const E* gsrc, bool pred) {
  if constexpr (sizeof(E) == 8)
    cp_async8(sdst, gsrc, pred);
  else
    cp_async4(sdst, gsrc, pred);
}
// cp.async 16 bytes (L2 only), zero fill when !pred.
VB_DEVINL void cp_async16(void* sdst, const void* gsrc, bool pred) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(smem_u32(sdst)), "l"(gsrc),
               "r"(pred ? 16 : 0));
}
// The barrier tracks this thread's prior cp.async copies (pending count +1 now, the async
// arrive on completion: zero net arrivals; the phase cannot complete before the copies land).
VB_DEVINL void cp_async_mbar_arrive(uint64_t* bar) {
  asm volatile("cp.async.mbarrier.arrive.shared::cta.b64 [%0];\n" ::"r"(smem_u32(bar)) : "memory");
}
// The barrier receives this thread's arrival once all its prior cp.async copies have completed
// (the pending count is not incremented: the arrival counts toward the phase's expected count).
VB_DEVINL void cp_async_mbar_arrive_noinc(uint64_t* bar) {
  asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];\n" ::"r"(smem_u32(bar)) : "memory");
}
VB_DEVINL void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::); }
template <int N>
VB_DEVINL void cp_async_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N)); }

// ---- mbarrier + TMA bulk copy (cp.async.bulk, SASS UBLKCP) ----
VB_DEVINL void mbar_init(uint64_t* bar, int count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(count)
               : "memory");
}
// Arrive on the barrier and add `bytes` to its expected transaction count.
VB_DEVINL void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}
// Add `bytes` to the current phase's expected transaction count (no arrival).
VB_DEVINL void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.expect_tx.relaxed.cta.shared::cta.b64 [%0], %1;\n" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}
// `cnt` arrivals at once.
VB_DEVINL void mbar_arrive_cnt(uint64_t* bar, uint32_t cnt) {
  asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0], %1;\n" ::"r"(smem_u32(bar)),
               "r"(cnt)
               : "memory");
}
VB_DEVINL void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];\n" ::"r"(smem_u32(bar)) : "memory");
}
VB_DEVINL void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n WAIT_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      " @!p bra WAIT_%=;\n}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
// 1-D bulk copy global -> shared (16-byte aligned addresses, size a multiple of 16), completing
// `bytes` of the barrier's transaction count.
VB_DEVINL void bulk_g2s(void* sdst, const void* gsrc, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n" ::"r"(
          smem_u32(sdst)),
      "l"(gsrc), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
// The same with an L2 cache policy (createpolicy): evict_first for streamed data, evict_last
// for data the CTA will read again soon.
VB_DEVINL void bulk_g2s_hint(void* sdst, const void* gsrc, uint32_t bytes, uint64_t* bar,
                             uint64_t policy) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], "
      "%2, [%3], %4;\n" ::"r"(smem_u32(sdst)),
      "l"(gsrc), "r"(bytes), "r"(smem_u32(bar)), "l"(policy)
      : "memory");
}
VB_DEVINL uint64_t policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;\n" : "=l"(p));
  return p;
}
VB_DEVINL uint64_t policy_evict_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;\n" : "=l"(p));
  return p;
}
// L2 prefetch of a contiguous global range (TMA unit; 16-byte aligned, size multiple of 16).
VB_DEVINL void bulk_prefetch_l2(const void* gsrc, uint32_t bytes) {
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;\n" ::"l"(gsrc), "r"(bytes) : "memory");
}
// C-fragment -> A-fragment of m8n8k4 DMMA: this lane's C values (row g, cols 2q, 2q+1) of an
// 8x8 tile; returns A[g][4*half + q] for the k-step covering tile columns 4*half..4*half+3.
VB_DEVINL double cfrag_to_afrag(double c0, double c1, int half, int lane) {
  const int src = (lane & ~3) | (2 * half + ((lane & 3) >> 1));
  const double v0 = __shfl_sync(0xffffffffu, c0, src);
  const double v1 = __shfl_sync(0xffffffffu, c1, src);
  return (lane & 1) ? v1 : v0;
}
// Order this thread's prior generic-proxy shared-memory accesses before later async-proxy ones.
VB_DEVINL void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory"); }
// Same for global memory: this thread's generic stores (the L panels it wrote) before later
// TMA (async-proxy) reads of them by any thread of the CTA (after a barrier).
VB_DEVINL void fence_proxy_async_global() {
  asm volatile("fence.proxy.async.global;\n" ::: "memory");
}

// Programmatic dependent launch (PDL): wait for the upstream grid's results / let the
// downstream grid start its prologue early.
VB_DEVINL void pdl_wait() { asm volatile("griddepcontrol.wait;\n" ::: "memory"); }
VB_DEVINL void pdl_launch_dependents() { asm volatile("griddepcontrol.launch_dependents;\n" ::); }

// Named barriers (bar.sync / bar.arrive on a subset of the CTA's warps).
VB_DEVINL void bar_group(int id, int nthreads) {
  asm volatile("bar.sync %0, %1;\n" ::"r"(id), "r"(nthreads) : "memory");
}
VB_DEVINL void bar_group_arrive(int id, int nthreads) {
  asm volatile("bar.arrive %0, %1;\n" ::"r"(id), "r"(nthreads) : "memory");
}

constexpr int LDS_T = 18;  // TRTRI32 scratch leading dim (16 columns used)

// Inverse of a 32x32 lower-triangular L (T[c*ldt+r] = L[r][c], tv[c] = 1/L[c][c]) by one
// warp: 8x8 diagonal blocks by substitution (lane = block column), then two levels of
// recursive doubling inv([[A,0],[B,C]]) = [[inv A, 0], [-inv C B inv A, inv C]] on DMMA.
// Output INV[k*ldi + n] = X[n][k], X = L^-1 (the TRSM's B operand layout); the 32x32 block
// of INV is fully written (zeros above the diagonal of X). S: 16 x LDS_T x 2 doubles with
// leading dimension lds.
VB_DEVINL void trtri32_dmma_warp(const double* T, int ldt, const double* tv, double* INV,
                                 int ldi, double* S, int lds, int lane) {
  const int g = lane >> 2, q = lane & 3;
  for (int e = lane; e < 32 * 32; e += 32) INV[(e >> 5) * ldi + (e & 31)] = 0.0;
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
        const double a = T[(o + ks * 4 + q) * ldt + o + 8 + g];  // B[g][k]
        const double bb = INV[(o + g) * ldi + o + ks * 4 + q];   // invA[k][g]
        dmma(t[p], a, bb);
      }
    }
#pragma unroll
    for (int p = 0; p < 2; ++p) {
      S[(p * 8 + g) * lds + 2 * q] = t[p][0];
      S[(p * 8 + g) * lds + 2 * q + 1] = t[p][1];
    }
    __syncwarp();
    double r[2][2] = {{0.0, 0.0}, {0.0, 0.0}};
#pragma unroll
    for (int p = 0; p < 2; ++p) {
      const int o = 16 * p;
#pragma unroll
      for (int ks = 0; ks < 2; ++ks) {
        const double a = INV[(o + 8 + ks * 4 + q) * ldi + o + 8 + g];  // invC[g][k]
        const double bb = S[(p * 8 + ks * 4 + q) * lds + g];            // Tm[k][g]
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
        S[(mt * 8 + g) * lds + nt * 8 + 2 * q] = t[mt][nt][0];
        S[(mt * 8 + g) * lds + nt * 8 + 2 * q + 1] = t[mt][nt][1];
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
      for (int nt = 0; nt < 2; ++nt) bb[nt] = S[(ks * 4 + q) * lds + nt * 8 + g];
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

}  // namespace vb
