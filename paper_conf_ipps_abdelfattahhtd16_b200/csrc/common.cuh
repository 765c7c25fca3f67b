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

}  // namespace vb
