// scan_bin.cu — step a1 of the hot path: one pass over the size
// arrays that validates every matrix (info init), computes the device max, and
// counting-sorts the valid matrices by n DESCENDING into one work list, so that the
// persistent factorisation kernels pop the largest (most flops) matrices first
// (longest-processing-time order).
//
// Paper: the size arrays live on the GPU, so integer kernels over them are needed
// (§III-A); the max computation and the aux kernels
// of the driver are "negligible"; processing matrices of nearly
// similar size together fixes load imbalance ("implicit sorting") —
// here replaced by an explicit sort, because the persistent kernels are not launched
// step by step over a max-size grid.
#include "common.cuh"
#include "internal.h"

namespace vb {

constexpr int kScanThreads = 1024;
constexpr int kKeys = 4096;  // sort keys: min(n, kKeys-1) (larger n share the top key)
constexpr int kCache = 8;    // items per thread whose key stays in registers (batch <= 8192)

__global__ void __launch_bounds__(kScanThreads, 1)
    scan_bin_kernel(const int* __restrict__ d_n, const int* __restrict__ d_ldda,
                    int* __restrict__ d_info, int batch, int max_n, int check_max, int ts,
                    Ctrl* __restrict__ ctrl, int* __restrict__ order) {
  // Let the dependent (factorisation) grid launch and reach its griddepcontrol.wait now.
  pdl_launch_dependents();
  __shared__ int hist[kKeys];
  __shared__ int wsum[kScanThreads / 32];
  __shared__ int wmax[kScanThreads / 32];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  for (int k = tid; k < kKeys; k += kScanThreads) hist[k] = 0;
  __syncthreads();

  // The first kCache items of each thread keep their sort key in registers for the scatter
  // pass (batch <= 8192 needs no second read of n / info); the loads of a thread's items are
  // issued together (unrolled) so their latencies overlap. key < 0: not sorted (invalid, n=0).
  int key[kCache];
  int mymax = 0;
#pragma unroll
  for (int u = 0; u < kCache; ++u) {
    const int i = tid + u * kScanThreads;
    key[u] = -1;
    if (i < batch) {
      const int n = d_n[i], ld = d_ldda[i];
      int code = 0;
      if (n < 0) code = -2;
      else if (ld < (n > 1 ? n : 1)) code = -4;
      else if (check_max && n > max_n) code = -7;
      d_info[i] = code;
      if (code == 0 && n > 0) {
        key[u] = n < kKeys ? n : kKeys - 1;
        mymax = n > mymax ? n : mymax;
      }
    }
  }
#pragma unroll
  for (int u = 0; u < kCache; ++u)
    if (key[u] >= 0) atomicAdd(&hist[key[u]], 1);
  for (int i = tid + kCache * kScanThreads; i < batch; i += kScanThreads) {
    const int n = d_n[i], ld = d_ldda[i];
    int code = 0;
    if (n < 0) code = -2;
    else if (ld < (n > 1 ? n : 1)) code = -4;
    else if (check_max && n > max_n) code = -7;
    d_info[i] = code;
    if (code == 0 && n > 0) {
      atomicAdd(&hist[n < kKeys ? n : kKeys - 1], 1);
      mymax = n > mymax ? n : mymax;
    }
  }
  for (int o = 16; o; o >>= 1) mymax = max(mymax, __shfl_xor_sync(kFull, mymax, o));
  if (lane == 0) wmax[warp] = mymax;
  __syncthreads();

  // Exclusive scan over keys in DESCENDING order: start[k] = #items with key > k.
  // Thread t owns the 4 keys kKeys-1-4t .. kKeys-4-4t (descending).
  constexpr int kPer = kKeys / kScanThreads;
  int local[kPer];
  int s = 0;
#pragma unroll
  for (int u = 0; u < kPer; ++u) {
    local[u] = hist[kKeys - 1 - (tid * kPer + u)];
    s += local[u];
  }
  int incl = s;
  for (int o = 1; o < 32; o <<= 1) {
    int v = __shfl_up_sync(kFull, incl, o);
    if (lane >= o) incl += v;
  }
  if (lane == 31) wsum[warp] = incl;
  __syncthreads();
  if (warp == 0) {
    int v = wsum[lane];
    int w = v;
    for (int o = 1; o < 32; o <<= 1) {
      int t = __shfl_up_sync(kFull, w, o);
      if (lane >= o) w += t;
    }
    wsum[lane] = w - v;  // exclusive warp offsets
    int m = wmax[lane];
    for (int o = 16; o; o >>= 1) m = max(m, __shfl_xor_sync(kFull, m, o));
    if (lane == 0) wmax[0] = m;
  }
  __syncthreads();
  int run = wsum[warp] + incl - s;  // exclusive start of this thread's first key
#pragma unroll
  for (int u = 0; u < kPer; ++u) {
    hist[kKeys - 1 - (tid * kPer + u)] = run;  // hist now holds start offsets
    run += local[u];
  }
  __syncthreads();
  if (tid == 0) {
    // start[k] = #items with key > k (descending order): the three ranges are contiguous.
    const int tks = ts < kWarpMaxN ? kWarpMaxN : (ts > kKeys - 1 ? kKeys - 1 : ts);
    const int bounds[kRanges + 1] = {0, hist[tks], hist[kWarpMaxN], hist[0]};
    for (int r = 0; r < kRanges; ++r) {
      ctrl->head[r] = 0;
      ctrl->start[r] = bounds[r];
      ctrl->count[r] = bounds[r + 1] - bounds[r];
    }
    ctrl->max_n = wmax[0];
  }
  __syncthreads();
#pragma unroll
  for (int u = 0; u < kCache; ++u)
    if (key[u] >= 0) order[atomicAdd(&hist[key[u]], 1)] = tid + u * kScanThreads;
  for (int i = tid + kCache * kScanThreads; i < batch; i += kScanThreads) {
    const int n = d_n[i];
    // re-derive validity exactly as above (info was written by this thread)
    if (d_info[i] == 0 && n > 0) {
      const int pos = atomicAdd(&hist[n < kKeys ? n : kKeys - 1], 1);
      order[pos] = i;
    }
  }
}

cudaError_t launch_scan_bin(const int* d_n, const int* d_ldda, int* d_info, int batch, int max_n,
                            bool check_max, Ctrl* ctrl, int* order, cudaStream_t stream) {
  scan_bin_kernel<<<1, kScanThreads, 0, stream>>>(d_n, d_ldda, d_info, batch, max_n,
                                                  check_max ? 1 : 0, potrf_ts(), ctrl, order);
  return cudaGetLastError();
}

}  // namespace vb
