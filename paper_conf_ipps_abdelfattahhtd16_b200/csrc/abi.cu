// abi.cu — the C ABI of libvbatched.so (declared and documented in include/vbatched.h).
// Host-side work is O(1) per call (argument checks, workspace, launches) except for the
// host-buffer streaming entry point and the pure-host partition helper.
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <mutex>
#include <numeric>
#include <vector>

#include "../../include/vbatched.h"
#include "common.cuh"
#include "internal.h"

namespace vb {

// Stream-ordered workspace comes from a library-owned memory pool per device (created once,
// release threshold 256 MB so that steady-state calls do no OS round trip). The caller's
// default pool and its attributes are never touched.
static cudaMemPool_t g_pool[64] = {};
static std::mutex g_pool_mu;

static cudaError_t lib_pool(cudaMemPool_t* out) {
  int dev;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (dev < 0 || dev >= 64) return cudaErrorInvalidDevice;
  std::lock_guard<std::mutex> lock(g_pool_mu);
  if (!g_pool[dev]) {
    cudaMemPoolProps props = {};
    props.allocType = cudaMemAllocationTypePinned;
    props.handleTypes = cudaMemHandleTypeNone;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = dev;
    cudaMemPool_t p;
    if ((e = cudaMemPoolCreate(&p, &props)) != cudaSuccess) return e;
    // Workspace stays mapped between calls up to 8 GiB: with a small threshold the pool trims
    // at every synchronisation and the next call re-maps its workspace (GEQRF's is ~0.8 GB for
    // 3000 x 512 and took 47 or 62 ms per call depending on whether it had been trimmed).
    uint64_t thr = 8ull << 30;
    cudaMemPoolSetAttribute(p, cudaMemPoolAttrReleaseThreshold, &thr);
    g_pool[dev] = p;
  }
  *out = g_pool[dev];
  return cudaSuccess;
}

cudaError_t ws_alloc(void** p, size_t bytes, cudaStream_t stream) {
  cudaMemPool_t pool;
  cudaError_t e = lib_pool(&pool);
  if (e != cudaSuccess) return e;
  return cudaMallocFromPoolAsync(p, bytes, pool, stream);
}

cudaError_t ws_free(void* p, cudaStream_t stream) { return cudaFreeAsync(p, stream); }

static bool uplo_ok(char u) { return u == 'L' || u == 'l' || u == 'U' || u == 'u'; }

template <typename E>
static int potrf_impl(char uplo, const int* d_n, E* const* dA, const int* d_ldda, int* d_info,
                      int batch, int max_n, bool check_max, cudaStream_t stream) {
  if (!uplo_ok(uplo)) return -1;
  const bool up = (uplo == 'U' || uplo == 'u');
  if (batch < 0) return -6;
  if (check_max && max_n < 0) return -7;
  if (batch == 0) return 0;
  if (check_max && max_n <= kWarpMaxN)  // all matrices on the warp path: no scan needed
    return (int)launch_potrf_direct(d_n, dA, d_ldda, d_info, batch, max_n, up, stream);
  void* ws = nullptr;
  const size_t bytes = sizeof(Ctrl) + sizeof(int) * (size_t)batch;
  cudaError_t e = ws_alloc(&ws, bytes, stream);
  if (e != cudaSuccess) return (int)e;
  Ctrl* ctrl = static_cast<Ctrl*>(ws);
  int* order = reinterpret_cast<int*>(ctrl + 1);
  e = launch_scan_bin(d_n, d_ldda, d_info, batch, max_n, check_max, ctrl, order, stream);
  if (e == cudaSuccess) {
    const int hint = check_max ? max_n : (1 << 30);
    if (hint > 0)
      e = launch_potrf_paths(d_n, dA, d_ldda, d_info, batch, hint, ctrl, order, up, stream);
  }
  cudaError_t e2 = ws_free(ws, stream);
  if (e == cudaSuccess) e = e2;
  return (int)e;
}


// LAPACK DPOTRS on the vbatched factor: two side-'L' TRSMs (forward then backward substitution).
static int potrs_impl(char uplo, const int* d_n, const int* d_nrhs, const double* const* dA,
                      const int* d_ldda, double* const* dB, const int* d_lddb, int batch,
                      int max_n, int max_nrhs, cudaStream_t stream) {
  const bool up = (uplo == 'U' || uplo == 'u');
  // 'L': L Y = B, L^T X = Y.  'U' (A = U^T U): U^T Y = B, U X = Y.
  int rc = trsm_launch('L', up ? 'U' : 'L', up ? 'T' : 'N', 'N', d_n, d_nrhs, 1.0, dA, d_ldda, dB,
                       d_lddb, batch, max_n, max_nrhs, stream);
  if (rc != 0) return rc;
  return trsm_launch('L', up ? 'U' : 'L', up ? 'N' : 'T', 'N', d_n, d_nrhs, 1.0, dA, d_ldda, dB,
                     d_lddb, batch, max_n, max_nrhs, stream);
}

__global__ void nrhs_if_ok_kernel(const int* __restrict__ info, const int* __restrict__ nrhs,
                                  int* __restrict__ out, int batch) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < batch; i += gridDim.x * blockDim.x)
    out[i] = info[i] == 0 ? nrhs[i] : 0;
}

}  // namespace vb

using namespace vb;

extern "C" {

int vbatched_dpotrf(char uplo, const int* d_n, double* const* dA_array, const int* d_ldda,
                    int* d_info, int batchCount, int max_n, vb_stream_t stream) {
  return potrf_impl(uplo, d_n, dA_array, d_ldda, d_info, batchCount, max_n, true,
                    (cudaStream_t)stream);
}

int vbatched_spotrf(char uplo, const int* d_n, float* const* dA_array, const int* d_ldda,
                    int* d_info, int batchCount, int max_n, vb_stream_t stream) {
  return potrf_impl(uplo, d_n, dA_array, d_ldda, d_info, batchCount, max_n, true,
                    (cudaStream_t)stream);
}

int vbatched_spotrf_nomax(char uplo, const int* d_n, float* const* dA_array, const int* d_ldda,
                          int* d_info, int batchCount, vb_stream_t stream) {
  return potrf_impl(uplo, d_n, dA_array, d_ldda, d_info, batchCount, 0, false,
                    (cudaStream_t)stream);
}

int vbatched_dpotrf_nomax(char uplo, const int* d_n, double* const* dA_array, const int* d_ldda,
                          int* d_info, int batchCount, vb_stream_t stream) {
  return potrf_impl(uplo, d_n, dA_array, d_ldda, d_info, batchCount, 0, false,
                    (cudaStream_t)stream);
}

size_t vbatched_dpotrf_workspace_size(int batchCount) {
  return sizeof(Ctrl) + sizeof(int) * (size_t)(batchCount > 0 ? batchCount : 0);
}

int vbatched_dpotrf_scan(char uplo, const int* d_n, const int* d_ldda, int* d_info, int batchCount,
                         int max_n, void* d_workspace, vb_stream_t stream) {
  if (!uplo_ok(uplo)) return -1;
  if (batchCount < 0) return -5;
  if (max_n < 0) return -6;
  if (batchCount == 0) return 0;
  if (!d_workspace) return -7;
  if (max_n <= kWarpMaxN) return 0;  // the factor phase validates directly (no sort needed)
  Ctrl* ctrl = static_cast<Ctrl*>(d_workspace);
  return (int)launch_scan_bin(d_n, d_ldda, d_info, batchCount, max_n, true, ctrl,
                              reinterpret_cast<int*>(ctrl + 1), (cudaStream_t)stream);
}

int vbatched_dpotrf_factor(char uplo, const int* d_n, double* const* dA_array, const int* d_ldda,
                           int* d_info, int batchCount, int max_n, void* d_workspace,
                           vb_stream_t stream) {
  if (!uplo_ok(uplo)) return -1;
  const bool up = (uplo == 'U' || uplo == 'u');
  if (batchCount < 0) return -6;
  if (max_n < 0) return -7;
  if (batchCount == 0) return 0;
  if (!d_workspace) return -8;
  if (max_n <= kWarpMaxN)
    return (int)launch_potrf_direct(d_n, dA_array, d_ldda, d_info, batchCount, max_n, up,
                                    (cudaStream_t)stream);
  Ctrl* ctrl = static_cast<Ctrl*>(d_workspace);
  return (int)launch_potrf_paths(d_n, dA_array, d_ldda, d_info, batchCount, max_n, ctrl,
                                 reinterpret_cast<int*>(ctrl + 1), up, (cudaStream_t)stream);
}

int vbatched_dgemm(char transA, char transB, const int* d_m, const int* d_n, const int* d_k,
                   double alpha, const double* const* dA_array, const int* d_ldda,
                   const double* const* dB_array, const int* d_lddb, double beta,
                   double* const* dC_array, const int* d_lddc, int batchCount, int max_m,
                   int max_n, int max_k, vb_stream_t stream) {
  auto okT = [](char t) { return t == 'N' || t == 'n' || t == 'T' || t == 't' || t == 'C' || t == 'c'; };
  if (!okT(transA)) return -1;
  if (!okT(transB)) return -2;
  if (batchCount < 0) return -14;
  if (max_m < 0) return -15;
  if (max_n < 0) return -16;
  if (max_k < 0) return -17;
  if (batchCount == 0) return 0;
  return gemm_launch(transA, transB, d_m, d_n, d_k, alpha, dA_array, d_ldda, dB_array, d_lddb, beta,
                     dC_array, d_lddc, batchCount, max_m, max_n, max_k, (cudaStream_t)stream);
}

int vbatched_dsyrk(char uplo, char trans, const int* d_n, const int* d_k, double alpha,
                   const double* const* dA_array, const int* d_ldda, double beta,
                   double* const* dC_array, const int* d_lddc, int batchCount, int max_n,
                   int max_k, vb_stream_t stream) {
  if (!(uplo == 'L' || uplo == 'l' || uplo == 'U' || uplo == 'u')) return -1;
  if (!(trans == 'N' || trans == 'n' || trans == 'T' || trans == 't' || trans == 'C' || trans == 'c')) return -2;
  if (batchCount < 0) return -11;
  if (max_n < 0) return -12;
  if (max_k < 0) return -13;
  if (batchCount == 0) return 0;
  return syrk_launch(uplo, trans, d_n, d_k, alpha, dA_array, d_ldda, beta, dC_array, d_lddc,
                     batchCount, max_n, max_k, (cudaStream_t)stream);
}

int vbatched_dtrsm(char side, char uplo, char transA, char diag, const int* d_m, const int* d_n,
                   double alpha, const double* const* dA_array, const int* d_ldda,
                   double* const* dB_array, const int* d_lddb, int batchCount, int max_m,
                   int max_n, vb_stream_t stream) {
  if (!(side == 'R' || side == 'r' || side == 'L' || side == 'l')) return -1;
  if (!(uplo == 'L' || uplo == 'l' || uplo == 'U' || uplo == 'u')) return -2;
  if (!(transA == 'N' || transA == 'n' || transA == 'T' || transA == 't' || transA == 'C' || transA == 'c')) return -3;
  if (!(diag == 'N' || diag == 'n' || diag == 'U' || diag == 'u')) return -4;
  if (batchCount < 0) return -12;
  if (max_m < 0) return -13;
  if (max_n < 0) return -14;
  if (batchCount == 0) return 0;
  return trsm_launch(side, uplo, transA, diag, d_m, d_n, alpha, dA_array, d_ldda, dB_array, d_lddb,
                     batchCount, max_m, max_n, (cudaStream_t)stream);
}

int vbatched_dpotrs(char uplo, const int* d_n, const int* d_nrhs, const double* const* dA_array,
                    const int* d_ldda, double* const* dB_array, const int* d_lddb, int batchCount,
                    int max_n, int max_nrhs, vb_stream_t stream) {
  if (!uplo_ok(uplo)) return -1;
  if (batchCount < 0) return -8;
  if (max_n < 0) return -9;
  if (max_nrhs < 0) return -10;
  if (batchCount == 0) return 0;
  return potrs_impl(uplo, d_n, d_nrhs, dA_array, d_ldda, dB_array, d_lddb, batchCount, max_n,
                    max_nrhs, (cudaStream_t)stream);
}

int vbatched_dposv(char uplo, const int* d_n, const int* d_nrhs, double* const* dA_array,
                   const int* d_ldda, double* const* dB_array, const int* d_lddb, int* d_info,
                   int batchCount, int max_n, int max_nrhs, vb_stream_t stream) {
  if (!uplo_ok(uplo)) return -1;
  if (batchCount < 0) return -9;
  if (max_n < 0) return -10;
  if (max_nrhs < 0) return -11;
  if (batchCount == 0) return 0;
  cudaStream_t st = (cudaStream_t)stream;
  int rc = potrf_impl(uplo, d_n, dA_array, d_ldda, d_info, batchCount, max_n, true, st);
  if (rc != 0) return rc;
  // matrices that failed (info != 0) keep B unchanged (LAPACK DPOSV): solve with nrhs = 0
  void* ws = nullptr;
  cudaError_t e = ws_alloc(&ws, sizeof(int) * (size_t)batchCount, st);
  if (e != cudaSuccess) return (int)e;
  int* nrhs_eff = static_cast<int*>(ws);
  nrhs_if_ok_kernel<<<std::min((batchCount + 255) / 256, 1024), 256, 0, st>>>(d_info, d_nrhs,
                                                                             nrhs_eff, batchCount);
  e = cudaGetLastError();
  if (e == cudaSuccess)
    rc = potrs_impl(uplo, d_n, nrhs_eff, dA_array, d_ldda, dB_array, d_lddb, batchCount, max_n,
                    max_nrhs, st);
  cudaError_t e2 = ws_free(ws, st);
  if (e != cudaSuccess) return (int)e;
  return rc != 0 ? rc : (int)e2;
}

int vbatched_partition_lpt(const int* h_n, int batchCount, int ngpu, int* h_owner) {
  if (batchCount < 0) return -2;
  if (ngpu < 1) return -3;
  std::vector<int> idx(batchCount);
  std::iota(idx.begin(), idx.end(), 0);
  std::stable_sort(idx.begin(), idx.end(), [&](int a, int b) { return h_n[a] > h_n[b]; });
  std::vector<double> load(ngpu, 0.0);
  for (int i : idx) {
    int best = 0;
    for (int r = 1; r < ngpu; ++r)
      if (load[r] < load[best]) best = r;
    const double n = h_n[i] > 0 ? (double)h_n[i] : 0.0;
    load[best] += n * n * n / 3.0;
    h_owner[i] = best;
  }
  return 0;
}

const char* vbatched_version(void) {
  static char buf[320];
  int occ[4] = {0, 4, 0, 0};  // without a device: the default v3 width, occupancies unknown (0)
  int dev_count = 0;
  if (cudaGetDeviceCount(&dev_count) == cudaSuccess && dev_count > 0) potrf_occupancy(occ);
  else cudaGetLastError();
  snprintf(buf, sizeof buf,
           "libvbatched 0.6 (sm_100a; DMMA m8n8k4 f64; n>%d: blocked NB=64, %d compute warps + TMA "
           "producer, %d CTAs/SM; 32<n<=%d: paired look-ahead small kernel, %d CTAs/SM; n<=32: "
           "warp per matrix; FP64 and FP32 storage, uplo L/U)",
           potrf_ts(), occ[1], occ[0], potrf_ts(), occ[3]);
  return buf;
}

int vbatched_dpotrf_kernel_launches(int max_n) { return max_n > 0 ? potrf_num_launches(max_n) : 0; }

const char* vbatched_dpotrf_kernel_names(int max_n) { return potrf_kernel_names(max_n); }

void* vbatched_host_alloc(size_t bytes) {
  void* p = nullptr;
  if (cudaHostAlloc(&p, bytes, cudaHostAllocDefault) != cudaSuccess) return nullptr;
  return p;
}

int vbatched_host_free(void* p) { return (int)cudaFreeHost(p); }

}  // extern "C"
