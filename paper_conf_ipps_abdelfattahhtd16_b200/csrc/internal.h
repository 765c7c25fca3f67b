// internal.h — host-side declarations shared by the translation units of libvbatched.so.
#pragma once
#include <cuda_runtime.h>

#include "common.cuh"

namespace vb {

// Size threshold: n > ts takes the NB=64 blocked kernel, 32 < n <= ts the small-matrix kernel
// (env VB_TS, default 128).
int potrf_ts();

cudaError_t launch_scan_bin(const int* d_n, const int* d_ldda, int* d_info, int batch, int max_n,
                            bool check_max, Ctrl* ctrl, int* order, cudaStream_t stream);

// Persistent factorisation over the sorted work list (blocked CTA path for n > 32,
// warp-per-matrix path for n <= 32). max_n_hint selects the launch configuration.
cudaError_t launch_potrf_paths(const int* d_n, double* const* dA, const int* d_ldda, int* d_info,
                               int batch, int max_n_hint, const Ctrl* ctrl, const int* order,
                               bool up, cudaStream_t stream);
// FP32 storage (SPOTRF): the same kernels with float loads/stores, FP64 arithmetic inside.
cudaError_t launch_potrf_paths(const int* d_n, float* const* dA, const int* d_ldda, int* d_info,
                               int batch, int max_n_hint, const Ctrl* ctrl, const int* order,
                               bool up, cudaStream_t stream);

int potrf_num_launches(int max_n_hint);
const char* potrf_kernel_names(int max_n_hint);  // the factorisation kernels after the scan
// max_n <= 32: one warp kernel that validates and factors directly (no scan).
cudaError_t launch_potrf_direct(const int* d_n, double* const* dA, const int* d_ldda, int* d_info,
                                int batch, int max_n, bool up, cudaStream_t stream);
cudaError_t launch_potrf_direct(const int* d_n, float* const* dA, const int* d_ldda, int* d_info,
                                int batch, int max_n, bool up, cudaStream_t stream);
void potrf_occupancy(int* out4);  // blocked CTAs/SM, blocked compute warps, 0, small CTAs/SM

// Stream-ordered scratch (pool-backed cudaMallocAsync).
cudaError_t ws_alloc(void** p, size_t bytes, cudaStream_t stream);
cudaError_t ws_free(void* p, cudaStream_t stream);

// vbatched BLAS launchers (blas.cu).
int gemm_launch(char ta, char tb, const int* d_m, const int* d_n, const int* d_k, double alpha,
                const double* const* dA, const int* d_lda, const double* const* dB,
                const int* d_ldb, double beta, double* const* dC, const int* d_ldc, int batch,
                int max_m, int max_n, int max_k, cudaStream_t stream);
int syrk_launch(char uplo, char trans, const int* d_n, const int* d_k, double alpha,
                const double* const* dA, const int* d_lda, double beta, double* const* dC,
                const int* d_ldc, int batch, int max_n, int max_k, cudaStream_t stream);
int trsm_launch(char side, char uplo, char ta, char diag, const int* d_m, const int* d_n,
                double alpha, const double* const* dA, const int* d_lda, double* const* dB,
                const int* d_ldb, int batch, int max_m, int max_n, cudaStream_t stream);

}  // namespace vb
