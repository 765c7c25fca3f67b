/*
 * vbatched.h — C ABI of the B200-native variable-size batched Cholesky library
 * (libvbatched.so, built from paper_conf_ipps_abdelfattahhtd16_b200/csrc/).
 *
 * Problem (Fig. 1; §III-A): a batch of k independent
 * dense matrices, matrix i being N_i x N_i with its own leading dimension LDA_i, each
 * factored as A_i = L_i L_i^T. A "vbatched" routine takes an array of pointers, the arrays
 * of sizes and leading dimensions (resident in GPU memory) and the batch
 * count; the max-given interface additionally takes the maximum size
 * (PAPER.md:388-412), the LAPACK-like one computes it on the GPU.
 *
 * Conventions for every routine below
 *  - Matrices are column-major doubles: element (r,c) of matrix i is dA_array[i][r + c*ldda[i]].
 *  - Pointer arguments prefixed d are DEVICE pointers on the current CUDA device; h = host.
 *    The caller owns every array; the library never frees or reallocates caller memory.
 *  - All int arguments are 32-bit. Offsets inside the library are computed in 64 bits.
 *  - Asynchronous: work is enqueued on `stream` (0 = legacy default stream); no host
 *    synchronisation and no device->host copy happens unless the routine says so. Internal
 *    workspace (O(batchCount) ints) is stream-ordered (cudaMallocFromPoolAsync/cudaFreeAsync
 *    on a memory pool the library creates per device; the caller's default pool and its
 *    attributes are not touched). The library's pool keeps up to 8 GiB of freed workspace
 *    mapped between calls (GEQRF/GETRF need O(batchCount (max_m + max_n)) doubles).
 *  - Return value: 0 = enqueued; -p = host-scalar argument number p (1-based) is invalid,
 *    nothing enqueued; > 0 = a cudaError_t from the launch.
 *  - batchCount == 0 returns 0 and enqueues nothing.
 *  - No CPU fallback exists: every arithmetic step runs in this library's CUDA kernels
 *    (sm_100a). If no device is present the call returns the CUDA error.
 */
#ifndef VBATCHED_H_
#define VBATCHED_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st* vb_stream_t; /* == cudaStream_t */

/* ---------------------------------------------------------------------------------------
 * vbatched_dpotrf — FP64 variable-size batched Cholesky, max-given interface.
 * Cite: PAPER.md:520-549 (§III-D, Algorithm 1: panel update (syrk) -> tile factorize (potf2)
 * -> panel factorize (trsm)); PAPER.md:724-812 (§III-E separated kernels); error reporting
 * follows LAPACK DPOTRF [7] (PAPER.md:2291-2297 lists it as future work).
 *
 *  uplo       'L' (lower): A_i = L L^T, the factor L overwrites the lower triangle of each A_i;
 *             only the lower triangle is referenced.
 *             'U' (upper): A_i = U^T U, U = L^T overwrites the upper triangle; only the upper
 *             triangle is referenced (the same factorisation on the transposed view, so the
 *             results are bit-identical to 'L' on the mirrored storage; SURVEY.md §8(f)
 *             NEXT-1, LAPACK DPOTRF). Anything else returns -1.
 *  d_n        [batchCount] matrix orders n_i (device).
 *  dA_array   [batchCount] device pointers to the matrices (device array of device ptrs).
 *  d_ldda     [batchCount] leading dimensions (device); must be >= max(1, n_i).
 *  d_info     [batchCount] output (device), LAPACK semantics per matrix:
 *               0  success;
 *               k>0 the leading minor of order k is not positive definite: the k-th pivot
 *                  was <= 0 or NaN. Columns 1..k-1 hold L of the leading block; the failing
 *                  pivot value is stored at (k,k); the rest of the referenced triangle is
 *                  implementation-defined (partially updated).
 *              -2  n_i < 0;  -4  ldda_i < max(1,n_i);  -7  n_i > max_n.  (matrix untouched)
 *  batchCount number of matrices (>= 0)                                      (-6 if < 0)
 *  max_n      an upper bound on every n_i (host)                              (-7 if < 0)
 *  stream     CUDA stream.
 * The other (unreferenced) strict triangle and rows n_i..ldda_i-1 are never WRITTEN. They are
 * not read either, with one exception: the 16-byte TMA bulk copies of the n_i > 128 path round
 * each column segment up to 16 bytes, so with uplo 'L' up to one padding element per column
 * (row n_i when n_i is odd; it lies inside ldda_i) may be read. Its value never reaches any
 * stored result, so NaN/Inf padding is harmless; it must only be readable memory (it is, since
 * ldda_i >= n_i + 1 whenever the copy reaches it).
 * Matrices must not overlap. Returns 0 / -p / cudaError_t as described above.
 */
int vbatched_dpotrf(char uplo, const int* d_n, double* const* dA_array, const int* d_ldda,
                    int* d_info, int batchCount, int max_n, vb_stream_t stream);

/* vbatched_spotrf — the same factorisation of FP32 matrices (the paper
 * tests single precision too). Arguments, layout, uplo, info codes and
 * ownership exactly as vbatched_dpotrf with float storage. B200 has no exact-FP32 tensor-core
 * MMA, so the kernels load FP32, compute in FP64 on the DMMA tensor cores (pivots, updates and
 * TRSM in FP64) and store the factor rounded to FP32; each stored column is re-read in FP32 by
 * later panels. Results are therefore at least as accurate as an FP32 LAPACK SPOTRF; info
 * follows the FP64 pivot test (!(p > 0)). ldda_i that is not a multiple of 4 (16 bytes) takes the
 * cp.async staging path instead of TMA bulk copies. */
int vbatched_spotrf(char uplo, const int* d_n, float* const* dA_array, const int* d_ldda,
                    int* d_info, int batchCount, int max_n, vb_stream_t stream);
/* FP32 LAPACK-like interface (no max_n; see vbatched_dpotrf_nomax). */
int vbatched_spotrf_nomax(char uplo, const int* d_n, float* const* dA_array, const int* d_ldda,
                          int* d_info, int batchCount, vb_stream_t stream);

/* LAPACK-like interface: identical to vbatched_dpotrf but max_n is not
 * needed; the device scan computes it (no host synchronisation: launch sizes assume the
 * worst case and idle CTAs exit). Argument numbers as above; there is no check -7. */
int vbatched_dpotrf_nomax(char uplo, const int* d_n, double* const* dA_array,
                          const int* d_ldda, int* d_info, int batchCount, vb_stream_t stream);

/* Two-phase form of vbatched_dpotrf with caller-owned workspace (same arguments, same
 * results; vbatched_dpotrf == scan + factor on an internal workspace):
 *   vbatched_dpotrf_workspace_size(batchCount) -> bytes of device workspace needed;
 *   vbatched_dpotrf_scan:   step a1 — validate n/ldda (writes info -2/-4/-7/0), compute the
 *                           device max, counting-sort the valid matrices by n descending
 *                           into the workspace;
 *   vbatched_dpotrf_factor: steps a2-a7 — the persistent factorisation kernel draining the
 *                           sorted work list written by the preceding scan on the same
 *                           workspace (must follow it in stream order, once).
 * d_workspace: device memory of at least vbatched_dpotrf_workspace_size bytes, 16-byte
 * aligned, not used concurrently by another call. Return codes are minus the argument
 * position in each function's own list (scan: uplo -1, batchCount -5, max_n -6, NULL
 * workspace -7; factor: uplo -1, batchCount -6, max_n -7, NULL workspace -8). */
size_t vbatched_dpotrf_workspace_size(int batchCount);
int vbatched_dpotrf_scan(char uplo, const int* d_n, const int* d_ldda, int* d_info,
                         int batchCount, int max_n, void* d_workspace, vb_stream_t stream);
int vbatched_dpotrf_factor(char uplo, const int* d_n, double* const* dA_array,
                           const int* d_ldda, int* d_info, int batchCount, int max_n,
                           void* d_workspace, vb_stream_t stream);

/* ---------------------------------------------------------------------------------------
 * vbatched_dpotrf_host — end-to-end variant on HOST memory (blocking).
 * Same problem and semantics as vbatched_dpotrf, but h_n, hA_array (host pointers to host
 * matrices, ideally pinned), h_ldda and h_info live in host memory. The library streams the
 * batch through a device staging ring in chunks: H2D copy of a chunk's matrices, factor
 * (the same kernels as vbatched_dpotrf), D2H copy back, with copies of neighbouring chunks
 * overlapping the factorisation. Each matrix's whole ldda x n column block is copied in
 * and back (the strict upper triangle and padding rows are returned unchanged).
 * Returns when every result is back in host memory. workspace_bytes bounds the device
 * staging memory (0 = library default, 6 GiB; the staging buffers are cached per device and reused by later calls). Argument checks as vbatched_dpotrf
 * (-2 n<0 and -4 ldda<max(1,n) are reported in h_info, -7 if n > max_n).
 * Extra return code: -9 = workspace_bytes too small for the largest matrix. */
int vbatched_dpotrf_host(char uplo, const int* h_n, double* const* hA_array, const int* h_ldda,
                         int* h_info, int batchCount, int max_n, size_t workspace_bytes,
                         vb_stream_t stream);

/* ---------------------------------------------------------------------------------------
 * vbatched BLAS used by the blocked factorisation (§III-E.2/3), exposed
 * as standalone entry points. Per-matrix dimension arrays are device arrays; dimensions are
 * assumed valid (MAGMA "_nocheck" convention); host scalars are checked.
 *
 * vbatched_dgemm: C_i = alpha op(A_i) op(B_i) + beta C_i, C_i m_i x n_i, op(A_i) m_i x k_i.
 *   transA, transB in {'N','T'} (args 1,2). max_m/max_n/max_k >= every m_i/n_i/k_i
 *   (args 15-17; -p if < 0; batchCount is arg 14). beta == 0 does not read C. (DMMA kernel.)
 */
int vbatched_dgemm(char transA, char transB, const int* d_m, const int* d_n, const int* d_k,
                   double alpha, const double* const* dA_array, const int* d_ldda,
                   const double* const* dB_array, const int* d_lddb, double beta,
                   double* const* dC_array, const int* d_lddc, int batchCount, int max_m,
                   int max_n, int max_k, vb_stream_t stream);

/* vbatched_dsyrk: C_i = alpha A_i A_i^T + beta C_i (trans 'N', A_i n_i x k_i) or
 *   alpha A_i^T A_i + beta C_i (trans 'T', A_i k_i x n_i), only the `uplo` triangle of C_i
 *   is referenced/updated. uplo in {'L','U'} (arg 1), trans in {'N','T'} (arg 2). */
int vbatched_dsyrk(char uplo, char trans, const int* d_n, const int* d_k, double alpha,
                   const double* const* dA_array, const int* d_ldda, double beta,
                   double* const* dC_array, const int* d_lddc, int batchCount, int max_n,
                   int max_k, vb_stream_t stream);

/* vbatched_dtrsm: solve op(A_i) X = alpha B_i (side 'L') or X op(A_i) = alpha B_i (side 'R'),
 *   X overwriting B_i (m_i x n_i); A_i triangular (uplo 'L'/'U'), op = transA ('N'/'T'),
 *   diag 'N' or 'U' (unit). Cholesky uses side 'R', uplo 'L', transA 'T', diag 'N'
 *   ("C2 = C2 C1^-T"). Implemented as an in-shared-memory inversion of the
 *   diagonal blocks (TRTRI) followed by DMMA GEMMs, the design PAPER.md:760-772 describes.
 *   Every side/uplo/transA/diag combination (side 'L' runs the side-'R' kernel on the
 *   transposed view: op(A) X = alpha B <=> X^T op(A)^T = alpha B^T).
 *   A is m_i x m_i for side 'L', n_i x n_i for side 'R'. Bad side -1, uplo -2, transA -3,
 *   diag -4. */
int vbatched_dtrsm(char side, char uplo, char transA, char diag, const int* d_m, const int* d_n,
                   double alpha, const double* const* dA_array, const int* d_ldda,
                   double* const* dB_array, const int* d_lddb, int batchCount, int max_m,
                   int max_n, vb_stream_t stream);

/* vbatched_dpotrs — solve A_i X_i = B_i with the factor vbatched_dpotrf left in dA_array
 * (the paper's "factorization and solve routines", PAPER.md:183-185;
 * LAPACK DPOTRS). uplo as passed to vbatched_dpotrf: 'L' solves L Y = B then L^T X = Y,
 * 'U' solves U^T Y = B then U X = Y — two vbatched_dtrsm (side 'L') launches.
 *  d_n, d_nrhs  [batchCount] orders n_i and right-hand-side counts nrhs_i (device);
 *  dB_array     B_i: n_i x nrhs_i, column-major, leading dimension d_lddb[i] >= max(1,n_i);
 *               overwritten by X_i. A_i is only read (its referenced triangle).
 *  max_n, max_nrhs: host upper bounds. Returns uplo -1, batchCount -8, max_n -9,
 *  max_nrhs -10 (host scalars), 0 or a cudaError_t. No per-matrix info (as DPOTRS). */
int vbatched_dpotrs(char uplo, const int* d_n, const int* d_nrhs, const double* const* dA_array,
                    const int* d_ldda, double* const* dB_array, const int* d_lddb,
                    int batchCount, int max_n, int max_nrhs, vb_stream_t stream);

/* vbatched_dposv — vbatched_dpotrf followed by vbatched_dpotrs (LAPACK DPOSV): A_i is
 * overwritten by its factor, B_i by X_i; d_info as vbatched_dpotrf, and a matrix with
 * info != 0 keeps B_i unchanged. Returns uplo -1, batchCount -9, max_n -10, max_nrhs -11. */
int vbatched_dposv(char uplo, const int* d_n, const int* d_nrhs, double* const* dA_array,
                   const int* d_ldda, double* const* dB_array, const int* d_lddb, int* d_info,
                   int batchCount, int max_n, int max_nrhs, vb_stream_t stream);

/* ---------------------------------------------------------------------------------------
 * vbatched_zpotrf / vbatched_cpotrf — variable-size batched complex Cholesky A_i = L_i L_i^H
 * (uplo 'L') or U_i^H U_i (uplo 'U') of Hermitian positive definite matrices (SURVEY.md §8(f)
 * NEXT-3; the paper's framework "supports complex precisions", §IV-A;
 * LAPACK ZPOTRF / CPOTRF semantics).
 *  dA_array   [batchCount] device pointers to complex matrices, interleaved (re, im) per element,
 *             column-major: element (r,c) of matrix i is ((T*)dA_array[i])[2*(r + c*ldda[i])]
 *             (+1 for the imaginary part); T = double (Z) or float (C). Only the `uplo`
 *             triangle is referenced; the diagonal's imaginary part is ignored on input and
 *             written as 0 in the factor. 16-byte (Z) / 8-byte (C) aligned.
 *  Everything else (d_n, d_ldda in elements, d_info codes incl. -2/-4/-7 and k > 0, max_n,
 *  return codes) exactly as vbatched_dpotrf. CPOTRF stores FP32 and computes in FP64 (as
 *  vbatched_spotrf). Complex products on the FP64 tensor cores are four real DMMAs.
 */
int vbatched_zpotrf(char uplo, const int* d_n, void* const* dA_array, const int* d_ldda,
                    int* d_info, int batchCount, int max_n, vb_stream_t stream);
int vbatched_cpotrf(char uplo, const int* d_n, void* const* dA_array, const int* d_ldda,
                    int* d_info, int batchCount, int max_n, vb_stream_t stream);

/* ---------------------------------------------------------------------------------------
 * vbatched_dgetrf — FP64 variable-size batched LU with partial pivoting, A_i = P_i L_i U_i
 * (the LU extension the paper names as future work, PAPER.md:2279-2285
 * §V, built from its vbatched kernels, §III-E; LAPACK DGETRF semantics).
 *
 *  d_m, d_n     [batchCount] rows m_i and columns n_i (device). Rectangular matrices allowed.
 *  dA_array     [batchCount] device pointers; A_i is m_i x n_i column-major with leading
 *               dimension d_ldda[i] >= max(1, m_i). On return: L_i strictly below the diagonal
 *               (unit diagonal not stored), U_i on and above it. Rows m_i..ldda_i-1 untouched.
 *  dipiv_array  [batchCount] device pointers to int arrays of min(m_i, n_i) entries: row k was
 *               interchanged with row ipiv[k] (1-based, LAPACK convention), in order.
 *  d_info       [batchCount] output: 0; k > 0 = U(k,k) is exactly zero (first such k, 1-based;
 *               the factorisation is completed, as LAPACK DGETRF); -1 m_i < 0; -2 n_i < 0;
 *               -4 ldda_i < max(1, m_i); -9 m_i > max_m or n_i > max_n (matrix untouched).
 *  max_m, max_n upper bounds on every m_i / n_i (host). max_m <= 1024 (the panel rows are held
 *               in registers): larger returns -8.
 * Pivot: the first row of maximal |a_ik| (IDAMAX). Arithmetic: panel (16 columns) in registers
 * with IEEE division for the multipliers, then the library's vbatched DTRSM (side L, lower,
 * unit) and DGEMM (DMMA) on the trailing matrix, one panel step at a time (PAPER.md:724-812,
 * the separated design). Returns 0 / -p (batchCount -7, max_m -8, max_n -9) / cudaError_t.
 */
int vbatched_dgetrf(const int* d_m, const int* d_n, double* const* dA_array, const int* d_ldda,
                    int* const* dipiv_array, int* d_info, int batchCount, int max_m, int max_n,
                    vb_stream_t stream);

/* ---------------------------------------------------------------------------------------
 * vbatched_dgeqrf — FP64 variable-size batched Householder QR, A_i = Q_i R_i (SURVEY.md §8(f)
 * NEXT-4; the QR extension of PAPER.md:2279-2285, built from the library's vbatched GEMM as the
 * paper's separated design; LAPACK DGEQRF semantics).
 *  d_m, d_n     [batchCount] rows / columns (device); rectangular allowed.
 *  dA_array     [batchCount] device pointers, m_i x n_i column-major, ldda_i >= max(1, m_i). On
 *               return R_i on and above the diagonal, the Householder vectors below it (v_k has
 *               an implicit unit leading entry), Q_i = H_1 ... H_k, H_j = I - tau_j v_j v_j^T.
 *  dtau_array   [batchCount] device pointers to min(m_i, n_i) doubles: the reflector scalars.
 *  d_info       [batchCount] output: 0; -1 m_i < 0; -2 n_i < 0; -4 ldda_i < max(1, m_i); -9 m_i >
 *               max_m or n_i > max_n (matrix untouched). QR itself never fails.
 *  max_m, max_n bounds (host); max_m <= 1024 (panel rows in registers), larger returns -8.
 * Reflectors: LAPACK DLARFG conventions (beta = -sign(alpha) sqrt(alpha^2 + ||x||^2), tau =
 * (beta - alpha)/beta, v = x/(alpha - beta); ||x|| = 0 gives tau = 0). Internal workspace:
 * (64 max_m + 128 max_n + 8448) doubles per matrix from the library's pool, the batch processed
 * in slices of at most ~4 GiB of workspace.
 * Returns 0 / -p (batchCount -7, max_m -8, max_n -9) / cudaError_t.
 */
int vbatched_dgeqrf(const int* d_m, const int* d_n, double* const* dA_array, const int* d_ldda,
                    double* const* dtau_array, int* d_info, int batchCount, int max_m, int max_n,
                    vb_stream_t stream);

/* ---------------------------------------------------------------------------------------
 * Host helpers (pure host, deterministic, no CUDA).
 * vbatched_partition_lpt: flop-balanced multi-GPU sharding: longest
 *   processing time first on cost n^3/3 — sort by n descending (ties by index), assign
 *   each matrix to the least-loaded rank (ties to the lowest rank). h_owner[i] in [0,ngpu).
 *   Returns 0, or -2 (batchCount < 0), -3 (ngpu < 1). */
int vbatched_partition_lpt(const int* h_n, int batchCount, int ngpu, int* h_owner);

/* Library version string and the tuning constants compiled in (for logs). */
const char* vbatched_version(void);

/* Number of kernel launches one vbatched_dpotrf call with this max_n enqueues (the scan plus
 * one persistent kernel per non-empty size range). For benchmarks' launch accounting. */
int vbatched_dpotrf_kernel_launches(int max_n);

/* Names of the factorisation kernels one vbatched_dpotrf call with this max_n launches after
 * the scan (for benchmark logs / roofline labels). Static string, never NULL. */
const char* vbatched_dpotrf_kernel_names(int max_n);

/* Pinned host memory helpers (cudaHostAlloc / cudaFreeHost) for the _host entry point. */
void* vbatched_host_alloc(size_t bytes);
int vbatched_host_free(void* p);

/* vbatched_dpotrf_host keeps a per-device staging ring (device buffers up to workspace_bytes,
 * pinned mirrors, 3 streams) between calls. This frees the current device's ring; call it
 * outside any vbatched_dpotrf_host call. Returns 0 or a cudaError_t. */
int vbatched_release_host_staging(void);

#ifdef __cplusplus
}
#endif
#endif /* VBATCHED_H_ */
