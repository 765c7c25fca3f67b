/* lapack_batch.c — CPU library baseline for bench.py (NOT the product, NOT the oracle).
 *
 * The paper's best CPU competitor is "MKL, one core per matrix" (PAPER.md:1705-1713,
 * 1857-1867): each matrix factored by a sequential LAPACK dpotrf, the matrices spread over all
 * cores. This file runs exactly that on the bench host: `nthreads` pthreads pull matrix
 * indices from an atomic counter (the caller passes them in LPT order) and call the LAPACK
 * `dpotrf_` resolved at run time from an already-loaded library (MKL inside libtorch_cpu.so,
 * or OpenBLAS), with MKL's per-thread thread count forced to 1 when that symbol exists; scipy's
 * bundled OpenBLAS (LP64, `scipy_dpotrf_`) with its global thread count set to 1.
 * Plain pointers, no torch types; nothing here is used by libvbatched or by the oracle.
 */
#define _GNU_SOURCE
#include <dlfcn.h>
#include <pthread.h>
#include <stdatomic.h>
#include <stddef.h>

typedef void (*dpotrf_fn)(const char* uplo, const int* n, double* a, const int* lda, int* info);
typedef int (*set_local_fn)(int);

struct job {
  dpotrf_fn potrf;
  set_local_fn set_local;
  double* const* A;
  const int* n;
  const int* ld;
  int* info;
  const int* order;
  int count;
  atomic_int next;
};

static void* worker(void* p) {
  struct job* j = (struct job*)p;
  if (j->set_local) j->set_local(1);
  for (;;) {
    const int k = atomic_fetch_add(&j->next, 1);
    if (k >= j->count) break;
    const int m = j->order ? j->order[k] : k;
    int info = 0;
    if (j->n[m] > 0) j->potrf("L", &j->n[m], j->A[m], &j->ld[m], &info);
    j->info[m] = info;
  }
  return NULL;
}

/* Returns 0 on success, -1 if `dpotrf_` cannot be resolved from `lib_path` (NULL = the global
 * symbol namespace), -2 on thread-creation failure. */
int lapack_batch_dpotrf(const char* lib_path, double* const* A, const int* n, const int* ld,
                        int* info, const int* order, int count, int nthreads) {
  void* h = lib_path ? dlopen(lib_path, RTLD_NOW | RTLD_GLOBAL) : RTLD_DEFAULT;
  if (!h) return -1;
  struct job j;
  j.potrf = (dpotrf_fn)dlsym(h, "dpotrf_");
  j.set_local = (set_local_fn)dlsym(h, "MKL_Set_Num_Threads_Local");
  if (!j.potrf) {  // scipy's bundled OpenBLAS (LP64): prefixed symbols, a global thread count
    j.potrf = (dpotrf_fn)dlsym(h, "scipy_dpotrf_");
    void (*set_global)(int) = (void (*)(int))dlsym(h, "scipy_openblas_set_num_threads");
    if (set_global) set_global(1);  /* one thread per dpotrf call; the workers give parallelism */
  }
  if (!j.potrf) return -1;
  j.A = A;
  j.n = n;
  j.ld = ld;
  j.info = info;
  j.order = order;
  j.count = count;
  atomic_init(&j.next, 0);
  if (nthreads < 1) nthreads = 1;
  if (nthreads > 1024) nthreads = 1024;
  pthread_t th[1024];
  int started = 0;
  for (; started < nthreads; ++started)
    if (pthread_create(&th[started], NULL, worker, &j) != 0) break;
  if (started == 0) return -2;
  for (int t = 0; t < started; ++t) pthread_join(th[t], NULL);
  return 0;
}

/* 1 if the library exposes MKL (the per-thread thread-count control), else 0. */
int lapack_batch_is_mkl(const char* lib_path) {
  void* h = lib_path ? dlopen(lib_path, RTLD_NOW | RTLD_GLOBAL) : RTLD_DEFAULT;
  return h && dlsym(h, "MKL_Set_Num_Threads_Local") ? 1 : 0;
}
