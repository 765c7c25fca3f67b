// vbgen device twin: fills a vbatched arena with the F1 family (see vbgen/__init__.py).
// Holds none of the method's arithmetic; integer hash + one double add per diagonal entry,
// bit-identical to the numpy version (pinned by tests/test_generator.py).
//
// Exported (C ABI, libvbgen.so):
//   int vbgen_fill_f1(uint64_t seed, int batch, const int* d_n, const int* d_ldda,
//                     double* const* d_A, const int* d_gidx, int nonspd_mod, int poison,
//                     cudaStream_t stream)
//     d_n/d_ldda/d_A/d_gidx: device arrays of length batch (d_gidx may be NULL -> gidx = i).
//     Writes the lower triangle (and, if poison bit 0 is set, NaN-payload sentinels into the
//     strict upper triangle and the padding rows n..ldda-1). Poison bit 1 selects upper
//     storage instead (the same symmetric matrix in the upper triangle, for uplo 'U'; the
//     sentinels then go to the strict lower triangle). Poison bit 2: the matrices are FP32
//     (d_A holds float*; each value is the F1 double rounded to nearest float, the poison
//     becomes a float NaN with a payload). Returns a cudaError_t.
#include <cstdint>
#include <cuda_runtime.h>

namespace {

__device__ __forceinline__ uint64_t splitmix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

constexpr uint64_t kPoison = 0x7FF8DEADBEEF0001ull;

// One CTA per matrix (grid-stride over matrices); threads stride over columns' rows.
__global__ void fill_f1_kernel(uint64_t seed, int batch, const int* __restrict__ d_n,
                               const int* __restrict__ d_ldda, double* const* __restrict__ d_A,
                               const int* __restrict__ d_gidx, int nonspd_mod, int poison) {
  const uint64_t s0 = splitmix64(seed);
  for (int b = blockIdx.x; b < batch; b += gridDim.x) {
    const int n = d_n[b];
    if (n <= 0) continue;
    const int ld = d_ldda[b];
    const uint64_t g = d_gidx ? (uint64_t)d_gidx[b] : (uint64_t)b;
    double* A = d_A[b];
    int kneg = -1;
    if (nonspd_mod > 0 && (int)(g % (uint64_t)nonspd_mod) == nonspd_mod - 1)
      kneg = (int)(splitmix64(s0 ^ g ^ 0x5EEDull) % (uint64_t)n);
    const bool up = (poison & 2) != 0, poi = (poison & 1) != 0, f32 = (poison & 4) != 0;
    const int rows = poi ? ld : n;
    for (int j = 0; j < n; ++j) {
      double* col = A + (size_t)j * ld;
      float* colf = reinterpret_cast<float*>(A) + (size_t)j * ld;
      const int i0 = (poi || up) ? 0 : j, i1 = (up && !poi) ? j + 1 : rows;
      for (int i = i0 + threadIdx.x; i < i1; i += blockDim.x) {
        double v;
        if (up ? (i <= j) : (i >= j && i < n)) {
          const int r = i > j ? i : j, c = i > j ? j : i;
          const uint64_t key = (g << 42) ^ ((uint64_t)r << 21) ^ (uint64_t)c;
          v = (double)(splitmix64(s0 ^ key) >> 11) * 0x1.0p-53;
          if (i == j) {
            v = v + (double)n;
            if (i == kneg) v = -v;
          }
        } else {
          v = __longlong_as_double((long long)kPoison);
        }
        if (f32)
          colf[i] = v == v ? (float)v : __int_as_float(0x7FC0BEEF);
        else
          col[i] = v;
      }
    }
  }
}

}  // namespace

extern "C" int vbgen_fill_f1(uint64_t seed, int batch, const int* d_n, const int* d_ldda,
                             double* const* d_A, const int* d_gidx, int nonspd_mod, int poison,
                             cudaStream_t stream) {
  if (batch <= 0) return 0;
  int grid = batch < 148 * 16 ? batch : 148 * 16;
  fill_f1_kernel<<<grid, 256, 0, stream>>>(seed, batch, d_n, d_ldda, d_A, d_gidx, nonspd_mod,
                                           poison);
  return (int)cudaGetLastError();
}
