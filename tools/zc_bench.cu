// Microbenchmark (tool): host<->device bandwidth of the copy engines vs GPU-initiated zero-copy
// access to pinned host memory (the two transfer modes of vbatched_dpotrf_host). 2 GiB buffers.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/zc_bench tools/zc_bench.cu
#include <cstdio>
#include <cuda_runtime.h>

template <int VEC, int UNROLL, int MODE>  // MODE 0: ldcv, 1: ldcg, 2: ld (default)
__global__ void zc_read(const double* __restrict__ h, double* __restrict__ d, size_t n) {
  using V = typename std::conditional<VEC == 2, double2, double>::type;
  const V* hv = reinterpret_cast<const V*>(h);
  V* dv = reinterpret_cast<V*>(d);
  const size_t nv = n / VEC, stride = (size_t)gridDim.x * blockDim.x;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < nv; i += stride * UNROLL) {
    V v[UNROLL];
#pragma unroll
    for (int u = 0; u < UNROLL; ++u) {
      const size_t k = i + u * stride;
      if (k < nv) v[u] = MODE == 0 ? __ldcv(hv + k) : MODE == 1 ? __ldcg(hv + k) : hv[k];
    }
#pragma unroll
    for (int u = 0; u < UNROLL; ++u) {
      const size_t k = i + u * stride;
      if (k < nv) dv[k] = v[u];
    }
  }
}

__global__ void zc_write(double2* __restrict__ h, const double2* __restrict__ d, size_t nv) {
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < nv; i += stride) h[i] = d[i];
}

int main() {
  const size_t bytes = 2ull << 30, n = bytes / 8;
  double *h, *d;
  cudaHostAlloc(&h, bytes, cudaHostAllocDefault);
  cudaMalloc(&d, bytes);
  for (size_t i = 0; i < n; i += 512) h[i] = 1.0;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  auto rep = [&](const char* name, auto f) {
    f();
    cudaDeviceSynchronize();
    cudaEventRecord(e0);
    f();
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    printf("{\"op\":\"%s\",\"GBps\":%.1f,\"err\":\"%s\"}\n", name, bytes / ms / 1e6,
           cudaGetErrorString(cudaGetLastError()));
    fflush(stdout);
  };
  rep("memcpy H2D (copy engine)", [&] { cudaMemcpyAsync(d, h, bytes, cudaMemcpyHostToDevice); });
  rep("memcpy D2H (copy engine)", [&] { cudaMemcpyAsync(h, d, bytes, cudaMemcpyDeviceToHost); });
  {  // both directions at once on two streams (H2D of one buffer, D2H of another)
    double *h2, *d2;
    cudaHostAlloc(&h2, bytes, cudaHostAllocDefault);
    cudaMalloc(&d2, bytes);
    cudaStream_t s1, s2;
    cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking);
    cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);
    for (int it = 0; it < 2; ++it) {
      cudaDeviceSynchronize();
      cudaEventRecord(e0);
      cudaEventRecord(e0, 0);
      cudaStreamWaitEvent(s1, e0, 0);
      cudaStreamWaitEvent(s2, e0, 0);
      cudaMemcpyAsync(d, h, bytes, cudaMemcpyHostToDevice, s1);
      cudaMemcpyAsync(h2, d2, bytes, cudaMemcpyDeviceToHost, s2);
      cudaEvent_t a, b;
      cudaEventCreate(&a);
      cudaEventCreate(&b);
      cudaEventRecord(a, s1);
      cudaEventRecord(b, s2);
      cudaStreamWaitEvent(0, a, 0);
      cudaStreamWaitEvent(0, b, 0);
      cudaEventRecord(e1, 0);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      if (it) printf("{\"op\":\"memcpy H2D + D2H concurrently (copy engines)\",\"GBps_each\":%.1f,\"GBps_total\":%.1f}\n",
                     bytes / ms / 1e6, 2 * bytes / ms / 1e6);
    }
    fflush(stdout);
  }
  for (size_t w : {1024, 2048, 4096, 6144}) {  // 2-D copies: rows of w bytes at an 8 KiB pitch
    char name[96];
    snprintf(name, sizeof name, "memcpy2D H2D width %zu B pitch 8192 B (GB/s of payload)", w);
    const size_t rows = bytes / 8192;
    cudaDeviceSynchronize();
    cudaEventRecord(e0);
    cudaMemcpy2DAsync(d, 8192, h, 8192, w, rows, cudaMemcpyHostToDevice);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    printf("{\"op\":\"%s\",\"GBps\":%.1f}\n", name, rows * w / ms / 1e6);
    fflush(stdout);
  }
  rep("kernel read 8B ldcv x4, 2x128/SM", [&] { zc_read<1, 4, 0><<<2 * sms, 128>>>(h, d, n); });
  rep("kernel read 16B ldcv x4, 2x128/SM", [&] { zc_read<2, 4, 0><<<2 * sms, 128>>>(h, d, n); });
  rep("kernel read 16B ldcg x4, 2x128/SM", [&] { zc_read<2, 4, 1><<<2 * sms, 128>>>(h, d, n); });
  rep("kernel read 16B ld x8, 4x256/SM", [&] { zc_read<2, 8, 2><<<4 * sms, 256>>>(h, d, n); });
  rep("kernel read 16B ldcg x8, 8x512/SM", [&] { zc_read<2, 8, 1><<<8 * sms, 512>>>(h, d, n); });
  rep("kernel write 16B, 4x256/SM", [&] { zc_write<<<4 * sms, 256>>>((double2*)h, (double2*)d, n / 2); });
  return 0;
}
