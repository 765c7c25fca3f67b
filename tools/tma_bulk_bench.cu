// Microbenchmark (tool, not library): achieved HBM->SMEM bandwidth of 1-D TMA bulk copies
// (cp.async.bulk + mbarrier ring) as a function of the copy size and ring depth, with
// 2 CTAs/SM and no compute, vs per-thread cp.async 8-byte copies of the same bytes.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tma_bulk_bench tma_bulk_bench.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); return 1; } } while (0)

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int STAGES>
__global__ void __launch_bounds__(256) bulk_kernel(const double* src, size_t nelem, int seg_bytes,
                                                   int stage_bytes, int iters, double* sink) {
  extern __shared__ __align__(128) unsigned char sm[];
  __shared__ uint64_t full[STAGES];
  const int tid = threadIdx.x;
  if (tid == 0) {
    for (int i = 0; i < STAGES; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su32(&full[i])));
    asm volatile("fence.proxy.async.shared::cta;");
  }
  __syncthreads();
  const int nseg = stage_bytes / seg_bytes;
  size_t base = ((size_t)blockIdx.x * 7919 * stage_bytes) % (nelem * 8 - (size_t)stage_bytes * iters);
  base &= ~(size_t)1023;
  auto issue = [&](int it) {
    const int st = it % STAGES;
    if (tid < 32) {
      if (tid == 0)
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(su32(&full[st])), "r"(stage_bytes) : "memory");
      __syncwarp();
      for (int s = tid; s < nseg; s += 32) {
        const char* g = (const char*)src + base + (size_t)it * stage_bytes + (size_t)s * seg_bytes;
        unsigned char* d = sm + (size_t)st * stage_bytes + (size_t)s * seg_bytes;
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                     :: "r"(su32(d)), "l"(g), "r"(seg_bytes), "r"(su32(&full[st])) : "memory");
      }
    }
  };
  for (int p = 0; p < STAGES - 1 && p < iters; ++p) issue(p);
  double acc = 0;
  for (int it = 0; it < iters; ++it) {
    const int st = it % STAGES;
    const uint32_t par = (it / STAGES) & 1;
    asm volatile("{\n .reg .pred p;\n W_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W_%=;\n}\n"
                 :: "r"(su32(&full[st])), "r"(par) : "memory");
    acc += ((double*)(sm + (size_t)st * stage_bytes))[tid];
    __syncthreads();
    if (it + STAGES - 1 < iters) { if (tid < 32) asm volatile("fence.proxy.async.shared::cta;"); issue(it + STAGES - 1); }
  }
  if (acc == 1.2345) sink[0] = acc;
}

__global__ void __launch_bounds__(256) cpasync_kernel(const double* src, size_t nelem, int stage_bytes, int iters, double* sink) {
  extern __shared__ __align__(128) unsigned char sm[];
  const int tid = threadIdx.x;
  constexpr int STAGES = 3;
  size_t base = ((size_t)blockIdx.x * 7919 * stage_bytes) % (nelem * 8 - (size_t)stage_bytes * iters);
  base &= ~(size_t)1023;
  const int per = stage_bytes / 8 / 256;
  auto issue = [&](int it) {
    const int st = it % STAGES;
    for (int e = 0; e < per; ++e) {
      const int idx = tid + e * 256;
      const char* g = (const char*)src + base + (size_t)it * stage_bytes + (size_t)idx * 8;
      unsigned char* d = sm + (size_t)st * stage_bytes + (size_t)idx * 8;
      asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" :: "r"(su32(d)), "l"(g));
    }
    asm volatile("cp.async.commit_group;");
  };
  for (int p = 0; p < STAGES - 1; ++p) issue(p);
  double acc = 0;
  for (int it = 0; it < iters; ++it) {
    asm volatile("cp.async.wait_group 1;");
    __syncthreads();
    acc += ((double*)(sm + (size_t)(it % STAGES) * stage_bytes))[tid];
    if (it + STAGES - 1 < iters) issue(it + STAGES - 1); else asm volatile("cp.async.commit_group;");
  }
  if (acc == 1.2345) sink[0] = acc;
}

int main() {
  const size_t nelem = (size_t)8 << 30 >> 3;  // 8 GiB buffer (>> L2)
  double* src; double* sink;
  CK(cudaMalloc(&src, nelem * 8)); CK(cudaMalloc(&sink, 64));
  CK(cudaMemset(src, 0, nelem * 8));
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const int stage_bytes = 24576, iters = 400;
  for (int seg : {512, 1024, 2048, 4096, 8192, 24576}) {
    for (int ctas : {2, 3}) {
      size_t smem = 3 * stage_bytes;
      CK(cudaFuncSetAttribute(bulk_kernel<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
      bulk_kernel<3><<<sms * ctas, 256, smem>>>(src, nelem, seg, stage_bytes, 10, sink);
      CK(cudaDeviceSynchronize());
      cudaEventRecord(e0);
      bulk_kernel<3><<<sms * ctas, 256, smem>>>(src, nelem, seg, stage_bytes, iters, sink);
      cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      double bytes = (double)sms * ctas * stage_bytes * iters;
      printf("{\"kind\":\"bulk\",\"seg_bytes\":%d,\"ctas_per_sm\":%d,\"stages\":3,\"GBps\":%.1f}\n", seg, ctas, bytes / ms / 1e6);
    }
  }
  for (int ctas : {2, 3}) {
    size_t smem = 3 * stage_bytes;
    CK(cudaFuncSetAttribute(cpasync_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    cpasync_kernel<<<sms * ctas, 256, smem>>>(src, nelem, stage_bytes, 10, sink);
    CK(cudaDeviceSynchronize());
    cudaEventRecord(e0);
    cpasync_kernel<<<sms * ctas, 256, smem>>>(src, nelem, stage_bytes, iters, sink);
    cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    double bytes = (double)sms * ctas * stage_bytes * iters;
    printf("{\"kind\":\"cp.async8\",\"ctas_per_sm\":%d,\"stages\":3,\"GBps\":%.1f}\n", ctas, bytes / ms / 1e6);
  }
  return 0;
}
