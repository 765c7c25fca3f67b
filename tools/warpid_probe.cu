// Probe (tool): which hardware warp slot (%warpid; SMSP = %warpid % 4) each warp of each CTA gets
// when several 4-warp CTAs share an SM.
#include <cstdio>
__global__ void probe(int* out) {
  unsigned wid, smid;
  asm volatile("mov.u32 %0, %%warpid;" : "=r"(wid));
  asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
  __shared__ volatile char pad[40000];
  pad[threadIdx.x] = 0;
  if ((threadIdx.x & 31) == 0) {
    int i = blockIdx.x * 4 + threadIdx.x / 32;
    out[3 * i] = smid; out[3 * i + 1] = threadIdx.x / 32; out[3 * i + 2] = wid;
  }
  long long t = clock64(); while (clock64() - t < 200000) {}
}
int main() {
  int* d; cudaMalloc(&d, 3 * 4 * 148 * 4 * sizeof(int));
  probe<<<148 * 4, 128>>>(d);
  cudaDeviceSynchronize();
  static int h[3 * 4 * 148 * 4];
  cudaMemcpy(h, d, sizeof h, cudaMemcpyDeviceToHost);
  int match = 0, tot = 0;
  for (int i = 0; i < 148 * 4 * 4; ++i) { tot++; if (h[3 * i + 2] % 4 == h[3 * i + 1] % 4) match++; }
  printf("warps whose slot %%4 == warp index %%4: %d / %d\n", match, tot);
  for (int b = 0; b < 148 * 4; ++b)
    if (h[3 * b * 4] < 2)
      printf("cta %d sm %d: slots %d %d %d %d\n", b, h[3 * b * 4], h[3 * b * 4 + 2], h[3 * (b * 4 + 1) + 2], h[3 * (b * 4 + 2) + 2], h[3 * (b * 4 + 3) + 2]);
  return 0;
}
