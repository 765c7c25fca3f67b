// Probe (tool): which hardware warp slot (%warpid; SMSP = %warpid % 4) each warp of each CTA gets
// when several 4-warp CTAs share an SM.
#include <cstdio>
__global__ void probe(int* out, int wpc) {
  unsigned wid, smid;
  asm volatile("mov.u32 %0, %%warpid;" : "=r"(wid));
  asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
  __shared__ volatile char pad[45000];
  pad[threadIdx.x] = 0;
  if ((threadIdx.x & 31) == 0) {
    int i = blockIdx.x * 8 + threadIdx.x / 32;
    out[3 * i] = smid; out[3 * i + 1] = threadIdx.x / 32; out[3 * i + 2] = wid;
  }
  long long t = clock64(); while (clock64() - t < 200000) {}
}
int main() {
  int* d; cudaMalloc(&d, 3 * 8 * 148 * 8 * sizeof(int));
  static int h[3 * 8 * 148 * 8];
  for (int wpc : {4, 5}) {
    const int ctas = wpc == 4 ? 4 : 3;
    cudaMemset(d, 0xff, sizeof h);
    probe<<<148 * ctas, 32 * wpc>>>(d, wpc);
    cudaDeviceSynchronize();
    cudaMemcpy(h, d, sizeof h, cudaMemcpyDeviceToHost);
    printf("== %d-warp CTAs, %d per SM\n", wpc, ctas);
    for (int b = 0; b < 148 * ctas; ++b)
      if (h[3 * b * 8] == 0) {
        printf("cta %d sm %d: slot%%4 of warps:", b, h[3 * b * 8]);
        for (int w = 0; w < wpc; ++w) printf(" %d", h[3 * (b * 8 + w) + 2] % 4);
        printf("  (slots");
        for (int w = 0; w < wpc; ++w) printf(" %d", h[3 * (b * 8 + w) + 2]);
        printf(")\n");
      }
  }
  return 0;
}
