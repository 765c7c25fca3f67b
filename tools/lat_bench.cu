// Microbenchmark (tool): dependent-chain latencies of the operations on the POTF2 pivot chain
// (DFMA, MUFU.RCP64H, rcp + Newton, shfl of a double, STS -> syncwarp -> LDS) and of the
// per-warp POTF2 routines of potrf.cu. One warp per SM, clock64 around 64-long chains.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include -o tools/lat_bench tools/lat_bench.cu
#include "../paper_conf_ipps_abdelfattahhtd16_b200/csrc/potrf.cu"
#include <cstdio>

using namespace vb;

constexpr int CH = 64;

__global__ void lat_kernel(double* out, long long* cyc, double seed) {
  __shared__ double buf[2][32];
  __shared__ double T[32 * 36];
  __shared__ double ws[64], sv[32], tv[32];
  const int lane = threadIdx.x;
  double x = seed + lane * 1e-3;
  long long t0, t1;
  // 0: DFMA chain
  t0 = clock64();
#pragma unroll 1
  for (int it = 0; it < CH; ++it)
#pragma unroll
  for (int i = 0; i < 8; ++i) asm volatile("fma.rn.f64 %0, %0, %1, %2;" : "+d"(x) : "d"(0.999999), "d"(1e-9));
  t1 = clock64();
  if (lane == 0) cyc[0] = (t1 - t0);
  // 1: MUFU.RCP64H chain
  t0 = clock64();
#pragma unroll 1
  for (int it = 0; it < CH; ++it)
#pragma unroll
  for (int i = 0; i < 8; ++i) asm volatile("rcp.approx.ftz.f64 %0, %0;" : "+d"(x));
  t1 = clock64();
  if (lane == 0) cyc[1] = (t1 - t0);
  // 2: rcp_nr chain
  x = 1.5 + lane;
  t0 = clock64();
#pragma unroll 1
  for (int it = 0; it < CH; ++it)
#pragma unroll
  for (int i = 0; i < 8; ++i) { x = rcp_nr(x); asm volatile("" : "+d"(x)); }
  t1 = clock64();
  if (lane == 0) cyc[2] = (t1 - t0);
  // 3: shfl of a double (from a varying lane)
  t0 = clock64();
#pragma unroll 1
  for (int it = 0; it < CH; ++it)
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    int lo, hi;
    asm volatile("mov.b64 {%0,%1}, %2;" : "=r"(lo), "=r"(hi) : "d"(x));
    asm volatile("shfl.sync.idx.b32 %0, %0, %1, 31, -1;" : "+r"(lo) : "r"(i & 31));
    asm volatile("shfl.sync.idx.b32 %0, %0, %1, 31, -1;" : "+r"(hi) : "r"(i & 31));
    asm volatile("mov.b64 %0, {%1,%2};" : "=d"(x) : "r"(lo), "r"(hi));
  }
  t1 = clock64();
  if (lane == 0) cyc[3] = (t1 - t0);
  // 4: STS -> __syncwarp -> LDS (other lane's value) chain
  t0 = clock64();
#pragma unroll 1
  for (int it = 0; it < CH; ++it)
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    asm volatile("st.shared.f64 [%0], %1;" :: "r"(smem_u32(&buf[i & 1][lane])), "d"(x) : "memory");
    __syncwarp();
    asm volatile("ld.shared.f64 %0, [%1];" : "=d"(x) : "r"(smem_u32(&buf[i & 1][(lane + 1) & 31])) : "memory");
  }
  t1 = clock64();
  if (lane == 0) cyc[4] = (t1 - t0);
  // 5: IEEE sqrt chain
  x = 2.0 + lane;
  t0 = clock64();
#pragma unroll 1
  for (int it = 0; it < CH; ++it)
#pragma unroll
  for (int i = 0; i < 8; ++i) { asm volatile("sqrt.rn.f64 %0, %0;" : "+d"(x)); asm volatile("add.rn.f64 %0, %0, 1.0;" : "+d"(x)); }
  t1 = clock64();
  if (lane == 0) cyc[5] = (t1 - t0);
  // 6: DMMA chain (accumulator dependence)
  double acc[2] = {x, x};
  t0 = clock64();
#pragma unroll 1
  for (int it = 0; it < CH; ++it)
#pragma unroll
  for (int i = 0; i < 8; ++i) asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};" : "+d"(acc[0]), "+d"(acc[1]) : "d"(1e-3), "d"(1e-3));
  t1 = clock64();
  if (lane == 0) cyc[6] = (t1 - t0);
  x += acc[0] + acc[1];
  // 7: potf2_regs_warp<16> (nb = 16), rows in registers
  for (int c = 0; c < 32; ++c) T[c * 36 + lane] = (c == lane) ? 40.0 + lane : 0.25 / (1 + ((lane * 7 + c * 3) % 5));
  __syncwarp();
  {
    double a[16];
#pragma unroll
    for (int c = 0; c < 16; ++c) a[c] = T[c * 36 + lane];
    __syncwarp();
    t0 = clock64();
    int info = potf2_regs_warp<16>(a, 16, lane, ws, sv, tv);
    __syncwarp();
    t1 = clock64();
    double s = info;
#pragma unroll
    for (int c = 0; c < 16; ++c) s += a[c];
    x += s;
    if (lane == 0) cyc[7] = (t1 - t0);
  }
  // 8: potf2_regs_warp<32> (nb = 32)
  {
    double a[32];
#pragma unroll
    for (int c = 0; c < 32; ++c) a[c] = T[c * 36 + lane];
    __syncwarp();
    t0 = clock64();
    int info = potf2_regs_warp<32>(a, 32, lane, ws, sv, tv);
    __syncwarp();
    t1 = clock64();
    double s = info;
#pragma unroll
    for (int c = 0; c < 32; ++c) s += a[c];
    x += s;
    if (lane == 0) cyc[8] = (t1 - t0);
  }
  // 9: potf2_block32 (16 + DMMA SYRK + 16, with smem and global stores)
  {
    __syncwarp();
    t0 = clock64();
    int info = potf2_block32(T, 36, 32, lane, out + 64, 32, ws, sv, tv);
    __syncwarp();
    t1 = clock64();
    x += info;
    if (lane == 0) cyc[9] = (t1 - t0);
  }
  out[lane] = x;
}

int main() {
  double* out;
  long long* cyc;
  cudaMalloc(&out, 8 * 4096);
  cudaMalloc(&cyc, 8 * 64);
  const char* names[] = {"dfma", "mufu_rcp64h", "rcp_nr", "shfl_f64", "sts_sync_lds", "sqrt_ieee+add",
                         "dmma_acc_chain", "potf2_regs16", "potf2_regs32", "potf2_block32"};
  const int per[] = {8 * CH, 8 * CH, 8 * CH, 8 * CH, 8 * CH, 8 * CH, 8 * CH, 1, 1, 1, 1, 1};
  for (int rep = 0; rep < 2; ++rep) {
    lat_kernel<<<1, 32>>>(out, cyc, 1.0);
    cudaDeviceSynchronize();
  }
  long long h[16];
  cudaMemcpy(h, cyc, sizeof h, cudaMemcpyDeviceToHost);
  for (int i = 0; i < 10; ++i)
    printf("{\"op\":\"%s\",\"cycles\":%.1f}\n", names[i], (double)h[i] / per[i]);
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
