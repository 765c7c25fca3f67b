// Microbenchmark (tool): is an FP32 FFMA k-loop faster than the FP64 DMMA k-loop for SPOTRF's
// trailing updates on B200? ("a real FP32 SPOTRF on FFMA ... or a measured
// argument"). Shared-memory-fed inner loops only (no global traffic), 64x64 output tiles, 128-thread
// CTAs, 4 CTAs per SM:
//   ffma_peak    8 independent FFMA chains per thread (issue ceiling of the FP32 pipe)
//   ffma_tile    register-tiled 4x8 outputs per thread, per k one LDS.128 (A) + two LDS.128 (B)
//   dmma_tile    the blocked kernel's k-loop shape: 4 warps x (16 rows x 64 cols), DMMA m8n8k4 f64
// Prints TFLOP/s (2 flops per FMA). Build:
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/ffma_bench tools/ffma_bench.cu
#include <cstdio>

__device__ __forceinline__ void dmma(double (&d)[2], double a, double b) {
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
               : "+d"(d[0]), "+d"(d[1]) : "d"(a), "d"(b));
}

__global__ void __launch_bounds__(128, 4) ffma_peak(float* out, int iters) {
  float a[8];
  for (int i = 0; i < 8; ++i) a[i] = threadIdx.x * 0.001f + i;
  const float b = 1.000001f, c = 0.999999f;
  for (int it = 0; it < iters; ++it)
#pragma unroll
    for (int i = 0; i < 8; ++i) a[i] = fmaf(a[i], b, c);
  float s = 0;
  for (int i = 0; i < 8; ++i) s += a[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

// 64x64 tile, k-slab of 64 in smem (A[k][64 rows], B[k][64 cols]); thread t: rows 4*(t%16).., cols 8*(t/16)..
__global__ void __launch_bounds__(128, 4) ffma_tile(float* out, int iters) {
  __shared__ __align__(16) float A[64][64], B[64][64];
  for (int e = threadIdx.x; e < 64 * 64; e += 128) {
    A[e / 64][e % 64] = 1e-3f * (e % 7);
    B[e / 64][e % 64] = 1e-3f * (e % 5);
  }
  __syncthreads();
  const int r0 = 4 * (threadIdx.x % 16), c0 = 8 * (threadIdx.x / 16);
  float acc[4][8] = {};
  for (int it = 0; it < iters; ++it) {
#pragma unroll 4
    for (int k = 0; k < 64; ++k) {
      const float4 a = *reinterpret_cast<const float4*>(&A[k][r0]);
      const float4 b0 = *reinterpret_cast<const float4*>(&B[k][c0]);
      const float4 b1 = *reinterpret_cast<const float4*>(&B[k][c0 + 4]);
      const float av[4] = {a.x, a.y, a.z, a.w};
      const float bv[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[i][j] = fmaf(av[i], bv[j], acc[i][j]);
    }
  }
  float s = 0;
  for (int i = 0; i < 4; ++i)
    for (int j = 0; j < 8; ++j) s += acc[i][j];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__global__ void __launch_bounds__(128, 4) dmma_tile(double* out, int iters) {
  __shared__ double A[16][68], B[16][68];
  for (int e = threadIdx.x; e < 16 * 64; e += 128) {
    A[e / 64][e % 64] = 1e-3 * (e % 7);
    B[e / 64][e % 64] = 1e-3 * (e % 5);
  }
  __syncthreads();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, g = lane >> 2, q = lane & 3;
  double acc[2][8][2] = {};
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int kk = 0; kk < 4; ++kk) {
      double fa[2], fb[8];
#pragma unroll
      for (int mt = 0; mt < 2; ++mt) fa[mt] = A[kk * 4 + q][warp * 16 + mt * 8 + g];
#pragma unroll
      for (int nt = 0; nt < 8; ++nt) fb[nt] = B[kk * 4 + q][nt * 8 + g];
#pragma unroll
      for (int mt = 0; mt < 2; ++mt)
#pragma unroll
        for (int nt = 0; nt < 8; ++nt) dmma(acc[mt][nt], fa[mt], fb[nt]);
    }
  }
  double s = 0;
  for (int mt = 0; mt < 2; ++mt)
    for (int nt = 0; nt < 8; ++nt) s += acc[mt][nt][0] + acc[mt][nt][1];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

// The SPOTRF blocked kernel's FFMA shape (potrf.cu k_loop_ffma): warp w owns rows 16w..16w+15 x
// 64 columns, lane (rg, cg) rows 16w + 4 rg .. +3, columns 4 cg .. +3 and 32 + 4 cg .. +3.
// MAP 0: rg = lane / 8, cg = lane % 8; MAP 1: rg = lane % 4, cg = lane / 4.
template <int MAP>
__global__ void __launch_bounds__(128) ffma_tile16(float* out, int iters) {
  __shared__ __align__(16) float A[16][64], B[16][64];
  for (int e = threadIdx.x; e < 16 * 64; e += 128) {
    A[e / 64][e % 64] = 1e-3f * (e % 7);
    B[e / 64][e % 64] = 1e-3f * (e % 5);
  }
  __syncthreads();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int rg = MAP ? (lane & 3) : (lane >> 3), cg = MAP ? (lane >> 2) : (lane & 7);
  const int r0 = warp * 16 + rg * 4;
  float acc[4][8] = {};
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int k = 0; k < 16; ++k) {
      const float4 a = *reinterpret_cast<const float4*>(&A[k][r0]);
      const float4 b0 = *reinterpret_cast<const float4*>(&B[k][cg * 4]);
      const float4 b1 = *reinterpret_cast<const float4*>(&B[k][32 + cg * 4]);
      const float av[4] = {a.x, a.y, a.z, a.w};
      const float bv[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[i][j] = fmaf(-av[i], bv[j], acc[i][j]);
    }
  }
  float s = 0;
  for (int i = 0; i < 4; ++i)
    for (int j = 0; j < 8; ++j) s += acc[i][j];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int grid = sms * 4;
  float* fo;
  double* dout;
  cudaMalloc(&fo, sizeof(float) * grid * 128);
  cudaMalloc(&dout, sizeof(double) * grid * 128);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  auto run = [&](const char* name, auto launch, double flops) {
    launch();
    cudaDeviceSynchronize();
    cudaEventRecord(e0);
    launch();
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    printf("{\"kernel\":\"%s\",\"tflops\":%.2f,\"ms\":%.3f}\n", name, flops / (ms * 1e-3) / 1e12, ms);
  };
  const int it1 = 20000, it2 = 400, it3 = 2000;
  run("ffma_peak (8 chains/thread, 4 CTAs x 128 thr per SM)",
      [&] { ffma_peak<<<grid, 128>>>(fo, it1); }, 2.0 * grid * 128 * 8 * (double)it1);
  run("ffma_tile (64x64 tile, 4x8 per thread, LDS.128 operands)",
      [&] { ffma_tile<<<grid, 128>>>(fo, it2); }, 2.0 * grid * 64.0 * 64 * 64 * it2);
  for (int cps = 3; cps <= 4; ++cps) {
    char nm[160];
    snprintf(nm, sizeof nm, "ffma_tile16 MAP0 (SPOTRF kernel shape, 16x64 per warp, %d CTAs/SM)", cps);
    run(nm, [&] { ffma_tile16<0><<<sms * cps, 128>>>(fo, it2 * 4); }, 2.0 * sms * cps * 64.0 * 64 * 16 * it2 * 4);
    snprintf(nm, sizeof nm, "ffma_tile16 MAP1 (SPOTRF kernel shape, 16x64 per warp, %d CTAs/SM)", cps);
    run(nm, [&] { ffma_tile16<1><<<sms * cps, 128>>>(fo, it2 * 4); }, 2.0 * sms * cps * 64.0 * 64 * 16 * it2 * 4);
  }
  run("dmma_tile (blocked-kernel k-loop shape, 16x64 per warp)",
      [&] { dmma_tile<<<grid, 128>>>(dout, it3); }, 2.0 * grid * 64.0 * 64 * 16 * it3);
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
