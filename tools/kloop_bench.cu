// Microbenchmark (tool, not library): the left-looking panel-update k-loop in isolation —
// TMA bulk copies into a full/empty mbarrier ring + DMMA m8n8k4 — to measure the DMMA rate
// the pipeline sustains without the diagonal block / TRSM / stores. Each CTA repeatedly
// computes acc(128 x NB) -= A[r0:r0+128, 0:K] * A[j0:j0+NB, 0:K]^T for row blocks of
// synthetic column-major matrices (n = 1024, ldda = 1024) in HBM.
// Variants: NB (32/64), KC, STAGES, warp tiling (8x1: 16 x NB per warp; 4x2: 32 x NB/2).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o kloop_bench kloop_bench.cu
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); return 1; } } while (0)

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void dmma(double (&d)[2], double a, double b) {
  asm("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};" : "+d"(d[0]), "+d"(d[1]) : "d"(a), "d"(b));
}
__device__ __forceinline__ void mwait(uint64_t* b, uint32_t par) {
  asm volatile("{\n .reg .pred p;\n W_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W_%=;\n}\n" :: "r"(su32(b)), "r"(par) : "memory");
}

template <int NB, int KC, int S, int WM, int WN, int MB = 128, int MINB = 2, int PRODW = 0, int FENCE = 0>  // WM x WN warps (+1 producer)
__global__ void __launch_bounds__(32 * (WM * WN + PRODW), MINB) kloop(const double* __restrict__ base, int nmat, int n, int K,
                                                int blocks_per_cta, double* sink) {
  constexpr int LDA = MB + 4, LDB = NB + 4, NW = WM * WN;
  constexpr int RW = MB / WM, CW = NB / WN, MT = RW / 8, NTT = CW / 8;
  extern __shared__ __align__(128) unsigned char sm[];
  double (*sa)[KC][LDA] = reinterpret_cast<double (*)[KC][LDA]>(sm);
  double (*sb)[KC][LDB] = reinterpret_cast<double (*)[KC][LDB]>(sm + sizeof(double) * S * KC * LDA);
  __shared__ uint64_t full[S], empty[S];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, g = lane >> 2, q = lane & 3;
  const int wrow = (warp % WM) * RW, wcol = (warp / WM) * CW;
  if (tid == 0) {
    for (int i = 0; i < S; ++i) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su32(&full[i])));
      asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(su32(&empty[i])), "n"(NW));
    }
    asm volatile("fence.proxy.async.shared::cta;");
  }
  __syncthreads();
  const int nk = K / KC;
  const long total = (long)blocks_per_cta * nk;
  auto chunk_src = [&](long c, int& kc, const double*& M, int& r0) {
    const long blk = c / nk;
    kc = (int)(c % nk);
    const long gb = (long)blockIdx.x * blocks_per_cta + blk;
    M = base + (size_t)(gb % nmat) * n * n;
    r0 = K;  // rows below the panel
  };
  uint32_t prod = 0;
  auto produce = [&]() {
    if ((long)prod >= total) return;
    int kc; const double* M; int r0;
    chunk_src(prod, kc, M, r0);
    const int st = prod % S; const uint32_t u = prod / S;
    if (lane == 0) {
      if (u > 0) mwait(&empty[st], (u - 1) & 1);
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(su32(&full[st])), "r"(KC * (MB + NB) * 8) : "memory");
    }
    __syncwarp();
    for (int c = lane; c < 2 * KC; c += 32) {
      if (c < KC) {
        const double* g0 = M + (size_t)(kc * KC + c) * n + r0;
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                     :: "r"(su32(&sa[st][c][0])), "l"(g0), "r"(MB * 8), "r"(su32(&full[st])) : "memory");
      } else {
        const double* g1 = M + (size_t)(kc * KC + c - KC) * n + (K - NB);
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                     :: "r"(su32(&sb[st][c - KC][0])), "l"(g1), "r"(NB * 8), "r"(su32(&full[st])) : "memory");
      }
    }
    ++prod;
  };
  if (PRODW) {
    if (warp == NW) {  // dedicated producer: run the whole ring, never compute
      for (long c = 0; c < total; ++c) produce();
      return;
    }
  } else if (warp == 0) for (int i = 0; i < S - 1; ++i) produce();
  double acc[MT][NTT][2] = {};
  double keep = 0;
  for (long c = 0; c < total; ++c) {
    if (!PRODW && warp == 0) produce();
    const int st = c % S;
    mwait(&full[st], (c / S) & 1);
#pragma unroll
    for (int kk = 0; kk < KC / 4; ++kk) {
      double fa[MT], fb[NTT];
#pragma unroll
      for (int mt = 0; mt < MT; ++mt) fa[mt] = -sa[st][kk * 4 + q][wrow + mt * 8 + g];
#pragma unroll
      for (int nt = 0; nt < NTT; ++nt) fb[nt] = sb[st][kk * 4 + q][wcol + nt * 8 + g];
#pragma unroll
      for (int mt = 0; mt < MT; ++mt)
#pragma unroll
        for (int nt = 0; nt < NTT; ++nt) dmma(acc[mt][nt], fa[mt], fb[nt]);
    }
    // FENCE 1: the production kernel's per-chunk fence.proxy.async before the release (orders
    // the generic-proxy LDS reads before the async-proxy refill); FENCE 2: the same fence once
    // per two chunks, releasing both slots after it
    if (FENCE == 1) asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    if (FENCE == 2) {
      if ((c & 1) || c + 1 == total) {
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        __syncwarp();
        if (lane == 0) {
          if (c & 1) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(su32(&empty[(c - 1) % S])) : "memory");
          asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(su32(&empty[st])) : "memory");
        }
      }
    } else {
    __syncwarp();
    if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(su32(&empty[st])) : "memory");
    }
    if ((c + 1) % nk == 0) {  // end of a row block: fold acc (keeps the compiler honest)
#pragma unroll
      for (int mt = 0; mt < MT; ++mt)
#pragma unroll
        for (int nt = 0; nt < NTT; ++nt) { keep += acc[mt][nt][0] + acc[mt][nt][1]; acc[mt][nt][0] = acc[mt][nt][1] = 0; }
    }
  }
  if (keep == 1.2345) sink[0] = keep;
}

template <int NB, int KC, int S, int WM, int WN, int MB = 128, int MINB = 2, int PRODW = 0, int FENCE = 0>
int run(const double* base, int nmat, int n, int K, double* sink, int sms, int cps = 2) {
  size_t smem = sizeof(double) * S * KC * (MB + 4 + NB + 4);
  CK(cudaFuncSetAttribute(kloop<NB, KC, S, WM, WN, MB, MINB, PRODW, FENCE>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  const int ctas = cps * sms, bpc = 48 / cps;
  kloop<NB, KC, S, WM, WN, MB, MINB, PRODW, FENCE><<<ctas, 32 * (WM * WN + PRODW), smem>>>(base, nmat, n, K, 2, sink);
  CK(cudaDeviceSynchronize());
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0);
  kloop<NB, KC, S, WM, WN, MB, MINB, PRODW, FENCE><<<ctas, 32 * (WM * WN + PRODW), smem>>>(base, nmat, n, K, bpc, sink);
  cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  double flops = 2.0 * ctas * bpc * (double)MB * NB * K;
  fflush(stdout);
  printf("{\"NB\":%d,\"KC\":%d,\"S\":%d,\"warps\":\"%dx%d\",\"MB\":%d,\"K\":%d,\"cps\":%d,\"prodw\":%d,\"fence\":%d,\"smem_KB\":%.1f,\"tflops\":%.2f}\n",
         NB, KC, S, WM, WN, MB, K, cps, PRODW, FENCE, smem / 1024.0, flops / ms / 1e9);
  fflush(stdout);
  return 0;
}

int main(int argc, char** argv) {
  const int n = 1024, nmat = 160;  // 1.34 GB of matrices (>> L2)
  double* base; double* sink;
  CK(cudaMalloc(&base, sizeof(double) * (size_t)nmat * n * n)); CK(cudaMalloc(&sink, 64));
  CK(cudaMemset(base, 0, sizeof(double) * (size_t)nmat * n * n));
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int only = argc > 1 ? atoi(argv[1]) : -1;  // -1: all variants; k: only variant k (ncu)
  for (int K : {256, 512}) {
    if (only < 0 || only == 0) run<64, 16, 3, 8, 1, 128, 2, 1>(base, nmat, n, K, sink, sms, 2);
    // the production shape: MB = 64 (4 consumer warps) + producer, 3 CTAs per SM
    if (only < 0 || only == 1) run<64, 16, 2, 4, 1, 64, 3, 1>(base, nmat, n, K, sink, sms, 3);
    if (only < 0 || only == 2) run<64, 16, 3, 4, 1, 64, 3, 1>(base, nmat, n, K, sink, sms, 3);
    if (only < 0 || only == 3) run<64, 16, 4, 4, 1, 64, 3, 1>(base, nmat, n, K, sink, sms, 3);
    if (only < 0 || only == 4) run<64, 16, 2, 4, 1, 64, 4, 1>(base, nmat, n, K, sink, sms, 4);
    // larger chunks (fewer ring handshakes per flop)
    if (only < 0 || only == 5) run<64, 32, 2, 4, 1, 64, 3, 1>(base, nmat, n, K, sink, sms, 3);
    if (only < 0 || only == 6) run<64, 32, 3, 4, 1, 64, 2, 1>(base, nmat, n, K, sink, sms, 2);
    if (only < 0 || only == 7) run<64, 8, 4, 4, 1, 64, 3, 1>(base, nmat, n, K, sink, sms, 3);
    // the per-chunk proxy fence of the production kernel, and once per two chunks
    if (only < 0 || only == 8) run<64, 16, 2, 4, 1, 64, 3, 1, 1>(base, nmat, n, K, sink, sms, 3);
    if (only < 0 || only == 9) run<64, 8, 4, 4, 1, 64, 3, 1, 1>(base, nmat, n, K, sink, sms, 3);
    if (only < 0 || only == 10) run<64, 8, 4, 4, 1, 64, 3, 1, 2>(base, nmat, n, K, sink, sms, 3);
    if (only < 0 || only == 11) run<64, 16, 3, 4, 1, 64, 3, 1, 2>(base, nmat, n, K, sink, sms, 3);
    // two CTAs per SM with deeper / larger rings (the production smem budget: ring <= 73 KB)
    if (only < 0 || only == 12) run<64, 32, 2, 4, 1, 64, 2, 1>(base, nmat, n, K, sink, sms, 2);
    if (only < 0 || only == 13) run<64, 16, 4, 4, 1, 64, 2, 1>(base, nmat, n, K, sink, sms, 2);
    if (only < 0 || only == 14) run<64, 16, 2, 4, 1, 64, 2, 1>(base, nmat, n, K, sink, sms, 2);
    if (only < 0 || only == 15) run<64, 8, 8, 4, 1, 64, 2, 1>(base, nmat, n, K, sink, sms, 2);
    if (only < 0 || only == 16) run<64, 8, 6, 4, 1, 64, 3, 1>(base, nmat, n, K, sink, sms, 3);
  }
  return 0;
}
