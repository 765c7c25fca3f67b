// host_stream.cu — vbatched_dpotrf_host: end-to-end factorisation of a batch that lives in
// HOST memory (include/vbatched.h). A native pipelined runtime: the batch is cut into
// chunks that fit a device staging ring of kBufs buffers; chunk c uses buffer c % kBufs and
// its own stream, so the H2D copy of chunk c+1, the factorisation of chunk c and the D2H copy
// of chunk c-1 overlap (two copy engines + compute). Contiguous host matrices are moved with
// one cudaMemcpyAsync per run. Every arithmetic step runs in the same CUDA kernels as
// vbatched_dpotrf (scan_bin + the persistent factorisation kernel).
#include <algorithm>
#include <cstdint>
#include <cstring>
#include <mutex>
#include <vector>

#include "../../include/vbatched.h"
#include "common.cuh"
#include "internal.h"

namespace vb {
namespace {

constexpr int kBufs = 3;

struct Run {            // a maximal run of host-contiguous matrices
  const double* host;   // host start
  size_t dev_off;       // byte offset in the device buffer
  size_t bytes;
};

struct Chunk {
  std::vector<int> idx;  // matrices (global indices) in this chunk
  std::vector<Run> runs;
  std::vector<size_t> dev_off;  // per matrix byte offset in the buffer
};

struct Slot {
  cudaStream_t stream = nullptr;
  cudaEvent_t done = nullptr;
  size_t dbuf_bytes = 0;
  char* dbuf = nullptr;     // matrices
  int* dmeta = nullptr;     // n[cap], ldda[cap], info[cap]
  double** dptr = nullptr;  // pointer array [cap]
  int* hmeta = nullptr;     // pinned mirror of dmeta
  double** hptr = nullptr;  // pinned mirror of dptr
  int cap = 0;
  int chunk = -1;           // chunk whose results are in flight
};

struct StageCache {
  Slot slots[kBufs];
};
constexpr int kMaxDevices = 64;
StageCache g_stage[kMaxDevices];
std::mutex g_stage_mutex;

}  // namespace
}  // namespace vb

using namespace vb;

extern "C" int vbatched_dpotrf_host(char uplo, const int* h_n, double* const* hA,
                                    const int* h_ldda, int* h_info, int batch, int max_n,
                                    size_t workspace_bytes, vb_stream_t user_stream) {
  if (uplo != 'L' && uplo != 'l' && uplo != 'U' && uplo != 'u') return -1;
  if (batch < 0) return -6;
  if (max_n < 0) return -7;
  if (batch == 0) return 0;
  if (workspace_bytes == 0) workspace_bytes = 6ull << 30;
  const size_t buf_bytes = (workspace_bytes / kBufs) & ~(size_t)255;

  // ---- host planning: validate (LAPACK codes), cut into chunks of <= buf_bytes
  std::vector<Chunk> chunks;
  Chunk cur;
  size_t cur_bytes = 0;
  int max_cnt = 0;
  const double* run_end = nullptr;
  auto flush = [&]() {
    if (!cur.idx.empty()) {
      max_cnt = std::max(max_cnt, (int)cur.idx.size());
      chunks.push_back(std::move(cur));
    }
    cur = Chunk();
    cur_bytes = 0;
    run_end = nullptr;
  };
  for (int i = 0; i < batch; ++i) {
    const int n = h_n[i], ld = h_ldda[i];
    if (n < 0) { h_info[i] = -2; continue; }
    if (ld < std::max(1, n)) { h_info[i] = -4; continue; }
    if (n > max_n) { h_info[i] = -7; continue; }
    h_info[i] = 0;
    if (n == 0) continue;
    const size_t bytes = (size_t)ld * (size_t)n * sizeof(double);
    if (bytes > buf_bytes) return -9;
    const bool contiguous = (run_end == hA[i]);
    size_t off = contiguous ? cur_bytes : ((cur_bytes + 255) & ~(size_t)255);
    if (off + bytes > buf_bytes) {
      flush();
      off = 0;
    }
    if (run_end == hA[i] && !cur.runs.empty()) {
      cur.runs.back().bytes += bytes;
    } else {
      cur.runs.push_back(Run{hA[i], off, bytes});
    }
    cur.idx.push_back(i);
    cur.dev_off.push_back(off);
    cur_bytes = off + bytes;
    run_end = hA[i] + (size_t)ld * n;
  }
  flush();
  if (chunks.empty()) return 0;

  // ---- device/pinned resources: a per-process staging cache (grown on demand, reused by
  // later calls on the same device; one caller at a time)
  std::lock_guard<std::mutex> lock(g_stage_mutex);
  cudaError_t e = cudaSuccess;
  int dev = 0;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return (int)e;
  if (dev < 0 || dev >= kMaxDevices) return (int)cudaErrorInvalidDevice;
  Slot* slots = g_stage[dev].slots;
  const int nslots = std::min<int>(kBufs, (int)chunks.size());
  size_t need = 0;
  for (const Chunk& c : chunks) need = std::max(need, c.runs.back().dev_off + c.runs.back().bytes);
  cudaEvent_t start_ev = nullptr;
  e = cudaEventCreateWithFlags(&start_ev, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaEventRecord(start_ev, (cudaStream_t)user_stream);
  for (int s = 0; s < nslots && e == cudaSuccess; ++s) {
    Slot& sl = slots[s];
    sl.chunk = -1;
    if (!sl.stream && (e = cudaStreamCreateWithFlags(&sl.stream, cudaStreamNonBlocking)) != cudaSuccess) break;
    if ((e = cudaStreamWaitEvent(sl.stream, start_ev, 0)) != cudaSuccess) break;
    if (!sl.done && (e = cudaEventCreateWithFlags(&sl.done, cudaEventDisableTiming)) != cudaSuccess) break;
    if (sl.dbuf_bytes < need) {
      if (sl.dbuf) cudaFree(sl.dbuf);
      sl.dbuf = nullptr;
      sl.dbuf_bytes = 0;
      if ((e = cudaMalloc(&sl.dbuf, need)) != cudaSuccess) break;
      sl.dbuf_bytes = need;
    }
    if (sl.cap < max_cnt) {
      if (sl.dmeta) cudaFree(sl.dmeta);
      if (sl.dptr) cudaFree(sl.dptr);
      if (sl.hmeta) cudaFreeHost(sl.hmeta);
      if (sl.hptr) cudaFreeHost(sl.hptr);
      sl.dmeta = nullptr; sl.dptr = nullptr; sl.hmeta = nullptr; sl.hptr = nullptr;
      sl.cap = 0;
      if ((e = cudaMalloc(&sl.dmeta, sizeof(int) * 3 * (size_t)max_cnt)) != cudaSuccess) break;
      if ((e = cudaMalloc(&sl.dptr, sizeof(double*) * (size_t)max_cnt)) != cudaSuccess) break;
      if ((e = cudaHostAlloc(&sl.hmeta, sizeof(int) * 3 * (size_t)max_cnt, 0)) != cudaSuccess) break;
      if ((e = cudaHostAlloc(&sl.hptr, sizeof(double*) * (size_t)max_cnt, 0)) != cudaSuccess) break;
      sl.cap = max_cnt;
    }
  }

  auto drain = [&](Slot& sl) -> cudaError_t {  // wait for the slot's chunk, scatter info
    if (sl.chunk < 0) return cudaSuccess;
    cudaError_t r = cudaEventSynchronize(sl.done);
    const Chunk& c = chunks[sl.chunk];
    const int cnt = (int)c.idx.size();
    for (int j = 0; j < cnt; ++j) h_info[c.idx[j]] = sl.hmeta[2 * sl.cap + j];
    sl.chunk = -1;
    return r;
  };

  for (int ci = 0; ci < (int)chunks.size() && e == cudaSuccess; ++ci) {
    Slot& sl = slots[ci % nslots];
    if ((e = drain(sl)) != cudaSuccess) break;
    const Chunk& c = chunks[ci];
    const int cnt = (int)c.idx.size();
    int cmax = 0;
    for (int j = 0; j < cnt; ++j) {
      const int i = c.idx[j];
      sl.hmeta[j] = h_n[i];
      sl.hmeta[sl.cap + j] = h_ldda[i];
      sl.hptr[j] = reinterpret_cast<double*>(sl.dbuf + c.dev_off[j]);
      cmax = std::max(cmax, h_n[i]);
    }
    for (const Run& r : c.runs)
      if ((e = cudaMemcpyAsync(sl.dbuf + r.dev_off, r.host, r.bytes, cudaMemcpyHostToDevice,
                               sl.stream)) != cudaSuccess) break;
    if (e != cudaSuccess) break;
    if ((e = cudaMemcpyAsync(sl.dmeta, sl.hmeta, sizeof(int) * 2 * (size_t)sl.cap,
                             cudaMemcpyHostToDevice, sl.stream)) != cudaSuccess) break;
    if ((e = cudaMemcpyAsync(sl.dptr, sl.hptr, sizeof(double*) * (size_t)cnt,
                             cudaMemcpyHostToDevice, sl.stream)) != cudaSuccess) break;
    int rc = vbatched_dpotrf(uplo, sl.dmeta, sl.dptr, sl.dmeta + sl.cap, sl.dmeta + 2 * sl.cap, cnt,
                             cmax, (vb_stream_t)sl.stream);
    if (rc != 0) { e = rc > 0 ? (cudaError_t)rc : cudaErrorInvalidValue; break; }
    for (const Run& r : c.runs)
      if ((e = cudaMemcpyAsync(const_cast<double*>(r.host), sl.dbuf + r.dev_off, r.bytes,
                               cudaMemcpyDeviceToHost, sl.stream)) != cudaSuccess) break;
    if (e != cudaSuccess) break;
    if ((e = cudaMemcpyAsync(sl.hmeta + 2 * sl.cap, sl.dmeta + 2 * sl.cap, sizeof(int) * (size_t)cnt,
                             cudaMemcpyDeviceToHost, sl.stream)) != cudaSuccess) break;
    if ((e = cudaEventRecord(sl.done, sl.stream)) != cudaSuccess) break;
    sl.chunk = ci;
  }
  for (int s = 0; s < nslots; ++s) {
    cudaError_t r = drain(slots[s]);
    if (e == cudaSuccess) e = r;
  }
  for (int s = 0; s < nslots; ++s)
    if (slots[s].stream) cudaStreamSynchronize(slots[s].stream);
  if (start_ev) cudaEventDestroy(start_ev);
  return (int)e;
}

// Frees the staging ring of the current device (device buffers, pinned mirrors, streams,
// events) that vbatched_dpotrf_host keeps between calls. Safe to call at any time outside a
// vbatched_dpotrf_host call; the next call re-creates what it needs.
extern "C" int vbatched_release_host_staging(void) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return (int)e;
  if (dev < 0 || dev >= kMaxDevices) return (int)cudaErrorInvalidDevice;
  std::lock_guard<std::mutex> lock(g_stage_mutex);
  for (Slot& sl : g_stage[dev].slots) {
    if (sl.stream) cudaStreamSynchronize(sl.stream);
    if (sl.dbuf) cudaFree(sl.dbuf);
    if (sl.dmeta) cudaFree(sl.dmeta);
    if (sl.dptr) cudaFree(sl.dptr);
    if (sl.hmeta) cudaFreeHost(sl.hmeta);
    if (sl.hptr) cudaFreeHost(sl.hptr);
    if (sl.done) cudaEventDestroy(sl.done);
    if (sl.stream) cudaStreamDestroy(sl.stream);
    sl = Slot();
  }
  return (int)cudaGetLastError();
}
