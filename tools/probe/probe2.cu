// Probe 2: copy-engine cost at block granularity (per-call vs cudaMemcpyBatchAsync vs
// coalesced runs) and the kernel path's store width, to decide the K4-CE design.
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <vector>
#include <algorithm>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { \
  printf("{\"error\":\"%s\",\"line\":%d}\n", cudaGetErrorString(e_), __LINE__); fflush(stdout); exit(1);} } while (0)

struct Timer {
  cudaEvent_t a, b; cudaStream_t s;
  Timer(cudaStream_t st) : s(st) { cudaEventCreate(&a); cudaEventCreate(&b); }
  void start() { cudaEventRecord(a, s); }
  float stop() { cudaEventRecord(b, s); cudaEventSynchronize(b); float ms; cudaEventElapsedTime(&ms, a, b); return ms; }
};
template <class F> static float best_of(int reps, cudaStream_t s, F f) {
  Timer t(s); float best = 1e30f;
  for (int r = 0; r < reps; ++r) { t.start(); f(); best = std::min(best, t.stop()); }
  return best;
}
static void emit(const char* name, size_t bytes, float ms, const char* extra = "") {
  printf("{\"probe\":\"%s\",\"bytes\":%zu,\"ms\":%.4f,\"GBps\":%.2f%s}\n", name, bytes, ms, bytes / (ms * 1e6), extra);
  fflush(stdout);
}

__global__ void st256_copy(const uint4* __restrict__ src, uint4* __restrict__ dst, size_t n16) {
  // 256-bit global stores (v8.b32) to the destination (host-mapped for D2H)
  size_t n32 = n16 / 2;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n32; i += (size_t)gridDim.x * blockDim.x) {
    uint4 a = src[2 * i], b = src[2 * i + 1];
    asm volatile("st.global.v8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(dst + 2 * i), "r"(a.x), "r"(a.y), "r"(a.z),
                 "r"(a.w), "r"(b.x), "r"(b.y), "r"(b.z), "r"(b.w) : "memory");
  }
}
__global__ void ld256_copy(const uint4* __restrict__ src, uint4* __restrict__ dst, size_t n16) {
  size_t n32 = n16 / 2;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n32; i += (size_t)gridDim.x * blockDim.x) {
    uint32_t r[8];
    asm volatile("ld.global.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];" : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]),
                 "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]) : "l"(src + 2 * i));
    dst[2 * i] = make_uint4(r[0], r[1], r[2], r[3]);
    dst[2 * i + 1] = make_uint4(r[4], r[5], r[6], r[7]);
  }
}

int main() {
  CK(cudaSetDevice(0));
  cudaStream_t s0, s1; CK(cudaStreamCreateWithFlags(&s0, cudaStreamNonBlocking)); CK(cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking));
  const size_t B = 1ull << 30;
  char *h, *d, *h2, *d2;
  CK(cudaHostAlloc(&h, B, cudaHostAllocMapped)); CK(cudaHostAlloc(&h2, B, cudaHostAllocMapped));
  CK(cudaMalloc(&d, B)); CK(cudaMalloc(&d2, B));
  memset(h, 1, B); memset(h2, 2, B);
  // per-call vs batch at several sizes; blocks scattered (every other slot) so runs don't merge
  for (size_t bs : {size_t(64) << 10, size_t(2) << 20, size_t(8) << 20, size_t(32) << 20}) {
    size_t n = (B / 2) / bs;
    std::vector<void*> dsts(n), srcs(n); std::vector<size_t> sizes(n, bs);
    for (size_t i = 0; i < n; ++i) { dsts[i] = d + 2 * i * bs; srcs[i] = h + 2 * i * bs; }
    char ex[64]; snprintf(ex, 64, ",\"block\":%zu,\"n\":%zu", bs, n);
    emit("ce_h2d_loop", n * bs, best_of(3, s0, [&] { for (size_t i = 0; i < n; ++i) cudaMemcpyAsync(dsts[i], srcs[i], bs, cudaMemcpyHostToDevice, s0); }), ex);
    cudaMemcpyAttributes attr{};
    attr.srcAccessOrder = cudaMemcpySrcAccessOrderStream;
    attr.flags = cudaMemcpyFlagPreferOverlapWithCompute;
    size_t aidx = 0, fail = 0;
    emit("ce_h2d_batch", n * bs, best_of(3, s0, [&] {
      cudaError_t e = cudaMemcpyBatchAsync(dsts.data(), srcs.data(), sizes.data(), n, &attr, &aidx, 1, &fail, s0);
      if (e) { printf("{\"batch_err\":\"%s\"}\n", cudaGetErrorString(e)); cudaGetLastError(); } }), ex);
    std::vector<void*> d2hd(n), d2hs(n);
    for (size_t i = 0; i < n; ++i) { d2hd[i] = h + 2 * i * bs; d2hs[i] = d + 2 * i * bs; }
    emit("ce_d2h_batch", n * bs, best_of(3, s0, [&] {
      cudaError_t e = cudaMemcpyBatchAsync(d2hd.data(), d2hs.data(), sizes.data(), n, &attr, &aidx, 1, &fail, s0);
      if (e) { printf("{\"batch_err\":\"%s\"}\n", cudaGetErrorString(e)); cudaGetLastError(); } }), ex);
    cudaEvent_t e; cudaEventCreate(&e);
    emit("ce_duplex_batch", 2 * n * bs, best_of(3, s0, [&] {
      cudaEventRecord(e, s0); cudaStreamWaitEvent(s1, e, 0);
      cudaMemcpyBatchAsync(dsts.data(), srcs.data(), sizes.data(), n, &attr, &aidx, 1, &fail, s0);
      cudaMemcpyBatchAsync(d2hd.data(), d2hs.data(), sizes.data(), n, &attr, &aidx, 1, &fail, s1);
      cudaEventRecord(e, s1); cudaStreamWaitEvent(s0, e, 0); }), ex);
  }
  // 256-bit kernel copies
  void *hd; CK(cudaHostGetDevicePointer(&hd, h, 0));
  for (int g : {148, 592}) {
    char ex[64]; snprintf(ex, 64, ",\"grid\":%d", g);
    emit("k256_d2h", B, best_of(5, s0, [&] { st256_copy<<<g, 512, 0, s0>>>((const uint4*)d, (uint4*)hd, B / 16); }), ex);
    emit("k256_h2d", B, best_of(5, s0, [&] { ld256_copy<<<g, 512, 0, s0>>>((const uint4*)hd, (uint4*)d, B / 16); }), ex);
  }
  CK(cudaGetLastError());
  // CE H2D concurrently with kernel D2H (mixed engines)
  {
    cudaEvent_t e; cudaEventCreate(&e);
    emit("mixed_ceh2d_kd2h", 2 * B, best_of(3, s0, [&] {
      cudaEventRecord(e, s0); cudaStreamWaitEvent(s1, e, 0);
      cudaMemcpyAsync(d2, h2, B, cudaMemcpyHostToDevice, s0);
      st256_copy<<<296, 512, 0, s1>>>((const uint4*)d, (uint4*)hd, B / 16);
      cudaEventRecord(e, s1); cudaStreamWaitEvent(s0, e, 0); }));
  }
  return 0;
}
