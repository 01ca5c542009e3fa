// Step-0 box probe: host-link rooflines and feasibility checks
// for the kernel-driven transfer engine.  Scratch tool, not part of libum.
//   (a) can a kernel dereference mapped pinned host memory (zero-copy LDG/STG)?
//   (b) does cp.async.bulk (TMA bulk) accept a host-mapped global address?
//   (c) how much host memory can be pinned and how fast?
// Prints one JSON object per measurement on stdout.
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cstring>
#include <vector>
#include <chrono>
#include <algorithm>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { \
  printf("{\"error\":\"%s\",\"line\":%d}\n", cudaGetErrorString(e_), __LINE__); fflush(stdout); exit(1);} } while (0)

__global__ void zc_copy(const uint4* __restrict__ src, uint4* __restrict__ dst, size_t n) {
  size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  size_t stride = (size_t)gridDim.x * blockDim.x;
  constexpr int U = 8;
  for (; i + (U - 1) * stride < n; i += U * stride) {
    uint4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) v[u] = src[i + u * stride];
#pragma unroll
    for (int u = 0; u < U; ++u) dst[i + u * stride] = v[u];
  }
  for (; i < n; i += stride) dst[i] = src[i];
}

__global__ void zero_v4(uint4* __restrict__ dst, size_t n) {
  size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  size_t stride = (size_t)gridDim.x * blockDim.x;
  uint4 z = make_uint4(0, 0, 0, 0);
  for (; i < n; i += stride) dst[i] = z;
}

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t cnt) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(cnt));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n WAIT_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      " @!p bra WAIT_%=;\n}\n" ::"r"(smem_u32(bar)), "r"(parity) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* sdst, const void* gsrc, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
      ::"r"(smem_u32(sdst)), "l"(gsrc), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void bulk_s2g(void* gdst, const void* ssrc, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
               ::"l"(gdst), "r"(smem_u32(ssrc)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N> __device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
template <int N> __device__ __forceinline__ void bulk_wait() {
  asm volatile("cp.async.bulk.wait_group %0;" ::"n"(N) : "memory");
}

// TMA-bulk staged copy: one elected thread per CTA drives an S-stage ring of CH-byte
// chunks: global(src) -> smem -> global(dst).  Chunks are grid-strided.
template <int S>
__global__ void bulk_copy(const char* __restrict__ src, char* __restrict__ dst, size_t bytes, uint32_t CH) {
  extern __shared__ __align__(128) char smem[];
  __shared__ __align__(8) uint64_t bar[S];
  if (threadIdx.x != 0) return;
  for (int s = 0; s < S; ++s) mbar_init(&bar[s], 1);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  size_t nch = bytes / CH;
  // my chunks: blockIdx.x + j*gridDim.x
  size_t mine = nch > blockIdx.x ? (nch - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
  auto chunk = [&](size_t j) { return (size_t)(blockIdx.x + j * gridDim.x) * CH; };
  for (size_t j = 0; j < mine && j < (size_t)S; ++j) {
    mbar_expect_tx(&bar[j], CH);
    bulk_g2s(smem + j * CH, src + chunk(j), CH, &bar[j]);
  }
  for (size_t j = 0; j < mine; ++j) {
    int s = j % S;
    mbar_wait(&bar[s], (j / S) & 1);
    bulk_s2g(dst + chunk(j), smem + s * CH, CH);
    bulk_commit();
    // refill the stage used by chunk j-1 once its store finished reading smem
    if (j >= 1 && j - 1 + S < mine) {
      bulk_wait_read<1>();
      int sp = (j - 1) % S;
      mbar_expect_tx(&bar[sp], CH);
      bulk_g2s(smem + sp * CH, src + chunk(j - 1 + S), CH, &bar[sp]);
    } else if (j == 0 && S == 1 && 1 < mine) {
      bulk_wait_read<0>();
    }
  }
  bulk_wait<0>();
}

// Zero-fill by TMA bulk store from a zeroed smem tile.
__global__ void bulk_zero(char* __restrict__ dst, size_t bytes, uint32_t CH) {
  extern __shared__ __align__(128) char smem[];
  for (uint32_t i = threadIdx.x * 16; i < CH; i += blockDim.x * 16) *(uint4*)(smem + i) = make_uint4(0, 0, 0, 0);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncthreads();
  if (threadIdx.x != 0) return;
  size_t nch = bytes / CH;
  for (size_t c = blockIdx.x; c < nch; c += gridDim.x) {
    bulk_s2g(dst + c * CH, smem, CH);
    bulk_commit();
  }
  bulk_wait<0>();
}

static double now_s() {
  return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

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

static long meminfo_kb(const char* key) {
  FILE* f = fopen("/proc/meminfo", "r"); if (!f) return -1;
  char line[256]; long v = -1;
  while (fgets(line, sizeof line, f)) if (!strncmp(line, key, strlen(key))) { sscanf(line + strlen(key), " %ld", &v); break; }
  fclose(f); return v;
}

int main(int argc, char** argv) {
  const char* mode = argc > 1 ? argv[1] : "bw";
  int dev = 0; CK(cudaSetDevice(dev));
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, dev));
  printf("{\"gpu\":\"%s\",\"sms\":%d,\"cc\":\"%d.%d\",\"unifiedAddressing\":%d,\"canMapHostMemory\":%d,\"pageableMemoryAccess\":%d,\"pciBus\":%d}\n",
         p.name, p.multiProcessorCount, p.major, p.minor, p.unifiedAddressing, p.canMapHostMemory,
         p.pageableMemoryAccess, p.pciBusID);
  cudaStream_t s0, s1; CK(cudaStreamCreateWithFlags(&s0, cudaStreamNonBlocking)); CK(cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking));

  if (!strcmp(mode, "bw")) {
    const size_t B = 1ull << 30;
    char *h1, *h2, *d1, *d2;
    double t0 = now_s();
    CK(cudaHostAlloc(&h1, B, cudaHostAllocMapped | cudaHostAllocPortable));
    CK(cudaHostAlloc(&h2, B, cudaHostAllocMapped | cudaHostAllocPortable));
    printf("{\"probe\":\"pin_2GiB_s\",\"s\":%.3f}\n", now_s() - t0);
    memset(h1, 1, B); memset(h2, 2, B);
    CK(cudaMalloc(&d1, B)); CK(cudaMalloc(&d2, B));
    CK(cudaMemset(d1, 3, B)); CK(cudaMemset(d2, 4, B));
    void *hd1, *hd2; CK(cudaHostGetDevicePointer(&hd1, h1, 0)); CK(cudaHostGetDevicePointer(&hd2, h2, 0));
    printf("{\"probe\":\"uva_same_ptr\",\"v\":%d}\n", (int)(hd1 == (void*)h1));
    // CE
    emit("ce_h2d", B, best_of(10, s0, [&] { cudaMemcpyAsync(d1, h1, B, cudaMemcpyHostToDevice, s0); }));
    emit("ce_d2h", B, best_of(10, s0, [&] { cudaMemcpyAsync(h1, d1, B, cudaMemcpyDeviceToHost, s0); }));
    {
      cudaEvent_t e; cudaEventCreate(&e);
      emit("ce_duplex", 2 * B, best_of(10, s0, [&] {
        cudaEventRecord(e, s0); cudaStreamWaitEvent(s1, e, 0);
        cudaMemcpyAsync(d1, h1, B, cudaMemcpyHostToDevice, s0);
        cudaMemcpyAsync(h2, d2, B, cudaMemcpyDeviceToHost, s1);
        cudaEventRecord(e, s1); cudaStreamWaitEvent(s0, e, 0); }));
    }
    // CE at block granularity: 64 KiB and 2 MiB calls
    for (size_t bs : {size_t(64) << 10, size_t(2) << 20}) {
      size_t n = (bs == (64u << 10)) ? 4096 : 256;
      char nm[64]; snprintf(nm, 64, "ce_h2d_calls_%zuKiB", bs >> 10);
      emit(nm, n * bs, best_of(5, s0, [&] { for (size_t i = 0; i < n; ++i) cudaMemcpyAsync(d1 + i * bs, h1 + i * bs, bs, cudaMemcpyHostToDevice, s0); }));
      snprintf(nm, 64, "ce_d2h_calls_%zuKiB", bs >> 10);
      emit(nm, n * bs, best_of(5, s0, [&] { for (size_t i = 0; i < n; ++i) cudaMemcpyAsync(h1 + i * bs, d1 + i * bs, bs, cudaMemcpyDeviceToHost, s0); }));
    }
    // zero-copy kernel
    size_t n4 = B / 16;
    for (int g : {148, 296, 592, 1184}) for (int t : {256, 512}) {
      char ex[64]; snprintf(ex, 64, ",\"grid\":%d,\"tpb\":%d", g, t);
      emit("zc_h2d", B, best_of(5, s0, [&] { zc_copy<<<g, t, 0, s0>>>((const uint4*)hd1, (uint4*)d1, n4); }), ex);
      emit("zc_d2h", B, best_of(5, s0, [&] { zc_copy<<<g, t, 0, s0>>>((const uint4*)d1, (uint4*)hd1, n4); }), ex);
    }
    CK(cudaGetLastError());
    {
      cudaEvent_t e; cudaEventCreate(&e);
      emit("zc_duplex", 2 * B, best_of(5, s0, [&] {
        cudaEventRecord(e, s0); cudaStreamWaitEvent(s1, e, 0);
        zc_copy<<<296, 512, 0, s0>>>((const uint4*)hd1, (uint4*)d1, n4);
        zc_copy<<<296, 512, 0, s1>>>((const uint4*)d2, (uint4*)hd2, n4);
        cudaEventRecord(e, s1); cudaStreamWaitEvent(s0, e, 0); }));
    }
    // verify zero-copy correctness
    {
      memset(h1, 0x5a, B); zc_copy<<<296, 512, 0, s0>>>((const uint4*)hd1, (uint4*)d1, n4); CK(cudaStreamSynchronize(s0));
      std::vector<char> chk(4096); CK(cudaMemcpy(chk.data(), d1 + B - 4096, 4096, cudaMemcpyDeviceToHost));
      printf("{\"probe\":\"zc_correct\",\"v\":%d}\n", (int)(chk[0] == 0x5a && chk[4095] == 0x5a));
    }
    // TMA bulk staged copy from/to host-mapped memory
    for (uint32_t CH : {16384u, 32768u, 65536u}) for (int g : {148, 296}) {
      int S = 4; size_t sm = (size_t)S * CH;
      if (sm > 200 * 1024) { S = 2; sm = 2 * CH; }
      auto kern = S == 4 ? bulk_copy<4> : bulk_copy<2>;
      CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm));
      char ex[96]; snprintf(ex, 96, ",\"grid\":%d,\"chunk\":%u,\"stages\":%d", g, CH, S);
      emit("tma_h2d", B, best_of(5, s0, [&] { kern<<<g, 32, sm, s0>>>((const char*)hd1, d1, B, CH); }), ex);
      CK(cudaGetLastError());
      emit("tma_d2h", B, best_of(5, s0, [&] { kern<<<g, 32, sm, s0>>>(d1, (char*)hd1, B, CH); }), ex);
      emit("tma_d2d", B, best_of(5, s0, [&] { kern<<<g, 32, sm, s0>>>(d2, d1, B, CH); }), ex);
      CK(cudaGetLastError());
    }
    {
      CK(cudaFuncSetAttribute(bulk_copy<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, 4 * 32768));
      memset(h1, 0x3c, B); bulk_copy<4><<<148, 32, 4 * 32768, s0>>>((const char*)hd1, d1, B, 32768); CK(cudaStreamSynchronize(s0));
      std::vector<char> chk(4096); CK(cudaMemcpy(chk.data(), d1 + B - 4096, 4096, cudaMemcpyDeviceToHost));
      printf("{\"probe\":\"tma_h2d_correct\",\"v\":%d}\n", (int)(chk[0] == 0x3c && chk[4095] == 0x3c));
      cudaEvent_t e; cudaEventCreate(&e);
      emit("tma_duplex", 2 * B, best_of(5, s0, [&] {
        cudaEventRecord(e, s0); cudaStreamWaitEvent(s1, e, 0);
        bulk_copy<4><<<148, 32, 4 * 32768, s0>>>((const char*)hd1, d1, B, 32768);
        bulk_copy<4><<<148, 32, 4 * 32768, s1>>>(d2, (char*)hd2, B, 32768);
        cudaEventRecord(e, s1); cudaStreamWaitEvent(s0, e, 0); }));
    }
    // HBM: write-only + copy
    {
      const size_t Z = 8ull << 30; char* dz; CK(cudaMalloc(&dz, Z));
      emit("hbm_memset", Z, best_of(10, s0, [&] { cudaMemsetAsync(dz, 0, Z, s0); }));
      emit("hbm_zero_v4", Z, best_of(10, s0, [&] { zero_v4<<<148 * 8, 512, 0, s0>>>((uint4*)dz, Z / 16); }));
      CK(cudaFuncSetAttribute(bulk_zero, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536));
      emit("hbm_bulk_zero", Z, best_of(10, s0, [&] { bulk_zero<<<148 * 2, 128, 65536, s0>>>(dz, Z, 65536); }));
      emit("hbm_copy_ce_rw", 2 * (Z / 2), best_of(10, s0, [&] { cudaMemcpyAsync(dz, dz + Z / 2, Z / 2, cudaMemcpyDeviceToDevice, s0); }));
      CK(cudaFree(dz));
    }
    CK(cudaFreeHost(h1)); CK(cudaFreeHost(h2)); CK(cudaFree(d1)); CK(cudaFree(d2));
  } else if (!strcmp(mode, "pin")) {
    // (c) pinning capacity: grab 8 GiB pinned chunks up to a cap (GiB) bounded by MemAvailable.
    long avail_kb = meminfo_kb("MemAvailable:");
    double cap_gib = argc > 2 ? atof(argv[2]) : 64;
    double lim = std::min(cap_gib, 0.6 * avail_kb / 1048576.0);
    printf("{\"probe\":\"pin_plan\",\"mem_available_gib\":%.1f,\"limit_gib\":%.1f}\n", avail_kb / 1048576.0, lim);
    std::vector<void*> ptrs; double t0 = now_s(); size_t got = 0; const size_t C = 8ull << 30;
    while ((got + C) / 1073741824.0 <= lim) {
      void* h; if (cudaHostAlloc(&h, C, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess) { cudaGetLastError(); break; }
      ptrs.push_back(h); got += C;
    }
    double t1 = now_s();
    printf("{\"probe\":\"pin_capacity\",\"gib\":%.1f,\"s\":%.2f,\"gib_per_s\":%.2f}\n", got / 1073741824.0, t1 - t0, got / 1073741824.0 / (t1 - t0));
    for (void* h : ptrs) cudaFreeHost(h);
    printf("{\"probe\":\"unpin_s\",\"s\":%.2f}\n", now_s() - t1);
  }
  return 0;
}
