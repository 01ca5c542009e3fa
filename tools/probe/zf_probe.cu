// Zero-fill probe: HBM write rate of the candidate zero-fill designs for the transfer
// kernel (K5 in the TMA path), over 32 GiB in 16 KiB units:
//   tma1   1 CTA/SM, one thread issues cp.async.bulk stores of a zeroed 16 KiB smem tile
//   tmaW   1 CTA/SM, lane 0 of each of W warps issues bulk stores (units split by warp)
//   stW    1 CTA/SM of W warps, st.global.v4 (8 in flight per thread), a unit per warp
//   memset cudaMemsetAsync
// Prints one JSON line per variant (best of 5, CUDA events).
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <cstdlib>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("{\"error\":\"%s\",\"line\":%d}\n", cudaGetErrorString(e_), __LINE__); return 1; } } while (0)

constexpr uint32_t CH = 16384;

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void k_tma(char* dst, unsigned long long units, int warps_issuing) {
  extern __shared__ __align__(128) char zero[];
  for (uint32_t i = threadIdx.x * 16; i < CH; i += blockDim.x * 16) *reinterpret_cast<uint4*>(zero + i) = make_uint4(0, 0, 0, 0);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncthreads();
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (lane != 0 || w >= warps_issuing) return;
  const unsigned long long ubeg = units * blockIdx.x / gridDim.x, uend = units * (blockIdx.x + 1) / gridDim.x;
  uint32_t n = 0;
  for (unsigned long long u = ubeg + w; u < uend; u += warps_issuing) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst + u * CH), "r"(smem_u32(zero)), "r"(CH) : "memory");
    if ((++n & 31) == 0) asm volatile("cp.async.bulk.commit_group;" ::: "memory");
  }
  asm volatile("cp.async.bulk.commit_group;" ::: "memory");
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

__global__ void k_st(char* dst, unsigned long long units) {
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
  const unsigned long long ubeg = units * blockIdx.x / gridDim.x, uend = units * (blockIdx.x + 1) / gridDim.x;
  const uint4 z = make_uint4(0, 0, 0, 0);
  for (unsigned long long u = ubeg + w; u < uend; u += nw) {
    uint4* d = reinterpret_cast<uint4*>(dst + u * CH);
#pragma unroll
    for (int k = 0; k < 32; ++k) d[k * 32 + lane] = z;
  }
}

int main() {
  int nsm;
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
  const size_t bytes = (size_t)(getenv("ZF_GIB") ? atoi(getenv("ZF_GIB")) : 32) << 30;
  const unsigned long long units = bytes / CH;
  char* d;
  CK(cudaMalloc(&d, bytes));
  CK(cudaFuncSetAttribute(k_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(9 * CH)));
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  auto run = [&](const char* name, int grid, auto fn) {
    float best = 1e30f;
    for (int r = 0; r < 6; ++r) {
      cudaEventRecord(a);
      fn();
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      if (r) best = ms < best ? ms : best;
    }
    cudaError_t e = cudaGetLastError();
    printf("{\"variant\":\"%s\",\"grid\":%d,\"ms\":%.3f,\"gbs\":%.1f,\"err\":\"%s\"}\n", name, grid, best, bytes / (best / 1e3) / 1e9,
           cudaGetErrorString(e));
    fflush(stdout);
  };
  for (int W : {1, 2, 4, 8}) {
    char nm[32];
    snprintf(nm, sizeof nm, "tma_warps%d", W);
    run(nm, nsm, [&] { k_tma<<<nsm, 32 * W, CH>>>(d, units, W); });
  }
  run("tma1_2ctas", 2 * nsm, [&] { k_tma<<<2 * nsm, 32, CH>>>(d, units, 1); });
  run("tma1_smem144k", nsm, [&] { k_tma<<<nsm, 32, 9 * CH>>>(d, units, 1); });
  for (int W : {4, 8, 16, 32}) {
    char nm[32];
    snprintf(nm, sizeof nm, "st_warps%d", W);
    run(nm, nsm, [&] { k_st<<<nsm, 32 * W>>>(d, units); });
  }
  run("st_warps8_x4ctas", 4 * nsm, [&] { k_st<<<4 * nsm, 256>>>(d, units); });
  run("memset", 0, [&] { cudaMemsetAsync(d, 0, bytes); });
  return 0;
}
