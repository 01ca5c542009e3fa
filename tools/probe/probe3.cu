// Probe 3: cost of the scan machinery for a directive-like kernel over 2^21 blocks.
// A: plain streaming (st read, key/st/map writes, no ordered output)
// B: A + ordered DISC appends via ticket + block scan + warp look-back (like k_directive)
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <algorithm>
#define FULL 0xffffffffu
constexpr int TPB = 512, IPT = 8, TILE = TPB * IPT;

__global__ void __launch_bounds__(TPB) kA(const uint8_t* st_in, uint8_t* st, uint32_t* key, uint32_t* map, uint32_t n, uint32_t seq) {
  uint32_t first = blockIdx.x * TILE + threadIdx.x * IPT;
#pragma unroll
  for (int k = 0; k < IPT; ++k) {
    uint32_t i = first + k;
    if (i < n && st_in[i] == 3) { st[i] = 4; key[i] = seq; map[i] = 0xffffffffu; }
  }
}

__global__ void __launch_bounds__(TPB) kA2(const uint8_t* st_in, uint8_t* st, uint32_t* key, uint32_t* map, uint32_t n, uint32_t seq) {
  // coalesced: item k of thread t is first_block + k*TPB + t
  uint32_t base = blockIdx.x * TILE + threadIdx.x;
#pragma unroll
  for (int k = 0; k < IPT; ++k) {
    uint32_t i = base + k * TPB;
    if (i < n && st_in[i] == 3) { st[i] = 4; key[i] = seq; map[i] = 0xffffffffu; }
  }
}

__device__ unsigned long long lookback(volatile unsigned long long* stt, uint32_t tile, unsigned long long agg) {
  const unsigned long long FA = 1ull << 62, FP = 2ull << 62, M = FA - 1;
  const int lane = threadIdx.x & 31;
  if (tile == 0) { if (lane == 0) stt[0] = FP | agg; __threadfence(); return 0; }
  if (lane == 0) stt[tile] = FA | agg;
  __threadfence();
  unsigned long long excl = 0; long long p = (long long)tile - 1;
  while (true) {
    long long idx = p - lane; unsigned long long v = FP;
    if (idx >= 0) { do { v = stt[idx]; } while ((v >> 62) == 0); }
    unsigned pm = __ballot_sync(FULL, (v >> 62) == 2);
    int stop = pm ? __ffs(pm) - 1 : 31;
    unsigned long long x = lane <= stop ? (v & M) : 0;
    for (int o = 16; o; o >>= 1) x += __shfl_xor_sync(FULL, x, o);
    excl += x; if (pm) break; p -= 32;
  }
  if (lane == 0) stt[tile] = FP | (excl + agg);
  __threadfence();
  return excl;
}

template <bool TICKET, bool COALESCED>
__global__ void __launch_bounds__(TPB) kB(const uint8_t* st_in, uint8_t* st, uint32_t* key, uint32_t* map, uint64_t* ring,
                                          unsigned long long* status, unsigned* ticket, uint32_t n, uint32_t seq) {
  __shared__ uint32_t s_tile; __shared__ unsigned long long s_sc[TPB / 32]; __shared__ unsigned long long s_ex;
  if (TICKET) { if (threadIdx.x == 0) s_tile = atomicAdd(ticket, 1u); __syncthreads(); }
  uint32_t tile = TICKET ? s_tile : blockIdx.x;
  uint32_t idx[IPT]; unsigned m = 0; uint32_t c = 0;
#pragma unroll
  for (int k = 0; k < IPT; ++k) {
    uint32_t i = COALESCED ? tile * TILE + k * TPB + threadIdx.x : tile * TILE + threadIdx.x * IPT + k;
    idx[k] = i;
    bool g = i < n && st_in[i] == 3; m |= (unsigned)g << k; c += g;
  }
  // block scan (simple)
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  unsigned long long x = c;
  for (int o = 1; o < 32; o <<= 1) { unsigned long long y = __shfl_up_sync(FULL, x, o); if (lane >= o) x += y; }
  if (lane == 31) s_sc[w] = x;
  __syncthreads();
  if (w == 0) { unsigned long long t = lane < TPB / 32 ? s_sc[lane] : 0; for (int o = 1; o < 32; o <<= 1) { unsigned long long y = __shfl_up_sync(FULL, t, o); if (lane >= o) t += y; } if (lane < TPB / 32) s_sc[lane] = t; }
  __syncthreads();
  unsigned long long pre = (w ? s_sc[w - 1] : 0) + x - c, tot = s_sc[TPB / 32 - 1];
  if (threadIdx.x < 32) { unsigned long long e = lookback(status, tile, tot); if (threadIdx.x == 0) s_ex = e; }
  __syncthreads();
  unsigned long long p = s_ex + pre;
#pragma unroll
  for (int k = 0; k < IPT; ++k) if ((m >> k) & 1) { uint32_t i = idx[k]; st[i] = 4; key[i] = seq; map[i] = 0xffffffffu; ring[p++] = ((unsigned long long)seq << 32) | i; }
}

int main() {
  const uint32_t n = 1u << 21, nt = n / TILE;
  uint8_t *st_in, *st; uint32_t *key, *map; uint64_t* ring; unsigned long long* status; unsigned* ticket;
  cudaMalloc(&st_in, n); cudaMalloc(&st, n); cudaMalloc(&key, 4 * n); cudaMalloc(&map, 4 * n); cudaMalloc(&ring, 8 * n);
  cudaMalloc(&status, 8 * nt); cudaMalloc(&ticket, 4);
  cudaMemset(st_in, 3, n / 2); cudaMemset(st_in + n / 2, 1, n / 2);   // half G
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  auto time = [&](const char* name, auto f) {
    float best = 1e9;
    for (int r = 0; r < 20; ++r) { cudaMemset(status, 0, 8 * nt); cudaMemset(ticket, 0, 4); cudaDeviceSynchronize();
      cudaEventRecord(a); f(); cudaEventRecord(b); cudaEventSynchronize(b); float ms; cudaEventElapsedTime(&ms, a, b); best = std::min(best, ms); }
    printf("{\"probe\":\"%s\",\"us\":%.2f,\"err\":\"%s\"}\n", name, best * 1e3, cudaGetErrorString(cudaGetLastError()));
  };
  time("A_strided", [&] { kA<<<nt, TPB>>>(st_in, st, key, map, n, 7); });
  time("A_coalesced", [&] { kA2<<<nt, TPB>>>(st_in, st, key, map, n, 7); });
  time("B_ticket_strided", [&] { kB<true, false><<<nt, TPB>>>(st_in, st, key, map, ring, status, ticket, n, 7); });
  time("B_ticket_coalesced", [&] { kB<true, true><<<nt, TPB>>>(st_in, st, key, map, ring, status, ticket, n, 7); });
  time("B_noticket_coalesced", [&] { kB<false, true><<<nt, TPB>>>(st_in, st, key, map, ring, status, ticket, n, 7); });
  time("memset_only", [&] {});
  return 0;
}
