// sm_100a kernels of libum: the state/directive kernels (K1/K2 classify + ordered
// compaction, K3 victim selection, K6 commit, K7 ring compaction, K8 directives), the
// TMA-staged transfer engine over mapped pinned host memory with zero-fill (K4/K5),
// and harness kernels (application stamp writes, content tags, host writes).
//
// Paper: "UVM Discard" (Zhu et al., IISWC'22).  PAPER L<n> = line of its text.
// Design: DESIGN.md §4 (data layout) and §5 (kernels).  No tensor cores: nothing here
// is a contraction.  Everything is integer/byte movement.
#include "um_internal.h"

#include <cstdio>
#include <cstdlib>
#include <algorithm>

namespace um {

#define FULL 0xffffffffu

__constant__ int c_dummy;

// ------------------------------------------------------------------------------------
// small helpers
// ------------------------------------------------------------------------------------
__device__ __forceinline__ char* hptr(const Tables& T, uint32_t hf) {
  return T.hchunks[hf / T.hpc] + (size_t)(hf % T.hpc) * T.B;
}

// Programmatic dependent launch (PDL): every paging-stream kernel lets its successor be
// scheduled as soon as all of its own CTAs are running (launch_dependents), and waits for
// its predecessor's completion and memory (griddepcontrol.wait) before touching state.
// The successor's launch latency then overlaps this kernel's execution.  Both are no-ops
// for a kernel launched without the PDL attribute.
__device__ __forceinline__ void pdl_enter() {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  asm volatile("griddepcontrol.wait;" ::: "memory");
}

// Packed per-block state word (Tables::sk): bits 0-2 = state, bits 3-31 = key (seq).
__device__ __forceinline__ uint8_t st_of(uint32_t w) { return (uint8_t)(w & 7u); }
__device__ __forceinline__ uint32_t key_of(uint32_t w) { return w >> 3; }
__device__ __forceinline__ uint32_t mk_sk(uint8_t st, uint32_t key) { return (key << 3) | st; }
__device__ __forceinline__ uint8_t ld_st(const Tables& T, uint32_t b) { return st_of(T.sk[b]); }
// liveness of ring entry (key kk, block b) whose ring holds state set {G} (USED) or {GE, GL} (DISC);
// a slot whose block did not enter the ring holds kDeadSlot (block id NONE: no state gather)
constexpr unsigned long long kDeadSlot = ~0ull;
__device__ __forceinline__ bool entry_live(const Tables& T, bool disc, uint32_t blk, uint32_t kk) {
  if (blk == UM_NONE) return false;
  const uint32_t w = T.sk[blk];
  const uint8_t ss = st_of(w);
  return (disc ? (ss == ST_GE || ss == ST_GL) : ss == ST_G) && key_of(w) == kk;
}

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}

__device__ __forceinline__ uint32_t iv_lo(const OpIv& iv, uint32_t j) { return iv.inl ? iv.ilo[j] : iv.lo[j]; }
__device__ __forceinline__ uint32_t iv_pre(const OpIv& iv, uint32_t j) { return iv.inl ? iv.ipre[j] : iv.pre[j]; }
__device__ __forceinline__ uint8_t iv_w(const OpIv& iv, uint32_t j) { return iv.inl ? iv.iw[j] : iv.wflag[j]; }

// Largest j in [0, m) with pre[j] <= g (pre strictly increasing, pre[0] = 0).
__device__ __forceinline__ uint32_t iv_find(const OpIv& iv, uint32_t g) {
  uint32_t lo = 0, hi = iv.m;  // answer in [lo, hi)
  while (hi - lo > 1) {
    uint32_t mid = (lo + hi) >> 1;
    if (iv_pre(iv, mid) <= g) lo = mid; else hi = mid;
  }
  return lo;
}

__device__ __forceinline__ void stat_add(const Tables& T, int slot, long long v) {
  if (v) atomicAdd((unsigned long long*)&T.ctl->stats[blockIdx.x & 7][slot], (unsigned long long)v);
}

// Transfer log (um_xlog_attach; off when T.xlog is null): one record per block whose move
// or zero-fill enters a work list the transfer engine executes.
__device__ __forceinline__ void xlog_put(const Tables& T, uint32_t seq, uint32_t blk, uint32_t kind, uint32_t prev) {
  if (!T.xlog) return;
  const unsigned long long p = atomicAdd(&T.ctl->xlog_n, 1ull);
  if (p < T.xlog_cap) T.xlog[p] = make_uint4(seq, blk, kind, prev);
}

// A G block b entering the D2H-only list (prefetch HOST, evict) at position pos: its
// dead pages (two-level) are recorded for the service kernel and not counted as moved.
__device__ __forceinline__ void d2h_listed(const Tables& T, uint32_t seq, uint32_t b, uint32_t pos, uint32_t prev) {
  uint32_t dm = 0u;
  if (T.pdead) {
    dm = T.pdead[b];
    T.d2h_dmask[pos] = dm;
    if (dm) {
      const long long d = (long long)__popc(dm) * T.P;
      stat_add(T, S_D2H, -d);
      stat_add(T, S_D2H_AV, d);
    }
  }
  if (T.xlog)
    for (uint32_t p = 0; p < T.ppc; ++p)
      if (!((dm >> p) & 1u)) xlog_put(T, seq, b * T.ppc + p, XL_D2H, prev);
}

// Exclusive block scan of a 64-bit value (two packed 31-bit counts add without carry).
template <int TPB>
__device__ __forceinline__ unsigned long long block_excl_scan(unsigned long long v, unsigned long long& total,
                                                              unsigned long long* sm) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  unsigned long long x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    unsigned long long y = __shfl_up_sync(FULL, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) sm[w] = x;
  __syncthreads();
  if (w == 0) {
    unsigned long long t = lane < TPB / 32 ? sm[lane] : 0ull;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      unsigned long long y = __shfl_up_sync(FULL, t, o);
      if (lane >= o) t += y;
    }
    if (lane < TPB / 32) sm[lane] = t;
  }
  __syncthreads();
  unsigned long long pre = (w ? sm[w - 1] : 0ull) + x - v;
  total = sm[TPB / 32 - 1];
  __syncthreads();
  return pre;
}

// Decoupled look-back (single pass).  Tiles are ordered by blockIdx: CTAs are
// dispatched in index order, so every predecessor of a waiting tile is resident or done.
// Returns the exclusive prefix of this tile.  Status word = flag(2b) | value(62b).
__device__ unsigned long long lookback(const Tables& T, uint32_t tile, unsigned long long agg) {
  volatile unsigned long long* st = T.tile_status;
  const unsigned long long FA = 1ull << 62, FP = 2ull << 62, M = FA - 1;
  if (tile == 0) {
    st[0] = FP | agg;
    __threadfence();
    return 0ull;
  }
  st[tile] = FA | agg;
  __threadfence();
  unsigned long long excl = 0;
  int p = (int)tile - 1;
  while (true) {
    unsigned long long v;
    do { v = st[p]; } while ((v >> 62) == 0);
    excl += v & M;
    if ((v >> 62) == 2) break;
    --p;
  }
  st[tile] = FP | (excl + agg);
  __threadfence();
  return excl;
}

// Warp-parallel decoupled look-back (called by all 32 lanes of warp 0): each round
// inspects 32 predecessors at once; the closest one holding an inclusive prefix ends the
// walk.  Returns the tile's exclusive prefix.
__device__ unsigned long long lookback_warp(const Tables& T, uint32_t tile, unsigned long long agg) {
  volatile unsigned long long* st = T.tile_status;
  const unsigned long long FA = 1ull << 62, FP = 2ull << 62, M = FA - 1;
  const int lane = threadIdx.x & 31;
  if (tile == 0) {
    if (lane == 0) st[0] = FP | agg;
    __threadfence();
    return 0ull;
  }
  if (lane == 0) st[tile] = FA | agg;
  __threadfence();
  // each round inspects 128 predecessors (4 independent loads per lane); the closest
  // one holding an inclusive prefix (or the start of the array) ends the walk
  unsigned long long excl = 0;
  long long p = (long long)tile - 1;
  while (true) {
    unsigned long long v[4];
    long long pbest = -1;  // largest index in this round holding an inclusive prefix
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const long long idx = p - lane - 32 * q;
      v[q] = 0;
      if (idx >= 0) {
        do { v[q] = st[idx]; } while ((v[q] >> 62) == 0);
        if ((v[q] >> 62) == 2 && idx > pbest) pbest = idx;
      }
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) {
      long long y = __shfl_xor_sync(FULL, pbest, o);
      pbest = y > pbest ? y : pbest;
    }
    const bool done = pbest >= 0 || p - 127 <= 0;   // a prefix found, or tile 0 reached
    unsigned long long x = 0;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const long long idx = p - lane - 32 * q;
      if (idx >= 0 && idx >= pbest) x += v[q] & M;
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) x += __shfl_xor_sync(FULL, x, o);
    excl += x;
    if (done) break;
    p -= 128;
  }
  if (lane == 0) st[tile] = FP | (excl + agg);
  __threadfence();
  return excl;
}

// Called by every thread at the end of a scanning CTA: the last CTA to finish clears
// the tile statuses and the ticket, so the next scanning launch starts clean.
__device__ void scan_finish(const Tables& T, uint32_t ntiles) {
  __shared__ int s_last;
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    unsigned int d = atomicAdd(&T.ctl->scan_done, 1u);
    s_last = (d == ntiles - 1);
  }
  __syncthreads();
  if (s_last) {
    __threadfence();
    for (uint32_t i = threadIdx.x; i < ntiles; i += blockDim.x) T.tile_status[i] = 0ull;
    if (threadIdx.x == 0) {
      T.ctl->scan_done = 0;
      T.ctl->scan_ticket = 0;
    }
    __threadfence();
  }
}


__device__ __forceinline__ unsigned long long pack2(uint32_t a, uint32_t b) {
  return (unsigned long long)a | ((unsigned long long)b << 31);
}
__device__ __forceinline__ uint32_t unpackA(unsigned long long v) { return (uint32_t)(v & 0x7fffffffull); }
__device__ __forceinline__ uint32_t unpackB(unsigned long long v) { return (uint32_t)((v >> 31) & 0x7fffffffull); }

// Sum of per-thread class counts over the CTA, then one atomic per class.
template <int NC>
__device__ __forceinline__ void block_counts_to(const Tables& T, uint32_t (&c)[NC], uint32_t* sm /*[NC]*/,
                                                const int (&slots)[NC], const long long (&mul)[NC]) {
  if (threadIdx.x < NC) sm[threadIdx.x] = 0;
  __syncthreads();
#pragma unroll
  for (int i = 0; i < NC; ++i) {
    uint32_t v = __reduce_add_sync(FULL, c[i]);
    if ((threadIdx.x & 31) == 0 && v) atomicAdd(&sm[i], v);
  }
  __syncthreads();
#pragma unroll
  for (int i = 0; i < NC; ++i)   // static indices: the slot tables stay in registers
    if (threadIdx.x == i && slots[i] >= 0) stat_add(T, slots[i], (long long)sm[i] * mul[i]);
}

// Multi-CTA scans do not add their counters with same-address atomics (thousands of
// CTAs serialise on one L2 atomic unit): each tile stores its block-reduced counts and
// the last CTA of the launch (scan_finish) sums them and adds once per counter.
template <int NC>
__device__ __forceinline__ void tile_counts(const Tables& T, uint32_t tile, uint32_t (&c)[NC], uint32_t* sm) {
  if (threadIdx.x < NC) sm[threadIdx.x] = 0;
  __syncthreads();
#pragma unroll
  for (int i = 0; i < NC; ++i) {
    uint32_t v = __reduce_add_sync(FULL, c[i]);
    if ((threadIdx.x & 31) == 0 && v) atomicAdd(&sm[i], v);
  }
  __syncthreads();
  if (threadIdx.x < NC) {
    T.tile_cnt[tile * 8 + threadIdx.x] = sm[threadIdx.x];
    __threadfence();
  }
}

template <int NC>
__device__ void scan_finish(const Tables& T, uint32_t ntiles, const int (&slots)[NC], const long long (&mul)[NC]) {
  __shared__ int s_last2;
  __shared__ unsigned long long s_sum[NC];
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    unsigned int d = atomicAdd(&T.ctl->scan_done, 1u);
    s_last2 = (d == ntiles - 1);
  }
  if (threadIdx.x < NC) s_sum[threadIdx.x] = 0;
  __syncthreads();
  if (s_last2) {
    __threadfence();
    for (int k = 0; k < NC; ++k) {
      unsigned long long acc = 0;
      for (uint32_t t = threadIdx.x; t < ntiles; t += blockDim.x) acc += ((volatile uint32_t*)T.tile_cnt)[t * 8 + k];
      for (int o = 16; o; o >>= 1) acc += __shfl_xor_sync(FULL, acc, o);
      if ((threadIdx.x & 31) == 0 && acc) atomicAdd(&s_sum[k], acc);
    }
    for (uint32_t i = threadIdx.x; i < ntiles; i += blockDim.x) T.tile_status[i] = 0ull;
    __syncthreads();
#pragma unroll
    for (int i = 0; i < NC; ++i)
      if (threadIdx.x == i && slots[i] >= 0) stat_add(T, slots[i], (long long)s_sum[i] * mul[i]);
    if (threadIdx.x == 0) {
      T.ctl->scan_done = 0;
      T.ctl->scan_ticket = 0;
    }
    __threadfence();
  }
}

// ------------------------------------------------------------------------------------
// init / poison
// ------------------------------------------------------------------------------------
__global__ void k_init(Tables T, int nh) {
  size_t tid = blockIdx.x * (size_t)blockDim.x + threadIdx.x, str = (size_t)gridDim.x * blockDim.x;
  for (size_t i = tid; i < T.nblocks; i += str) {
    T.sk[i] = mk_sk(ST_U, 0);
    T.frame_of[i] = UM_NONE;
    T.map[i] = UM_NONE;
    T.hframe[i] = UM_NONE;
    T.pin[i] = 0;
  }
  for (size_t i = tid; i < T.nframes; i += str) T.free_stack[i] = T.nframes - 1 - (uint32_t)i;
  for (size_t i = tid; i < (size_t)nh; i += str) T.hfree_stack[i] = (uint32_t)(nh - 1 - i);
  if (tid == 0) {
    Ctl* c = T.ctl;
    c->used_head = c->used_tail = c->disc_head = c->disc_tail = 0;
    c->free_top = (int)T.nframes;
    c->hfree_top = nh;
    c->n_need = c->n_rekey = c->f0 = c->n_vict = c->n_d2h = c->err = 0;
    c->scan_ticket = c->scan_done = c->app_units = c->vict_done = 0;
    c->minkeep[0] = c->minkeep[1] = ~0ull;
    c->k_want = 0;
    c->need_acc = 0;
    c->reach_tile = ~0u;
    for (int j = 0; j < 8; ++j)
      for (int i = 0; i < S_N; ++i) c->stats[j][i] = 0;
    c->need_cnt[0] = c->need_cnt[1] = 0;
    c->k0_take = c->k0_pend = 0;
    c->vs_combo = 0;
    c->vs_fin = 0;
    c->first_skip = ~0u;
    c->vt_reach = 0;
  }
}

__global__ void k_poison(char* p, size_t bytes) {
  size_t n = bytes / 16;
  uint4 v = make_uint4(0xA5A5A5A5u, 0xA5A5A5A5u, 0xA5A5A5A5u, 0xA5A5A5A5u);
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    reinterpret_cast<uint4*>(p)[i] = v;
}

// ------------------------------------------------------------------------------------
// K1+K2: classify a GPU-destination sub-op and compact its work lists in ascending
// block order (warp ballot/popc-free: per-thread counts + block scan + decoupled
// look-back).  Transitions that need no frame are committed here (refresh, revive
// GE->G with re-map, revalidate GL->G: PAPER L217, L229, L190); blocks that need a
// frame (U/H/HD) are listed for K3/K4.  Every rekeyed block is appended to USED at
// used_tail + rank with key = seq, in ascending block order.
// ------------------------------------------------------------------------------------
// Ordered ranks with a coalesced item mapping: item (k, t) of a tile is element
// tbase + k*TPB + t, so ascending order = (k, warp, lane).  Each warp ballots its 32
// flags per k (two flag kinds A and B); lane 0 stores the packed popc counts
// (A | B << 16) of every k; one warp exclusive-scans the IPT x NW counts in smem.  The
// rank of a flagged item is then  warp offset + popc(ballot & lanes below).  Returns the
// packed tile totals (<= TILE < 2^16 each).
template <int TPB, int IPT>
__device__ __forceinline__ uint32_t ordered_offsets(const unsigned (&ba)[IPT], const unsigned (&bb)[IPT], uint32_t* sm) {
  constexpr int NW = TPB / 32, NE = IPT * NW, PER = (NE + 31) / 32;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  if (lane == 0) {
#pragma unroll
    for (int k = 0; k < IPT; ++k) sm[k * NW + w] = (uint32_t)__popc(ba[k]) | ((uint32_t)__popc(bb[k]) << 16);
  }
  __syncthreads();
  if (w == 0) {
    uint32_t v[PER], sum = 0;
#pragma unroll
    for (int q = 0; q < PER; ++q) {
      const int i = lane * PER + q;
      v[q] = i < NE ? sm[i] : 0u;
      sum += v[q];
    }
    uint32_t x = sum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      uint32_t y = __shfl_up_sync(FULL, x, o);
      if (lane >= o) x += y;
    }
    uint32_t ex = x - sum;
#pragma unroll
    for (int q = 0; q < PER; ++q) {
      const int i = lane * PER + q;
      if (i < NE) sm[i] = ex;
      ex += v[q];
    }
    if (lane == 31) sm[NE] = x;
  }
  __syncthreads();
  return sm[NE];
}

__device__ __forceinline__ unsigned lanemask_lt() {
  unsigned m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// K1/K2 for a sub-op that fits one CTA (k_plan_small): classify, pin, list the blocks
// needing a frame in ascending order, and give every block of the sub-op its USED slot
// tail0 + (its rank in the sub-op) -- the same dead-slot rule as the streaming kernel
// below, so the host knows every ring tail exactly.
template <int TPB, int IPT>
__device__ __forceinline__ void classify_single(const Tables& T, const OpIv& iv, uint32_t g0, uint32_t n, uint32_t seq,
                                                int touch, unsigned long long tail0) {
  constexpr int TILE = TPB * IPT, NW = TPB / 32;
  __shared__ uint32_t s_off[IPT * NW + 1];
  __shared__ uint32_t s_cnt[6];
  // the sub-op's slice of the interval list (<= TILE intervals), staged in smem so the
  // per-item interval search runs in shared memory
  __shared__ uint32_t s_lo[TILE], s_pre[TILE + 1];
  __shared__ uint32_t s_j0, s_m;
  const int w = threadIdx.x >> 5;
  const bool list = iv.blist != nullptr;   // uniform: fault-list form, no interval lookup
  if (!list) {
    if (threadIdx.x == 0) {
      const uint32_t ja = iv.inl ? iv_find(iv, g0) : iv.tj[0];
      const uint32_t jb = iv.inl ? iv_find(iv, g0 + n - 1) : iv.tj[1];
      s_j0 = ja;
      s_m = jb - ja + 1;
    }
    __syncthreads();
    const uint32_t j0 = s_j0, m = s_m;
    for (uint32_t q = threadIdx.x; q <= m; q += blockDim.x) {
      if (q < m) s_lo[q] = iv_lo(iv, j0 + q);
      s_pre[q] = iv_pre(iv, j0 + q);
    }
    __syncthreads();
  }
  const uint32_t m = list ? 0u : s_m;
  const unsigned long long kseq = (unsigned long long)seq << 32;
  uint32_t b[IPT];
  uint8_t s[IPT];
  unsigned bN[IPT];
  uint32_t cls = 0;   // 4 bits per class U H HD G GE GL
  uint32_t jlo = 0;
#pragma unroll
  for (int k = 0; k < IPT; ++k) {
    const uint32_t idx = k * TPB + threadIdx.x;
    b[k] = 0;
    s[k] = 0xff;
    if (idx < n) {
      const uint32_t g = g0 + idx;
      if (list) {
        b[k] = iv.blist[g] & 0x7fffffffu;
      } else {
        uint32_t lo = jlo, hi = m;  // largest j with s_pre[j] <= g (items ascend per thread)
        while (hi - lo > 1) {
          const uint32_t mid = (lo + hi) >> 1;
          if (s_pre[mid] <= g) lo = mid; else hi = mid;
        }
        jlo = lo;
        b[k] = s_lo[lo] + (g - s_pre[lo]);
      }
      s[k] = ld_st(T, b[k]);   // all state loads before any store (stores could alias them)
    }
  }
#pragma unroll
  for (int k = 0; k < IPT; ++k) {
    const uint32_t idx = k * TPB + threadIdx.x;
    bool nd = false;
    if (idx < n) {
      T.pin[b[k]] = seq;
      // a hit (touch of G / GL) keeps its key: its slot is dead from the start
      T.used_ring[(tail0 + idx) & T.cap_mask] = (touch && (s[k] == ST_G || s[k] == ST_GL)) ? kDeadSlot : (kseq | b[k]);
      nd = s[k] <= ST_HD;
      cls += 1u << (4 * s[k]);
    }
    bN[k] = __ballot_sync(FULL, nd);
  }
  const uint32_t tt = ordered_offsets<TPB, IPT>(bN, bN, s_off);
  const unsigned lt = lanemask_lt();
#pragma unroll
  for (int k = 0; k < IPT; ++k) {
    const uint32_t idx = k * TPB + threadIdx.x;
    if (idx >= n) continue;
    const uint32_t bb = b[k];
    const uint8_t ss = s[k];
    if ((bN[k] >> (threadIdx.x & 31)) & 1) {
      const uint32_t pN = (s_off[k * NW + w] & 0xffffu) + __popc(bN[k] & lt);
      T.need[pN] = bb;
      T.needk[pN] = ss;
      T.needhf[pN] = (ss == ST_H) ? T.hframe[bb] : UM_NONE;
    } else if (ss == ST_GE) {   // revive: re-map the frame kept since the discard (L229)
      T.sk[bb] = mk_sk(ST_G, seq);
      T.map[bb] = T.frame_of[bb];
    } else if (!touch) {
      T.sk[bb] = mk_sk(ST_G, seq);   // refresh (G) / revalidate (GL -> G, L190)
    }
  }
  // counters (classes: U H HD G GE GL)
  const long long B = T.B;
  const uint32_t c0 = cls & 15u, c1 = (cls >> 4) & 15u, c2 = (cls >> 8) & 15u, c3 = (cls >> 12) & 15u,
                 c4 = (cls >> 16) & 15u, c5 = (cls >> 20) & 15u;
  uint32_t v[6];
  if (touch) {
    // faults: U+H+HD+GE ; hits: G+GL ; remaps: GE ; h2d: H ; zf: U+HD ; h2d_av: HD
    v[0] = c0 + c1 + c2 + c4; v[1] = c3 + c5; v[2] = c4;
  } else {
    v[0] = c3; v[1] = c4; v[2] = c5;
  }
  v[3] = c1; v[4] = c0 + c2; v[5] = c2;
  const int slots_t[6] = {S_FAULTS, S_HITS, S_REMAPS, S_H2D, S_ZF, S_H2D_AV};
  const int slots_p[6] = {S_REFRESH, S_REMAPS, S_REVAL, S_H2D, S_ZF, S_H2D_AV};
  const long long mul[6] = {1, 1, 1, B, B, B};
  if (threadIdx.x == 0) {
    T.ctl->n_need = tt & 0xffffu;
    T.ctl->n_rekey = n;
  }
  block_counts_to<6>(T, v, s_cnt, touch ? slots_t : slots_p, mul);
}

// ------------------------------------------------------------------------------------
// Streaming K1/K2 for multi-CTA sub-ops: no inter-CTA ordering at all.
//  * USED: every block of the sub-op gets the slot used_tail + (its rank in the sub-op)
//    with entry (seq, b), rekeyed or not.  The rank is the block's position in the
//    sorted distinct list, so the slots are in ascending block order; an entry whose
//    block does not take key = seq in state G here is dead by the liveness rule
//    (st == G && key == entry key) and stays dead, since seq is never reissued.
//  * need list: its order is not observable (frame ids and the victim<->newcomer
//    pairing are internal), so slots come from one atomic per CTA.
//  * counters: per-tile partials summed by the last CTA (no same-address atomics).
// ------------------------------------------------------------------------------------

// Exclusive CTA scan of one 32-bit count per thread; returns the prefix, total in `tot`.
template <int TPB>
__device__ __forceinline__ uint32_t cta_excl_scan(uint32_t v, uint32_t& tot, uint32_t* sm /*[TPB/32]*/) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint32_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint32_t y = __shfl_up_sync(FULL, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) sm[w] = x;
  __syncthreads();
  if (w == 0) {
    uint32_t t = lane < TPB / 32 ? sm[lane] : 0u;
    uint32_t ti = t;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      uint32_t y = __shfl_up_sync(FULL, ti, o);
      if (lane >= o) ti += y;
    }
    if (lane < TPB / 32) sm[lane] = ti - t;   // exclusive warp offsets
    if (lane == TPB / 32 - 1) sm[TPB / 32] = ti;
  }
  __syncthreads();
  const uint32_t pre = sm[w] + x - v;
  tot = sm[TPB / 32];
  __syncthreads();
  return pre;
}

// Last-CTA epilogue of a streaming launch: the CTA that finishes last (completion
// ticket) sums the per-tile counter partials and adds them once.  Returns true in
// that CTA (uniformly), so the caller can publish launch-wide results.
template <int NC>
__device__ bool grid_finish(const Tables& T, const int (&slots)[NC], const long long (&mul)[NC]) {
  __shared__ int s_last;
  __shared__ unsigned long long s_sum[NC];
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    s_last = atomicAdd(&T.ctl->scan_done, 1u) == gridDim.x - 1;
  }
  if (threadIdx.x < NC) s_sum[threadIdx.x] = 0;
  __syncthreads();
  if (!s_last) return false;
  __threadfence();
  const uint32_t nt = gridDim.x;
  for (int k = 0; k < NC; ++k) {
    unsigned long long acc = 0;
    for (uint32_t t = threadIdx.x; t < nt; t += blockDim.x) acc += ((volatile uint32_t*)T.tile_cnt)[t * 8 + k];
    for (int o = 16; o; o >>= 1) acc += __shfl_xor_sync(FULL, acc, o);
    if ((threadIdx.x & 31) == 0 && acc) atomicAdd(&s_sum[k], acc);
  }
  __syncthreads();
#pragma unroll
  for (int i = 0; i < NC; ++i)
    if (threadIdx.x == i && slots[i] >= 0) stat_add(T, slots[i], (long long)s_sum[i] * mul[i]);
  if (threadIdx.x == 0) T.ctl->scan_done = 0;
  return true;
}

template <int IPT, bool LIST, int TPB>
__device__ __forceinline__ void classify_body(const Tables& T, const OpIv& iv, uint32_t g0, uint32_t n, uint32_t seq,
                                              int touch, unsigned long long tail0, int npar, int k0) {
  constexpr int TILE = TPB * IPT, NW = TPB / 32, NWORD = TILE / 32;
  constexpr int PERL = (NWORD + 31) / 32;   // bitmap words per lane in the warp prefix
  // Interval lookup without a search: the tile's interval slice [ja, jb] is staged as
  // d[q] = lo - pre (block = rank + d), and the start of every slice interval but the
  // first sets one bit of a TILE-bit map at its in-tile position.  The interval of item
  // i is then the number of set bits in [0, i] (a prefix of word popcounts plus one
  // masked popc), so every item costs O(1) instead of a log2(TILE)-step dependent search.
  __shared__ uint32_t s_d[TILE];
  __shared__ uint32_t s_bits[NWORD];
  __shared__ uint32_t s_wpre[NWORD];
  __shared__ uint32_t s_base;
  __shared__ uint32_t s_off[IPT * NW + 1];
  __shared__ uint32_t s_cnt[2 * NW];
  const uint32_t tile = blockIdx.x, tbase = tile * TILE, gt = g0 + tbase;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint32_t b[IPT];
  if constexpr (LIST) {
    // fault-list form: one coalesced load per item, no interval slice, no barrier
#pragma unroll
    for (int k = 0; k < IPT; ++k) {
      const uint32_t idx = tbase + k * TPB + threadIdx.x;
      b[k] = idx < n ? iv.blist[g0 + idx] & 0x7fffffffu : 0u;
    }
  } else {
    const uint32_t ja = iv.inl ? iv_find(iv, gt) : iv.tj[2 * tile];
    const uint32_t jb = iv.inl ? iv_find(iv, g0 + min(n, tbase + TILE) - 1) : iv.tj[2 * tile + 1];
    const uint32_t m = jb - ja + 1;   // <= TILE (every slice interval holds an item of the tile)
    uint32_t qlo[IPT], qpre[IPT];
#pragma unroll
    for (int r = 0; r < IPT; ++r) {
      const uint32_t q = r * TPB + threadIdx.x;
      if (q < m) {
        qlo[r] = iv_lo(iv, ja + q);
        qpre[r] = iv_pre(iv, ja + q);
      }
    }
    for (int i = threadIdx.x; i < NWORD; i += TPB) s_bits[i] = 0u;
    __syncthreads();
#pragma unroll
    for (int r = 0; r < IPT; ++r) {
      const uint32_t q = r * TPB + threadIdx.x;
      if (q < m) {
        s_d[q] = qlo[r] - qpre[r];
        if (q) {
          const uint32_t pos = qpre[r] - gt;   // in (0, TILE)
          atomicOr(&s_bits[pos >> 5], 1u << (pos & 31));
        }
      }
    }
    __syncthreads();
    if (PERL > 1 && w == 0) {
      // one warp: exclusive prefix of the word popcounts (PERL consecutive words per lane)
      uint32_t c[PERL], sum = 0;
#pragma unroll
      for (int i = 0; i < PERL; ++i) {
        c[i] = lane * PERL + i < NWORD ? __popc(s_bits[lane * PERL + i]) : 0u;
        sum += c[i];
      }
      uint32_t x = sum;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(FULL, x, o);
        if (lane >= o) x += y;
      }
      x -= sum;
#pragma unroll
      for (int i = 0; i < PERL; ++i) {
        if (lane * PERL + i < NWORD) s_wpre[lane * PERL + i] = x;
        x += c[i];
      }
    }
    if (PERL > 1) __syncthreads();
    uint32_t wexcl = 0;   // PERL == 1: lane l holds the set bits in words [0, l)
    if (PERL == 1) {
      const uint32_t c = lane < NWORD ? __popc(s_bits[lane]) : 0u;
      uint32_t x = c;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(FULL, x, o);
        if (lane >= o) x += y;
      }
      wexcl = x - c;
    }
    const unsigned le = lanemask_lt() | (1u << lane);
#pragma unroll
    for (int k = 0; k < IPT; ++k) {
      const uint32_t idx = tbase + k * TPB + threadIdx.x;
      const int wi = k * NW + w;   // bitmap word of item (k, thread): in-tile position k*TPB + tid
      const uint32_t wp = PERL == 1 ? __shfl_sync(FULL, wexcl, wi & 31) : s_wpre[wi];
      const uint32_t j = wp + __popc(s_bits[wi] & le);
      b[k] = g0 + idx + s_d[j];
    }
  }
  const unsigned long long kseq = (unsigned long long)seq << 32;
  uint8_t s[IPT];
  uint32_t cls = 0;   // per-class counts (<= IPT < 32 each), 5 bits per class U H HD G GE GL
#pragma unroll
  for (int k = 0; k < IPT; ++k) {
    const uint32_t idx = tbase + k * TPB + threadIdx.x;
    s[k] = idx < n ? ld_st(T, b[k]) : (uint8_t)0xff;
  }
  // second dependent loads, all issued before any store (stores could alias them): the
  // host frame of an H block, the kept frame of a GE block
  uint32_t aux[IPT];
#pragma unroll
  for (int k = 0; k < IPT; ++k) {
    aux[k] = UM_NONE;
    if (s[k] == ST_H) aux[k] = T.hframe[b[k]];
    else if (s[k] == ST_GE) aux[k] = T.frame_of[b[k]];
  }
  unsigned bN[IPT];
#pragma unroll
  for (int k = 0; k < IPT; ++k) {
    const uint32_t idx = tbase + k * TPB + threadIdx.x;
    if (idx < n) {
      T.pin[b[k]] = seq;
      // a hit (touch of G / GL) keeps its key: its slot is dead from the start
      T.used_ring[(tail0 + idx) & T.cap_mask] = (touch && (s[k] == ST_G || s[k] == ST_GL)) ? kDeadSlot : (kseq | b[k]);
      cls += 1u << (5 * s[k]);
    }
    bN[k] = __ballot_sync(FULL, s[k] <= ST_HD);   // 0xff (no item) is > ST_HD
  }
  // need-list slots: one atomic per CTA for the base, then warp-ballot ranks so that
  // consecutive lanes write consecutive slots (coalesced stores)
  const uint32_t tot = ordered_offsets<TPB, IPT>(bN, bN, s_off) & 0xffffu;
  if (threadIdx.x == 0) {
    if (k0) {
      // k = 0 is certain (the host's bound), so no victim kernel runs: one 64-bit atomic
      // gives this CTA its need-list base (high word) and a ticket (low word); the CTA
      // with the last ticket knows the sub-op's need count and does the victim kernels'
      // k = 0 bookkeeping.  Nothing else in this launch reads what it writes.
      Ctl* c = T.ctl;
      const unsigned long long old = atomicAdd(&c->need_tk, ((unsigned long long)tot << 32) | 1ull);
      s_base = (uint32_t)(old >> 32);
      if ((uint32_t)old == gridDim.x - 1) {
        const uint32_t nn = s_base + tot;
        const int f0 = c->free_top;
        c->n_need = nn;
        c->need_cnt[npar ^ 1] = 0;   // the other parity slot, as the victim kernels do
        c->n_vict = 0;
        c->f0 = (uint32_t)f0;
        c->free_top = f0 - (int)min((uint32_t)f0, nn);
        c->used_tail += n;
        c->need_tk = 0;
      }
    } else {
      s_base = tot ? atomicAdd(&T.ctl->need_cnt[npar], tot) : 0u;
    }
  }
  __syncthreads();
  const uint32_t base = s_base;
  const unsigned lt = lanemask_lt();
#pragma unroll
  for (int k = 0; k < IPT; ++k) {
    const uint8_t ss = s[k];
    if (ss == 0xff) continue;
    const uint32_t bb = b[k];
    if (ss <= ST_HD) {
      const uint32_t pos = base + (s_off[k * (TPB / 32) + w] & 0xffffu) + __popc(bN[k] & lt);
      T.need[pos] = bb;
      T.needk[pos] = ss;
      T.needhf[pos] = aux[k];
    } else if (ss == ST_GE) {      // revive: re-map the frame kept since the discard (L229)
      T.sk[bb] = mk_sk(ST_G, seq);
      T.map[bb] = aux[k];
    } else if (!touch) {
      T.sk[bb] = mk_sk(ST_G, seq);   // refresh (G) / revalidate (GL -> G, L190)
    }
  }
  // counters (classes: U H HD G GE GL).  A thread's class counts (<= IPT each) are
  // repacked 8 bits per class into two words and warp-summed (<= 32 * IPT = 128 per
  // class); thread 0 sums the warps' words from shared memory and adds the counters:
  // two reductions and one barrier instead of one reduction per counter
  static_assert(32 * IPT < 256, "8-bit class lanes");
  const uint32_t lo4 = (cls & 31u) | (((cls >> 5) & 31u) << 8) | (((cls >> 10) & 31u) << 16) |
                       (((cls >> 15) & 31u) << 24);
  const uint32_t hi2 = ((cls >> 20) & 31u) | (((cls >> 25) & 31u) << 8);
  const uint32_t wl = __reduce_add_sync(FULL, lo4), wh = __reduce_add_sync(FULL, hi2);
  if (lane == 0) {
    s_cnt[w] = wl;          // s_cnt: 2 * NW words
    s_cnt[NW + w] = wh;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t c0 = 0, c1 = 0, c2 = 0, c3 = 0, c4 = 0, c5 = 0;
#pragma unroll
    for (int i = 0; i < NW; ++i) {
      const uint32_t a = s_cnt[i], e = s_cnt[NW + i];
      c0 += a & 255u; c1 += (a >> 8) & 255u; c2 += (a >> 16) & 255u; c3 += a >> 24;
      c4 += e & 255u; c5 += e >> 8;
    }
    const long long B = T.B;
    // only non-zero counters (a uniform batch, e.g. all U, adds two instead of six)
    auto add = [&](int slot, long long v) {
      if (v) stat_add(T, slot, v);
    };
    if (touch) {
      // faults: U+H+HD+GE ; hits: G+GL ; remaps: GE
      add(S_FAULTS, c0 + c1 + c2 + c4);
      add(S_HITS, c3 + c5);
      add(S_REMAPS, c4);
    } else {
      add(S_REFRESH, c3);   // refreshes, remaps, revalidations
      add(S_REMAPS, c4);
      add(S_REVAL, c5);
    }
    add(S_H2D, (long long)c1 * B);          // h2d, zf, h2d_avoided
    add(S_ZF, (long long)(c0 + c2) * B);
    add(S_H2D_AV, (long long)c2 * B);
    if (blockIdx.x == 0) T.ctl->n_rekey = n;   // USED slots appended
  }
}

// 4 items per thread, 8 CTAs/SM (A/B on B200: 8 items per thread at 6 CTAs/SM spills and
// runs the 2^21-block touch in 42 vs 30 us); the interval form (bitmap prefix, one more
// live array) runs 6 CTAs/SM (40 registers) so that it does not spill
template <bool LIST, int TPB>
__global__ void __launch_bounds__(TPB, (LIST ? 2048 : 1536) / TPB) k_classify(Tables T, const __grid_constant__ OpIv iv, uint32_t g0,
                                                              uint32_t n, uint32_t seq, int touch,
                                                              unsigned long long tail0, int npar, int k0) {
  pdl_enter();
  classify_body<4, LIST, TPB>(T, iv, g0, n, seq, touch, tail0, npar, k0);
}

// ------------------------------------------------------------------------------------
// K3: victim selection + reclaim (PAPER §5.5: free -> (unused, empty) ->
// discarded FIFO -> used LRU; §5.3: discarded victims need no transfer; A10:
// valid victims are written back).  One CTA scans each ring from its head in windows,
// ranks live & unpinned entries with a block scan and takes the first k; the head
// advances over the maximal prefix of dead or consumed entries.
// ------------------------------------------------------------------------------------
__device__ __forceinline__ void victims_body(const Tables& T, uint32_t seq, int evict_mode, uint32_t want) {
  __shared__ unsigned long long s_scan[kVictTPB / 32];
  __shared__ unsigned long long s_minkeep;
  __shared__ uint32_t s_cnt[4];
  Ctl* c = T.ctl;
  const int f0 = c->free_top;
  const uint32_t nn = evict_mode ? 0u : c->n_need;
  uint32_t k;
  if (evict_mode) k = want > (uint32_t)f0 ? want - (uint32_t)f0 : 0u;
  else k = nn > (uint32_t)f0 ? nn - (uint32_t)f0 : 0u;
  uint32_t found = 0;
  const uint32_t W = kVictTPB * kVictIPT;
  for (int r = 0; r < 2; ++r) {
    const int ring = r == 0 ? RING_DISC : RING_USED;
    uint64_t* R = ring == RING_DISC ? T.disc_ring : T.used_ring;
    unsigned long long* headp = ring == RING_DISC ? &c->disc_head : &c->used_head;
    const unsigned long long head = *headp;
    const unsigned long long tail = ring == RING_DISC ? c->disc_tail : c->used_tail;
    unsigned long long pos = head, newhead = head;
    bool blocked = false;
    while (found < k && pos < tail) {
      const uint32_t w = (uint32_t)min((unsigned long long)W, tail - pos);
      const uint32_t first = threadIdx.x * kVictIPT;
      // three load phases (ring entries, their state words, pins of live entries), each
      // with all kVictIPT loads of a thread in flight
      uint32_t bb[kVictIPT], kk[kVictIPT], wv[kVictIPT];
      unsigned candm = 0, livem = 0;
      uint32_t cc = 0;
#pragma unroll
      for (int q = 0; q < kVictIPT; ++q) {
        const unsigned long long e = first + q < w ? R[(pos + first + q) & T.cap_mask] : ~0ull;
        bb[q] = (uint32_t)e;
        kk[q] = (uint32_t)(e >> 32);
      }
#pragma unroll
      for (int q = 0; q < kVictIPT; ++q) wv[q] = bb[q] != UM_NONE ? T.sk[bb[q]] : 0u;
#pragma unroll
      for (int q = 0; q < kVictIPT; ++q) {
        const uint8_t ss = st_of(wv[q]);
        const bool live = bb[q] != UM_NONE && (ring == RING_DISC ? (ss == ST_GE || ss == ST_GL) : ss == ST_G) &&
                          key_of(wv[q]) == kk[q];
        livem |= (unsigned)live << q;
        wv[q] = live ? T.pin[bb[q]] : UM_NONE;
      }
#pragma unroll
      for (int q = 0; q < kVictIPT; ++q) {
        const bool cand = wv[q] < T.pfloor;   // live and not pinned by an in-flight sub-op
        candm |= (unsigned)cand << q;
        cc += cand;
      }
      unsigned long long tot;
      uint32_t rank = (uint32_t)block_excl_scan<kVictTPB>(cc, tot, s_scan);
      if (threadIdx.x == 0) s_minkeep = ~0ull;
      __syncthreads();
      unsigned long long mykeep = ~0ull;
#pragma unroll
      for (int q = 0; q < kVictIPT; ++q) {
        bool sel = false;
        if ((candm >> q) & 1) {
          uint32_t rr = found + rank++;
          if (rr < k) {
            T.victim[rr] = bb[q];
            sel = true;
          }
        }
        if (((livem >> q) & 1) && !sel && mykeep == ~0ull) mykeep = pos + first + q;
      }
      if (mykeep != ~0ull) atomicMin(&s_minkeep, mykeep);
      __syncthreads();
      if (!blocked) {
        if (s_minkeep != ~0ull) {
          newhead = s_minkeep;
          blocked = true;
        } else {
          newhead = pos + w;
        }
      }
      found = (uint32_t)min((unsigned long long)k, found + tot);
      pos += w;
      __syncthreads();
    }
    if (threadIdx.x == 0) *headp = newhead;
  }
  __syncthreads();
  // Reclaim the victims.  G victims are written back (A10).  In a GPU sub-op victim j's
  // frame goes to need item f0 + j; when that item migrates in from a host frame, the
  // fused swap exchanges the two (the victim's bytes land in the host frame the new
  // block's bytes leave), so no host frame is allocated for it.  Other G victims take
  // host frames from the free stack in victim order.
  const int htop = c->hfree_top;
  uint32_t gbase = 0, abase = 0;
  uint32_t nGL = 0;
  for (uint32_t base = 0; base < found; base += kVictTPB) {
    const uint32_t j = base + threadIdx.x;
    uint32_t v = 0, fr = UM_NONE, swap_hf = UM_NONE;
    uint8_t ss = 0;
    uint32_t isG = 0, needA = 0;
    if (j < found) {
      v = T.victim[j];
      const uint8_t nk = evict_mode ? (uint8_t)0xff : T.needk[(uint32_t)f0 + j];   // independent of v
      ss = ld_st(T, v);
      fr = T.frame_of[v];
      isG = ss == ST_G;
      if (isG && nk == ST_H) swap_hf = T.needhf[(uint32_t)f0 + j];
      needA = isG && swap_hf == UM_NONE;
    }
    unsigned long long tot, totA;
    uint32_t gr = (uint32_t)block_excl_scan<kVictTPB>(isG, tot, s_scan) + gbase;
    uint32_t ar = (uint32_t)block_excl_scan<kVictTPB>(needA, totA, s_scan) + abase;
    if (j < found) {
      uint32_t hf = swap_hf;
      if (needA) {
        int idx = htop - 1 - (int)ar;
        if (idx >= 0) hf = T.hfree_stack[idx];
        else atomicExch(&c->err, 2u);  // host-frame pool exhausted -> UM_ENOMEM
      }
      T.vframe[j] = fr;
      T.vkind[j] = ss;
      T.vhf[j] = hf;
      T.sk[v] = mk_sk(isG ? ST_H : ST_HD, 0);
      if (T.phz) T.phz[v] = 0u;   // written back whole (dead pages read as zero by rule)
      T.map[v] = UM_NONE;
      T.frame_of[v] = UM_NONE;
      T.hframe[v] = hf;
      nGL += ss == ST_GL;
      if (evict_mode) {
        T.free_stack[f0 + j] = fr;
        if (isG) {
          T.d2h_frame[gr] = fr;
          T.d2h_hf[gr] = hf;
          d2h_listed(T, seq, v, gr, ss);
        }
      }
    }
    gbase += (uint32_t)tot;
    abase += (uint32_t)totA;
  }
  {
    uint32_t v[4] = {threadIdx.x == 0 ? found : 0u, threadIdx.x == 0 ? gbase : 0u,
                     threadIdx.x == 0 ? found - gbase : 0u, nGL};
    const int slots[4] = {S_EVICT, S_D2H, S_D2H_AV, S_UNMAPS};
    const long long mul[4] = {1, (long long)T.B, (long long)T.B, 1};
    block_counts_to<4>(T, v, s_cnt, slots, mul);
  }
  if (threadIdx.x == 0) {
    c->hfree_top = max(0, htop - (int)abase);
    if (evict_mode) {
      c->free_top = f0 + (int)found;
      c->n_d2h = gbase;
    } else {
      c->f0 = (uint32_t)f0;
      c->n_vict = found;
      c->free_top = f0 - (int)min((uint32_t)f0, nn);
      c->used_tail += c->n_rekey;
    }
  }
}

__global__ void __launch_bounds__(kVictTPB) k_victims(Tables T, uint32_t seq, int evict_mode, uint32_t want,
                                                      int npar) {
  pdl_enter();
  if (!evict_mode && threadIdx.x == 0) {
    // publish the streaming classify's need count; clear the other parity slot for the
    // next multi-CTA sub-op (nothing reads it until then)
    T.ctl->n_need = T.ctl->need_cnt[npar];
    T.ctl->need_cnt[npar ^ 1] = 0;
  }
  __syncthreads();
  victims_body(T, seq, evict_mode, want);
}

// K1+K2+K3 for a sub-op that fits one tile: one CTA classifies, compacts and selects
// victims (saves a launch per small op; same code as the multi-CTA kernels).
__global__ void __launch_bounds__(kVictTPB) k_plan_small(Tables T, const __grid_constant__ OpIv iv, uint32_t g0, uint32_t n, uint32_t seq,
                                                         int touch, unsigned long long tail0) {
  pdl_enter();
  classify_single<kVictTPB, kSmallPlan / kVictTPB>(T, iv, g0, n, seq, touch, tail0);
  __syncthreads();
  __threadfence_block();
  victims_body(T, seq, 0, 0);
}

// ------------------------------------------------------------------------------------
// K3 (wide): the same victim rule for large sub-ops, over all SMs, without a look-back
// chain.  The victims are the first k candidates (live, not pinned) of DISC[head,tail)
// ++ USED[head,tail) (PAPER §5.5); which of them comes first in the victim
// list is not observable (frame ids and the victim <-> newcomer pairing are internal),
// only the set is.
//  Pass 1 (k_victims_scan): a persistent grid takes tiles of 2048 entries in ascending
//   order from a ticket; each tile writes its candidates' blocks, in ring order, to its
//   own scratch slice, and its candidate count and first kept-live positions to its
//   tile record, then adds the count to a running total.  A tile is not read at all if
//   the total of the (earlier-ticketed) tiles finished so far already reaches k: the k-th
//   candidate lies before it.  No tile waits for another.  The last CTA to finish scans
//   the tile counts, finds the tile holding the k-th candidate (reach), writes every
//   tile's exclusive candidate prefix, advances the ring heads and does the frame
//   bookkeeping.
//  Pass 2 (k_victims_apply): tile t <= reach reclaims its first min(count, k - prefix)
//   candidates as victims prefix .. prefix + take - 1, gathered from its scratch slice.
// ------------------------------------------------------------------------------------
constexpr int kVsTPB = 256, kVsIPT = 8, kVsTile = kVsTPB * kVsIPT;   // victim scan tiles
#ifdef UM_VS_TRACE
// Diagnostic build only (tools/vs_trace.py): per-CTA %globaltimer stamps of the victim
// kernels.  [4b] start, [4b+1] end, [4b+2] tiles, [4b+3] end of the first tile of scan
// CTA b; [6000 + 2b] apply CTA b; [8000], [8007], [8001] finalize start, after the tile
// passes, end; [8002], [8003] examined tiles, k.
__device__ unsigned long long g_vs_tr[8192];
__device__ __forceinline__ unsigned long long vs_now() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#define VS_TR(i, v) (g_vs_tr[(i)] = (unsigned long long)(v))
#else
#define VS_TR(i, v) ((void)0)
#endif
constexpr int kVaPass = 128;   // victims per warp pass of k_victims_apply

__global__ void __launch_bounds__(kVsTPB, 4) k_victims_scan(Tables T, uint32_t seq, int evict_mode, uint32_t want,
                                                            int npar, int prefetch) {
  pdl_enter();
#ifdef UM_VS_TRACE
  uint32_t tr_tiles = 0;
  if (threadIdx.x == 0 && blockIdx.x < 1500) VS_TR(4 * blockIdx.x, vs_now());
#endif
  constexpr int NW = kVsTPB / 32;
  __shared__ uint32_t s_off[kVsIPT * NW + 1];
  __shared__ unsigned long long s_dh, s_ld, s_uh, s_lu, s_mk[2];
  __shared__ uint32_t s_k, s_nn, s_f0, s_tile, s_skip;
  __shared__ int s_last;
  Ctl* c = T.ctl;
  if (threadIdx.x == 0) {
    s_dh = c->disc_head;
    s_ld = c->disc_tail - c->disc_head;
    s_uh = c->used_head;
    s_lu = c->used_tail - c->used_head;
    const uint32_t f0 = (uint32_t)c->free_top;
    const uint32_t nn = evict_mode ? want : c->need_cnt[npar];
    s_k = nn > f0 ? nn - f0 : 0u;
    s_nn = nn;
    s_f0 = f0;
    if (blockIdx.x == 0 && !evict_mode) {
      c->n_need = nn;              // publish the streaming classify's need count
      c->need_cnt[npar ^ 1] = 0;   // and clear the other parity slot (read by no one now)
    }
  }
  __syncthreads();
  if (s_k == 0) {
    // nothing to evict (the sub-op's need fits the free frames): one CTA records an
    // empty victim list, the others exit.  free_top and used_tail are advanced by
    // k_victims_apply, which runs after this grid completes (other CTAs of this grid may
    // still be reading free_top).
    if (blockIdx.x == 0 && threadIdx.x == 0) {
      c->n_vict = 0;
      c->f0 = s_f0;
      c->k0_take = evict_mode ? 0u : min(s_f0, s_nn);
      c->k0_pend = evict_mode ? 0u : 1u;
    }
    return;
  }
  const unsigned long long L = s_ld + s_lu;
  const uint32_t k = s_k;
  const uint32_t ntiles = (uint32_t)((L + kVsTile - 1) / kVsTile);
  const int w = threadIdx.x >> 5;
  const unsigned lt = lanemask_lt();
  const unsigned me = 1u << (threadIdx.x & 31);
  // CTA b starts on tile b (every grid CTA is resident); later tiles come from a ticket,
  // tile gridDim.x + t.  Tickets and the running candidate total share one 64-bit word,
  // so a ticket comes with a consistent snapshot: every count in it was added by a
  // finished tile, which has a smaller index.  If the snapshot reaches k, tiles [0, t)
  // hold >= k candidates and tile t is not read.
  if (threadIdx.x == 0) {
    s_tile = blockIdx.x;
    s_skip = 0;
  }
  while (true) {
    __syncthreads();
    const uint32_t tile = s_tile, snap = s_skip;
    __syncthreads();   // s_tile / s_skip are rewritten below
    if (tile >= ntiles) break;
    if (snap >= k) {   // later tickets skip as well
      if (threadIdx.x == 0) atomicMin(&c->first_skip, tile);
      break;
    }
    unsigned long long nxt = 0;
#ifdef UM_VS_TRACE
    ++tr_tiles;
#endif
    if (threadIdx.x == 0) {
      if (prefetch) nxt = atomicAdd(&c->vs_combo, 1ull);
      s_mk[0] = s_mk[1] = ~0ull;
    }
    const unsigned long long tbase = (unsigned long long)tile * kVsTile;
    // three load phases, each with all kVsIPT loads in flight: ring entries, the state
    // words of their blocks (liveness), the pin words of live entries
    uint32_t bb[kVsIPT], kk[kVsIPT], wv[kVsIPT];
    unsigned bC[kVsIPT], bL[kVsIPT];
#pragma unroll
    for (int q = 0; q < kVsIPT; ++q) {
      const unsigned long long idx = tbase + q * kVsTPB + threadIdx.x;
      unsigned long long e = ~0ull;
      if (idx < L) {
        const bool disc = idx < s_ld;
        const unsigned long long pos = disc ? s_dh + idx : s_uh + (idx - s_ld);
        e = (disc ? T.disc_ring : T.used_ring)[pos & T.cap_mask];
      }
      bb[q] = (uint32_t)e;
      kk[q] = (uint32_t)(e >> 32);
    }
#pragma unroll
    for (int q = 0; q < kVsIPT; ++q) wv[q] = bb[q] != UM_NONE ? T.sk[bb[q]] : 0u;
#pragma unroll
    for (int q = 0; q < kVsIPT; ++q) {
      const unsigned long long idx = tbase + q * kVsTPB + threadIdx.x;
      const uint8_t ss = st_of(wv[q]);
      const bool live = bb[q] != UM_NONE && (idx < s_ld ? (ss == ST_GE || ss == ST_GL) : ss == ST_G) &&
                        key_of(wv[q]) == kk[q];
      wv[q] = live ? T.pin[bb[q]] : UM_NONE;   // not a candidate unless live and unpinned
      bL[q] = __ballot_sync(FULL, live);
    }
#pragma unroll
    for (int q = 0; q < kVsIPT; ++q) bC[q] = __ballot_sync(FULL, wv[q] < T.pfloor);
    const uint32_t cnt = ordered_offsets<kVsTPB, kVsIPT>(bC, bC, s_off) & 0xffffu;
    unsigned long long mk0 = ~0ull, mk1 = ~0ull;   // first live entry kept (pinned), per ring
    uint32_t* scr = T.vscratch + tbase;
#pragma unroll
    for (int q = 0; q < kVsIPT; ++q) {
      if (bC[q] & me) scr[(s_off[q * NW + w] & 0xffffu) + __popc(bC[q] & lt)] = bb[q];
      else if (bL[q] & me) {
        const unsigned long long idx = tbase + q * kVsTPB + threadIdx.x;
        if (idx < s_ld) mk0 = min(mk0, idx);
        else mk1 = min(mk1, idx);
      }
    }
    if (mk0 != ~0ull) atomicMin(&s_mk[0], mk0);
    if (mk1 != ~0ull) atomicMin(&s_mk[1], mk1);
    __syncthreads();
    if (threadIdx.x == 0) {
      uint32_t* rec = T.tile_cnt + (size_t)tile * 8;
      rec[0] = cnt;
      *reinterpret_cast<unsigned long long*>(rec + 2) = s_mk[0];
      *reinterpret_cast<unsigned long long*>(rec + 4) = s_mk[1];
      // no fence: the records are read by the finalizing CTA after the completion
      // counter below (fenced), the scratch slice by k_victims_apply (next launch)
      // without prefetch the next ticket comes with this tile's count (one atomic)
      if (prefetch) {
        if (cnt) atomicAdd(&c->vs_combo, (unsigned long long)cnt << 32);
      } else {
        // Paced tickets: a CTA takes the next tile only while the tiles already handed
        // out are not expected to hold the k-th candidate (estimate: the candidate
        // density of the finished tiles); otherwise it waits until they finish (every
        // grid CTA is resident, and tiles in flight depend on nothing) and takes a
        // ticket then only if the count still falls short.  Without the pacing, CTAs
        // that finish early take tickets before the wave's counts are in, about
        // doubling the tiles read past the k-th candidate.
        unsigned long long v = atomicAdd(&c->vs_combo, (unsigned long long)cnt << 32) + ((unsigned long long)cnt << 32);
        unsigned int fin = atomicAdd(&c->vs_fin, 1u) + 1u;
        while (true) {
          const unsigned long long tot = v >> 32;
          const unsigned int issued = (unsigned int)min((unsigned long long)ntiles, (unsigned long long)gridDim.x + (uint32_t)v);
          const unsigned int inflight = issued > fin ? issued - fin : 0u;
          if (tot >= k || issued >= ntiles && inflight == 0) {
            nxt = v | 0xffffffffull;   // stop: enough candidates, or every tile handed out
            break;
          }
          if (!inflight || tot + (unsigned long long)inflight * tot / fin < k) {
            nxt = atomicAdd(&c->vs_combo, 1ull);
            break;
          }
          __nanosleep(128);
          v = *(volatile unsigned long long*)&c->vs_combo;
          fin = *(volatile unsigned int*)&c->vs_fin;
        }
      }
      s_tile = (uint32_t)nxt == 0xffffffffu ? ntiles : gridDim.x + (uint32_t)nxt;
      s_skip = (uint32_t)(nxt >> 32);
#ifdef UM_VS_TRACE
      if (tr_tiles == 1 && blockIdx.x < 1500) VS_TR(4 * blockIdx.x + 3, vs_now());
#endif
    }
  }
  // completion: the last CTA of the grid finalizes
  __syncthreads();
#ifdef UM_VS_TRACE
  if (threadIdx.x == 0 && blockIdx.x < 1500) {
    VS_TR(4 * blockIdx.x + 1, vs_now());
    VS_TR(4 * blockIdx.x + 2, tr_tiles);
  }
#endif
  if (threadIdx.x == 0) {
    __threadfence();
    s_last = atomicAdd(&c->scan_done, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (!s_last) return;
  __threadfence();
#ifdef UM_VS_TRACE
  if (threadIdx.x == 0) VS_TR(8000, vs_now());
#endif
  __shared__ unsigned long long s_sc[kVsTPB / 32];
  __shared__ uint32_t s_reach;
  __shared__ unsigned long long s_kd, s_ku;
  const uint32_t fs = *(volatile uint32_t*)&c->first_skip;
  // tiles [0, E) were all examined: below the first skipped ticket and below the first
  // tile never handed out (paced tickets may stop short of both)
  const unsigned long long handed = (unsigned long long)gridDim.x + (uint32_t)*(volatile unsigned long long*)&c->vs_combo;
  const uint32_t E = (uint32_t)min(min((unsigned long long)ntiles, (unsigned long long)fs), handed);
  if (threadIdx.x == 0) {
    s_reach = ~0u;
    s_kd = s_ku = ~0ull;
  }
  __syncthreads();
  // Tiles [0, E) in chunks of kFinS (one chunk up to 2048 tiles = 4M ring entries):
  //  1. stage the chunk's candidate counts in shared memory (a strided load: all of a
  //     thread's loads in flight, neighbouring lanes on neighbouring records);
  //  2. each thread takes a contiguous run of kFinR tiles: block scan -> exclusive
  //     candidate prefix ex (plus the carry of earlier chunks); per tile take = the
  //     victims it supplies (ex >= k: none, else min(count, k - ex)), the reach tile (ex
  //     < k <= ex + count), and its apply passes of <= kVaPass victims; a second block
  //     scan places them in the work table, one 16-byte entry per pass {victim base,
  //     tile, scratch offset, count}, so the apply's warps are balanced whatever the
  //     spread of victims over tiles (a dense tile holds up to 2048);
  //  3. inclusive prefixes back to shared memory; the first kept live entry of every
  //     tile before the reach tile (inclusive prefix < k) is min-reduced with strided
  //     loads again.
  // L2 reads (ld.global.cg): written by other CTAs of this grid, ordered by the fenced
  // completion counter.
  constexpr int kFinR = 8, kFinS = kFinR * kVsTPB;
  __shared__ __align__(16) uint32_t s_fc[kFinS];
  const uint32_t* tc = T.tile_cnt;
  unsigned long long carry = 0, pcarry = 0, kd = ~0ull, ku = ~0ull;
  for (uint32_t c0 = 0; c0 < E; c0 += kFinS) {
    const uint32_t ce = min((uint32_t)kFinS, E - c0);
    {
      uint32_t v[kFinR];
#pragma unroll
      for (int q = 0; q < kFinR; ++q) {
        const uint32_t i = q * kVsTPB + threadIdx.x;
        v[q] = i < ce ? __ldcg(tc + (size_t)(c0 + i) * 8) : 0u;
      }
#pragma unroll
      for (int q = 0; q < kFinR; ++q) s_fc[q * kVsTPB + threadIdx.x] = v[q];
    }
    __syncthreads();
    uint32_t v[kFinR], sum = 0;
    {
      const uint4* r = reinterpret_cast<const uint4*>(s_fc + threadIdx.x * kFinR);
      const uint4 a = r[0], b = r[1];
      v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w; v[4] = b.x; v[5] = b.y; v[6] = b.z; v[7] = b.w;
    }
#pragma unroll
    for (int q = 0; q < kFinR; ++q) sum += v[q];
    unsigned long long tot, ptot;
    const unsigned long long ex0 = carry + block_excl_scan<kVsTPB>(sum, tot, s_sc);
    uint32_t np = 0;
    unsigned long long e = ex0;
#pragma unroll
    for (int q = 0; q < kFinR; ++q) {
      const uint32_t take = e >= k ? 0u : (uint32_t)min((unsigned long long)v[q], k - e);
      if (e < k && e + v[q] >= k) s_reach = c0 + threadIdx.x * kFinR + q;   // exactly one tile
      np += (take + kVaPass - 1) / kVaPass;
      e += v[q];
    }
    uint32_t q0 = (uint32_t)(pcarry + block_excl_scan<kVsTPB>(np, ptot, s_sc));
    e = ex0;
#pragma unroll
    for (int q = 0; q < kFinR; ++q) {
      const uint32_t take = e >= k ? 0u : (uint32_t)min((unsigned long long)v[q], k - e);
      const uint32_t t = c0 + threadIdx.x * kFinR + q;
      for (uint32_t off = 0; off < take; off += kVaPass)
        T.vpass[q0++] = make_ulonglong2((unsigned long long)(e + off) | ((unsigned long long)t << 32),
                                        (unsigned long long)off | ((unsigned long long)min((uint32_t)kVaPass, take - off) << 32));
      e += v[q];
      s_fc[threadIdx.x * kFinR + q] = (uint32_t)min(e, (unsigned long long)k);   // inclusive, clamped
    }
    __syncthreads();
#pragma unroll
    for (int q = 0; q < kFinR; ++q) {
      const uint32_t i = q * kVsTPB + threadIdx.x;
      if (i < ce && s_fc[i] < k) {   // before the reach tile
        const unsigned long long* rec = reinterpret_cast<const unsigned long long*>(tc + (size_t)(c0 + i) * 8 + 2);
        kd = min(kd, __ldcg(rec));
        ku = min(ku, __ldcg(rec + 1));
      }
    }
    carry += tot;
    pcarry += ptot;
    __syncthreads();   // s_fc is restaged by the next chunk
  }
  if (kd != ~0ull) atomicMin(&s_kd, kd);
  if (ku != ~0ull) atomicMin(&s_ku, ku);
  const uint32_t found = (uint32_t)min((unsigned long long)k, carry);
  const uint32_t npass = (uint32_t)pcarry;
  __syncthreads();
#ifdef UM_VS_TRACE
  if (threadIdx.x == 0) VS_TR(8007, vs_now());
#endif
  const uint32_t reach = s_reach;
  if (threadIdx.x == 0) {
    unsigned long long kd = s_kd, ku = s_ku;   // positions in the concatenated index space
    if (reach != ~0u) {
      const unsigned long long bound = (unsigned long long)reach * kVsTile;
      if (bound < s_ld) {
        kd = min(kd, bound);
        ku = min(ku, s_ld);   // USED not reached: its head stays
      } else {
        ku = min(ku, bound);
      }
    }
    c->disc_head = kd != ~0ull ? s_dh + kd : c->disc_tail;
    c->used_head = ku != ~0ull ? s_uh + (ku - s_ld) : c->used_tail;
    c->n_vict = found;
    c->vt_reach = npass;
    stat_add(T, S_EVICT, found);
    const int f0 = (int)s_f0;
    c->f0 = (uint32_t)f0;
    if (evict_mode) {
      c->free_top = f0 + (int)found;
    } else {
      c->free_top = f0 - (int)min((uint32_t)f0, s_nn);
      c->used_tail += c->n_rekey;
    }
    c->scan_done = 0;
    c->vs_combo = 0;
    c->vs_fin = 0;
    c->first_skip = ~0u;
#ifdef UM_VS_TRACE
    VS_TR(8001, vs_now());
    VS_TR(8002, E);
    VS_TR(8003, k);
#endif
  }
  __threadfence();
}

// 512-thread CTAs, 2 per SM (62 registers): the same resident warps as 4 x 256 in one
// wave, and a quarter of the CTAs to dispatch when there is nothing to do (k = 0)
__global__ void __launch_bounds__(kVaTPB, 2) k_victims_apply(Tables T, int evict_mode, uint32_t seq) {
  pdl_enter();
  constexpr int TPB = kVaTPB, AIPT = 4, CH = 32 * AIPT;
  __shared__ uint32_t s_cnt[8];
  Ctl* c = T.ctl;
  const uint32_t found = c->n_vict;
  if (found == 0) {            // uniform: no victims, no counters
    if (blockIdx.x == 0 && threadIdx.x == 0 && c->k0_pend) {   // bookkeeping of the k = 0 scan
      c->free_top -= (int)c->k0_take;
      c->used_tail += c->n_rekey;
      c->k0_pend = 0;
    }
    return;
  }
  const int f0 = (int)c->f0;   // free_top when the victims were chosen (set by the scan)
  const uint32_t npass = c->vt_reach;
  const int lane = threadIdx.x & 31;
  const unsigned lt = lanemask_lt();
  uint32_t nG = 0, nAv = 0, nGL = 0;
  // One warp per pass of the scan's work table: pass q of tile t reclaims the tile's
  // victims prefix + q * CH + [0, CH), out of its first take = min(count, found -
  // prefix) candidates.  Item (i, lane) = victim base + 32 i + lane (coalesced); each
  // load phase keeps AIPT loads of a lane in flight; one host-frame pop (and D2H-list
  // append) per pass.
  static_assert(CH == kVaPass, "pass size");
#ifdef UM_VS_TRACE
  if (threadIdx.x == 0 && blockIdx.x < 1000) VS_TR(6000 + 2 * blockIdx.x, vs_now());
#endif
  const uint32_t nwarps = gridDim.x * (TPB / 32);
  for (uint32_t p = blockIdx.x * (TPB / 32) + (threadIdx.x >> 5); p < npass; p += nwarps) {
    // entry {victim index of the pass's first victim | tile << 32, offset in the tile's
    // candidates | victims in the pass << 32}
    const ulonglong2 ent = T.vpass[p];
    const uint32_t j0 = (uint32_t)ent.x, tile = (uint32_t)(ent.x >> 32);
    const uint32_t pn = (uint32_t)(ent.y >> 32);
    const uint32_t* scr = T.vscratch + (size_t)tile * kVsTile + (uint32_t)ent.y;
    {
      uint32_t v[AIPT], fr[AIPT], hf[AIPT];
      uint8_t ss[AIPT], nk[AIPT];
#pragma unroll
      for (int q = 0; q < AIPT; ++q) {
        const uint32_t i = q * 32 + lane;
        v[q] = i < pn ? scr[i] : UM_NONE;
        nk[q] = (i < pn && !evict_mode) ? T.needk[(uint32_t)f0 + j0 + i] : (uint8_t)0xff;
      }
#pragma unroll
      for (int q = 0; q < AIPT; ++q) {
        ss[q] = v[q] != UM_NONE ? ld_st(T, v[q]) : (uint8_t)0xff;
        fr[q] = v[q] != UM_NONE ? T.frame_of[v[q]] : UM_NONE;
      }
#pragma unroll
      for (int q = 0; q < AIPT; ++q) {
        // a write-back victim's bytes land in the host frame of the block migrating into
        // its frame (fused swap, R5) when there is one
        hf[q] = (ss[q] == ST_G && nk[q] == ST_H) ? T.needhf[(uint32_t)f0 + j0 + q * 32 + lane] : UM_NONE;
      }
      unsigned bA[AIPT], bD[AIPT];
      uint32_t tA = 0, tD = 0;
#pragma unroll
      for (int q = 0; q < AIPT; ++q) {
        const bool isG = ss[q] == ST_G;
        bA[q] = __ballot_sync(FULL, isG && hf[q] == UM_NONE);
        bD[q] = __ballot_sync(FULL, evict_mode && isG);
        tA += __popc(bA[q]);
        tD += __popc(bD[q]);
      }
      int hb = 0;
      uint32_t hav = 0, db = 0;
      if (lane == 0) {
        if (tA) {
          const int old = atomicSub(&c->hfree_top, (int)tA);
          const int avail = old < 0 ? 0 : (old < (int)tA ? old : (int)tA);
          if (avail < (int)tA) {
            atomicAdd(&c->hfree_top, (int)tA - avail);
            atomicExch(&c->err, 2u);   // host-frame pool exhausted -> UM_ENOMEM
          }
          hb = old;
          hav = (uint32_t)avail;
        }
        if (tD) db = atomicAdd(&c->n_d2h, tD);
      }
      hb = __shfl_sync(FULL, hb, 0);
      hav = __shfl_sync(FULL, hav, 0);
      db = __shfl_sync(FULL, db, 0);
      uint32_t rA = 0, rD = 0;   // ranks: earlier passes q, then lanes below
#pragma unroll
      for (int q = 0; q < AIPT; ++q) {
        if ((bA[q] >> lane) & 1u) {
          const uint32_t r = rA + __popc(bA[q] & lt);
          hf[q] = r < hav ? T.hfree_stack[hb - 1 - (int)r] : UM_NONE;
        }
        rA += __popc(bA[q]);
      }
#pragma unroll
      for (int q = 0; q < AIPT; ++q) {
        const uint32_t j = j0 + q * 32 + lane;
        if (v[q] != UM_NONE) {
          const bool isG = ss[q] == ST_G;
          T.victim[j] = v[q];
          T.vframe[j] = fr[q];
          T.vkind[j] = ss[q];
          T.vhf[j] = hf[q];
          T.sk[v[q]] = mk_sk(isG ? ST_H : ST_HD, 0);
          if (T.phz) T.phz[v[q]] = 0u;
          T.map[v[q]] = UM_NONE;
          T.frame_of[v[q]] = UM_NONE;
          T.hframe[v[q]] = hf[q];
          nG += isG;
          nAv += !isG;
          nGL += ss[q] == ST_GL;
          if (evict_mode) {
            T.free_stack[f0 + j] = fr[q];
            if (isG) {
              const uint32_t d = db + rD + __popc(bD[q] & lt);
              T.d2h_frame[d] = fr[q];
              T.d2h_hf[d] = hf[q];
              d2h_listed(T, seq, v[q], d, ss[q]);
            }
          }
        }
        rD += __popc(bD[q]);
      }
    }
  }
  uint32_t cnt3[3] = {nG, nAv, nGL};
  const int slots[3] = {S_D2H, S_D2H_AV, S_UNMAPS};
  const long long mul[3] = {(long long)T.B, (long long)T.B, 1};
  block_counts_to<3>(T, cnt3, s_cnt, slots, mul);
#ifdef UM_VS_TRACE
  if (threadIdx.x == 0 && blockIdx.x < 1000) VS_TR(6001 + 2 * blockIdx.x, vs_now());
#endif
}

// ------------------------------------------------------------------------------------
// K4/K5/K6: the transfer engine.  One elected thread per CTA drives a kXferStages-deep
// ring of TMA bulk copies (cp.async.bulk, mbarrier complete_tx) through shared memory.
// Work unit = one kXferChunk slice of one frame.  Fused swap per unit: the victim's
// bytes (HBM) and the new owner's bytes (mapped pinned host memory) are loaded into
// smem together; only after both loads land are the stores issued (victim -> host,
// new -> HBM), so the write-after-read hazard on the frame is resolved inside the
// unit and both PCIe directions stay busy.  Blocks needing zeros get a bulk store of a
// zeroed smem tile instead (zero-fill, PAPER L200 / Fig. 2 (7)).  Metadata of a newly
// resident block is committed by the CTA that handles its first chunk.
// ------------------------------------------------------------------------------------
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
      " @!p bra WAIT_%=;\n}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* sdst, const void* gsrc, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_u32(sdst)),
               "l"(gsrc), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void bulk_s2g(void* gdst, const void* ssrc, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(gdst), "r"(smem_u32(ssrc)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read1() { asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// The plan of need item i of the current sub-op (K6 decides it from K3's output):
// destination frame (free stack first, then victim frames in victim order), the
// victim's write-back destination, the newcomer's source host frame, zero-fill, and
// whether the newcomer's host frame was handed to the victim (fused swap, R5).
__device__ __forceinline__ XItem item_plan(const Tables& T, uint32_t i, uint32_t f0, uint32_t nfu) {
  XItem x;
  const uint8_t kd = T.needk[i];
  const uint32_t hf = T.needhf[i];
  x.flags = 0;
  x.dst_hf = UM_NONE;
  if (i < nfu) {
    x.fr = T.free_stack[f0 - 1 - i];
  } else {
    const uint32_t j = i - f0;
    x.fr = T.vframe[j];
    if (T.vkind[j] == ST_G && T.vhf[j] != UM_NONE) {
      x.dst_hf = T.vhf[j];
      x.flags |= XI_D2H;
      if (x.dst_hf == hf) x.flags |= XI_SWAP;
    }
  }
  if (kd == ST_H) {
    x.src_hf = hf != UM_NONE ? hf : T.zero_hf;
    x.flags |= XI_H2D;
  } else {
    x.src_hf = UM_NONE;
    x.flags |= XI_ZF;
  }
  return x;
}

// K6 commit of need item i: the block becomes G in its frame; a host frame it leaves
// is recycled unless it was handed to the victim.
__device__ __forceinline__ void item_commit(const Tables& T, uint32_t i, const XItem& x, uint32_t seq) {
  const uint32_t bb = T.need[i];
  T.sk[bb] = mk_sk(ST_G, seq);
  T.frame_of[bb] = x.fr;
  T.map[bb] = x.fr;
  const uint32_t hf = T.needhf[i];
  if (T.needk[i] == ST_H && hf != UM_NONE) {
    T.hframe[bb] = UM_NONE;
    if (!(x.flags & XI_SWAP)) {
      int idx = atomicAdd(&T.ctl->hfree_top, 1);
      T.hfree_stack[idx] = hf;
    }
  }
}

// Page masks of need item i (two-level, NEXT-1; all zero at single level): the
// newcomer's dead pages (zero-filled instead of migrated) and zero-content
// pages (migrated from the zero page) when it comes from the host, and the dead pages of
// the victim whose frame it takes (not written back, L196-198).
struct ItemPages { uint32_t ndead, nhz, vdead; };
__device__ __forceinline__ ItemPages item_pages(const Tables& T, uint32_t i, const XItem& x, uint32_t f0) {
  ItemPages m{0u, 0u, 0u};
  if (!T.pdead) return m;
  if (x.flags & XI_H2D) {
    const uint32_t b = T.need[i];
    m.ndead = T.pdead[b];
    m.nhz = T.phz[b];
  }
  if (x.flags & XI_D2H) m.vdead = T.pdead[T.victim[i - f0]];
  return m;
}

// Transfer-log records of need item i (one per page at two levels): the newcomer's
// migration or zero-fill and, when its frame comes from a valid victim, the victim's
// write-back of its live pages.
__device__ __forceinline__ void item_log(const Tables& T, uint32_t i, const XItem& x, uint32_t seq, uint32_t f0,
                                         const ItemPages& m) {
  if (!T.xlog) return;
  const uint32_t b = T.need[i], k = T.needk[i];
  for (uint32_t p = 0; p < T.ppc; ++p)
    xlog_put(T, seq, b * T.ppc + p, ((x.flags & XI_H2D) && !((m.ndead >> p) & 1u)) ? XL_H2D : XL_ZF, k);
  if (x.flags & XI_D2H) {
    const uint32_t v = T.victim[i - f0];
    for (uint32_t p = 0; p < T.ppc; ++p)
      if (!((m.vdead >> p) & 1u)) xlog_put(T, seq, v * T.ppc + p, XL_D2H, T.vkind[i - f0]);
  }
}

// Two-level byte counters: the planning kernels count whole chunks; dead pages of a
// migrating newcomer are zero-filled instead (h2d -> zf + h2d_avoided) and dead pages
// of a written-back victim are not moved (d2h -> d2h_avoided).
__device__ __forceinline__ void item_page_stats(const Tables& T, const ItemPages& m) {
  const long long P = T.P;
  if (m.ndead) {
    const long long d = (long long)__popc(m.ndead) * P;
    stat_add(T, S_H2D, -d);
    stat_add(T, S_ZF, d);
    stat_add(T, S_H2D_AV, d);
  }
  if (m.vdead) {
    const long long d = (long long)__popc(m.vdead) * P;
    stat_add(T, S_D2H, -d);
    stat_add(T, S_D2H_AV, d);
  }
}

struct Unit {
  char* frame;        // frame chunk (HBM)
  char* d2h_dst;      // host chunk receiving the old content, or null
  const char* h2d_src;// host chunk with the new content, or null
  bool zf;            // zero-fill the frame chunk
  __device__ bool pure_zf() const { return zf && !d2h_dst; }
};

// One item's plan as the transfer loop needs it (block-base pointers and page masks).
struct SPlan {
  char* frame;          // the item's destination frame (HBM)
  char* d2h;            // host frame receiving the victim's (or D2H-only block's) bytes, or null
  const char* h2d;      // host frame holding the newcomer's bytes, or null (zero-fill)
  uint32_t dmask;       // pages not written back (dead in the victim / D2H-only block)
  uint32_t zmask;       // pages zero-filled instead of migrated (dead in the newcomer)
  uint32_t hzmask;      // pages migrated from the zero page (zero content on the host)
};

// K4.  Each CTA takes a contiguous range of CH-byte units.  Warp 0 moves data: it runs
// the units that need a load (write-back, migration, or both: the fused swap) through an
// S-stage load -> store ring driven by lane 0 (cp.async.bulk + mbarrier).  Warps 1-3
// zero-fill: each takes a third of the range and bulk-stores a zeroed smem tile into its
// pure zero-fill units, and commits (state, mapping, host-frame release, counters, log)
// the items whose first unit lies in its third.  Zero-fill (HBM) and transfers (PCIe)
// thus overlap inside every CTA.  Plans are computed 32 items at a time, one per lane
// (independent loads), into the warp's shared-memory slots; a commit changes nothing a
// plan reads.  D2H-only lists (prefetch HOST, evict) use warp 0 alone.
constexpr int kSvcWarps = 4;

__global__ void __launch_bounds__(32 * kSvcWarps, 1) k_service(Tables T, int mode, uint32_t seq) {
  pdl_enter();
  // The frames were last written through the generic proxy (application kernel, an
  // earlier sub-op's zero-fill commit path): order those writes before this kernel's
  // bulk copies (async proxy).  The wait of programmatic dependent launch makes the
  // predecessors' writes visible, but not to the async proxy.
  asm volatile("fence.proxy.async.global;" ::: "memory");
  extern __shared__ __align__(128) char smem[];
  __shared__ __align__(8) uint64_t bar[kXferStages];
  __shared__ SPlan s_plw[kSvcWarps][32];
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  SPlan* s_pl = s_plw[warp];
  const uint32_t CH = T.B < kXferChunk ? T.B : kXferChunk;
  const uint32_t cpb = T.B / CH;
  const uint32_t upp = T.P / CH;   // units per page (single level: the whole block)
  char* zero = smem;
  char* stA = smem + CH;                      // S stages of CH (victim/old bytes)
  char* stB = smem + CH + kXferStages * CH;   // S stages of CH (new bytes)
  for (uint32_t i = threadIdx.x * 16; i < CH; i += 32 * kSvcWarps * 16)
    *reinterpret_cast<uint4*>(zero + i) = make_uint4(0, 0, 0, 0);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  Ctl* c = T.ctl;
  const uint32_t n_items = mode == SVC_SUBOP ? c->n_need : c->n_d2h;
  const uint32_t f0 = c->f0;
  const uint32_t nfu = min(f0, n_items);
  const unsigned long long units = (unsigned long long)n_items * cpb;
  const unsigned long long ubeg = units * blockIdx.x / gridDim.x;
  const unsigned long long uend = units * (blockIdx.x + 1) / gridDim.x;
  if (threadIdx.x == 0) {
    for (int s = 0; s < kXferStages; ++s) mbar_init(&bar[s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();   // zero tile and barriers visible to every warp
  const uint32_t lcpb = 31 - __clz(cpb), lupp = 31 - __clz(upp);
  // plans of items [b0, b0 + 32) (warp-collective); commit items whose first unit is in
  // [cb, ce) (a zero-fill warp's third of the range)
  uint32_t batch = UM_NONE;
  auto plan_batch = [&](uint32_t b0, bool commit, unsigned long long cb, unsigned long long ce) {
    __syncwarp();                       // every lane is done with the previous batch
    const uint32_t i = b0 + lane;
    if (i < n_items) {
      SPlan q;
      if (mode == SVC_SUBOP) {
        const XItem x = item_plan(T, i, f0, nfu);
        const ItemPages pg = item_pages(T, i, x, f0);
        q.frame = T.frames + (size_t)x.fr * T.B;
        q.d2h = (x.flags & XI_D2H) ? hptr(T, x.dst_hf) : nullptr;
        q.h2d = (x.flags & XI_H2D) ? hptr(T, x.src_hf) : nullptr;
        q.dmask = pg.vdead;
        q.zmask = (x.flags & XI_H2D) ? pg.ndead : 0xffffffffu;
        q.hzmask = pg.nhz;
        const unsigned long long u0 = (unsigned long long)i << lcpb;
        if (commit && u0 >= cb && u0 < ce) {
          item_log(T, i, x, seq, f0, pg);
          item_page_stats(T, pg);
          item_commit(T, i, x, seq);
        }
      } else {
        const uint32_t hf = T.d2h_hf[i];
        q.frame = T.frames + (size_t)T.d2h_frame[i] * T.B;
        q.d2h = hf != UM_NONE ? hptr(T, hf) : nullptr;
        q.h2d = nullptr;
        q.dmask = T.pdead ? T.d2h_dmask[i] : 0u;
        q.zmask = 0u;
        q.hzmask = 0u;
      }
      s_pl[lane] = q;
    }
    batch = b0;
    __syncwarp();
  };
  auto plan_of = [&](uint32_t i, bool commit, unsigned long long cb, unsigned long long ce) -> const SPlan& {
    if (batch == UM_NONE || i - batch >= 32u) plan_batch(i, commit, cb, ce);
    return s_pl[i - batch];
  };
  // pages of an item whose units only need the zero tile (nothing to load or write back)
  auto pure_pages = [&](const SPlan& q) -> uint32_t {
    const uint32_t zf = q.h2d ? q.zmask : 0xffffffffu;
    const uint32_t wb = q.d2h ? ~q.dmask : 0u;
    return mode == SVC_SUBOP ? (zf & ~wb) : 0u;
  };
  if (warp != 0) {
    // zero-fill warps: units [zb, ze) (a third of the CTA's range), walked as (item,
    // chunk) pairs with shifts; lane 0 issues
    if (mode != SVC_SUBOP) return;
    const unsigned long long span = uend - ubeg;
    const unsigned long long zb = ubeg + span * (warp - 1) / (kSvcWarps - 1);
    const unsigned long long ze = ubeg + span * warp / (kSvcWarps - 1);
    if (zb >= ze) return;
    const uint32_t i_lo = (uint32_t)(zb >> lcpb), i_end = (uint32_t)((ze + cpb - 1) >> lcpb);
    const uint32_t ch_lo = (uint32_t)(zb & (cpb - 1)), ch_end_last = (uint32_t)(((ze - 1) & (cpb - 1)) + 1);
    uint32_t issued = 0;
    for (uint32_t i = i_lo; i < i_end; ++i) {
      const SPlan& q = plan_of(i, true, zb, ze);
      const uint32_t pm = pure_pages(q);
      if (!pm || lane != 0) continue;
      const uint32_t cb = i == i_lo ? ch_lo : 0u, ce = i + 1 == i_end ? ch_end_last : cpb;
      for (uint32_t ch = cb; ch < ce; ++ch) {
        if (!((pm >> (ch >> lupp)) & 1u)) continue;
        bulk_s2g(q.frame + (size_t)ch * CH, zero, CH);
        if ((++issued & 31) == 0) bulk_commit();
      }
    }
    if (lane == 0) {
      bulk_commit();
      bulk_wait_all();
      asm volatile("fence.proxy.async.global;" ::: "memory");   // bulk writes before generic readers
    }
    return;
  }
  // warp 0: the units with a load, through the S-stage TMA ring (cursor: item ci, chunk cch).
  // A CTA with an empty range still reaches the D2H-only completion count below.
  const uint32_t i_lo = (uint32_t)(ubeg >> lcpb), i_end = (uint32_t)((uend + cpb - 1) >> lcpb);
  const uint32_t ch_end_last = (uint32_t)(((uend - 1) & (cpb - 1)) + 1);
  uint32_t ci = i_lo, cch = (uint32_t)(ubeg & (cpb - 1));
  auto unit_of = [&](const SPlan& q, uint32_t ch) -> Unit {
    const size_t coff = (size_t)ch * CH;
    const uint32_t pg = ch >> lupp;
    Unit x;
    x.frame = q.frame + coff;
    x.d2h_dst = (q.d2h && !((q.dmask >> pg) & 1u)) ? q.d2h + coff : nullptr;
    const bool mig = q.h2d && !((q.zmask >> pg) & 1u);
    x.h2d_src = mig ? (((q.hzmask >> pg) & 1u) ? hptr(T, T.zero_hf) : q.h2d) + coff : nullptr;
    x.zf = mode == SVC_SUBOP && !mig;
    return x;
  };
  auto next_xfer = [&](Unit& x) -> bool {
    while (ubeg < uend && ci < i_end) {
      const SPlan& q = plan_of(ci, false, 0, 0);
      const uint32_t ce = ci + 1 == i_end ? ch_end_last : cpb;
      // pages with a load: not pure zero-fill (sub-op), live pages to write back (D2H-only)
      const uint32_t keep = mode == SVC_SUBOP ? ~pure_pages(q) : (q.d2h ? ~q.dmask : 0u);
      while (cch < ce && !((keep >> (cch >> lupp)) & 1u)) ++cch;
      if (cch < ce) {
        x = unit_of(q, cch++);
        return true;
      }
      ++ci;
      cch = 0;
    }
    return false;
  };
  Unit U[kXferStages];
  auto issue_loads = [&](int s, const Unit& x) {
    if (lane != 0) return;
    const uint32_t bytes = (x.d2h_dst ? CH : 0u) + (x.h2d_src ? CH : 0u);
    mbar_expect_tx(&bar[s], bytes);
    if (x.d2h_dst) bulk_g2s(stA + s * CH, x.frame, CH, &bar[s]);
    if (x.h2d_src) bulk_g2s(stB + s * CH, x.h2d_src, CH, &bar[s]);
  };
  unsigned long long loaded = 0;
  for (int s = 0; s < kXferStages; ++s) {
    if (!next_xfer(U[s])) break;
    issue_loads(s, U[s]);
    ++loaded;
  }
  for (unsigned long long k = 0; k < loaded; ++k) {
    const int s = (int)(k % kXferStages);
    if (lane == 0) {
      mbar_wait(&bar[s], (uint32_t)((k / kXferStages) & 1));
      const Unit& x = U[s];
      if (x.d2h_dst) bulk_s2g(x.d2h_dst, stA + s * CH, CH);
      if (x.h2d_src) bulk_s2g(x.frame, stB + s * CH, CH);
      else if (x.zf) bulk_s2g(x.frame, zero, CH);
      bulk_commit();
    }
    if (k >= 1 && loaded == k - 1 + kXferStages) {
      const int sp = (int)((k - 1) % kXferStages);
      Unit y;
      if (next_xfer(y)) {
        if (lane == 0) bulk_wait_read1();
        U[sp] = y;
        issue_loads(sp, U[sp]);
        ++loaded;
      }
    }
  }
  if (lane == 0) {
    bulk_wait_all();
    asm volatile("fence.proxy.async.global;" ::: "memory");   // bulk writes before generic readers
    if (mode == SVC_D2H_ONLY) {
      __threadfence();
      unsigned int d = atomicAdd(&c->app_units, 1u);
      if (d == gridDim.x - 1) {
        c->n_d2h = 0;
        c->app_units = 0;
      }
    }
  }
}

// ------------------------------------------------------------------------------------
// K4-CE support: K6 plans + commits every need item on the device and exports the plan
// (XItem records) for the host to turn into copy-engine batches; zero-fill of the
// items that need it runs as a kernel on the copy streams.
// ------------------------------------------------------------------------------------
__global__ void k_plan_commit(Tables T, uint32_t seq) {
  pdl_enter();
  const uint32_t n = T.ctl->n_need, f0 = T.ctl->f0, nfu = min(f0, n);
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    XItem x = item_plan(T, i, f0, nfu);
    T.xitems[i] = x;
    T.hx[i] = x;            // pinned host mirror (mapped)
    item_log(T, i, x, seq, f0, ItemPages{0u, 0u, 0u});   // single level only
    item_commit(T, i, x, seq);
  }
  // every thread's plan writes are performed system-wide before its CTA takes a ticket;
  // the CTA with the last ticket publishes {n, seq} for the host's spin
  __threadfence_system();
  __syncthreads();
  if (threadIdx.x == 0 && atomicAdd(&T.ctl->pc_done, 1u) == gridDim.x - 1) {
    T.ctl->pc_done = 0;
    __threadfence_system();
    volatile unsigned int* f = T.hflag;
    f[1] = n;
    __threadfence_system();
    f[0] = seq;
  }
}

// HBM fills are done in segments of kFillSeg bytes: the segment's metadata is looked up
// once (thread 0 -> smem) and 256 threads then stream 16-byte stores, 8 per thread in
// flight, so the per-segment lookup latency is amortised over 256 KiB of writes.
constexpr uint32_t kFillSeg = 256u << 10;

template <int TPB = 256>
__device__ __forceinline__ void fill_segment(uint4* dst, uint32_t n16, uint4 v) {
  uint32_t t = threadIdx.x;
  for (; t + 7 * TPB < n16; t += 8 * TPB) {
#pragma unroll
    for (int k = 0; k < 8; ++k) dst[t + k * TPB] = v;
  }
  for (; t < n16; t += TPB) dst[t] = v;
}

__global__ void __launch_bounds__(256) k_zero_items(Tables T, uint32_t i0, uint32_t i1) {
  __shared__ char* s_dst;
  const uint32_t SEG = T.B < kFillSeg ? T.B : kFillSeg;
  const uint32_t spb = T.B / SEG;
  const unsigned long long units = (unsigned long long)(i1 - i0) * spb;
  for (unsigned long long u = blockIdx.x; u < units; u += gridDim.x) {
    if (threadIdx.x == 0) {
      const XItem x = T.xitems[i0 + (uint32_t)(u / spb)];
      s_dst = (x.flags & XI_ZF) ? T.frames + (size_t)x.fr * T.B + (size_t)(u % spb) * SEG : nullptr;
    }
    __syncthreads();
    char* d = s_dst;
    __syncthreads();
    if (d) fill_segment(reinterpret_cast<uint4*>(d), SEG / 16, make_uint4(0, 0, 0, 0));
  }
}

// ------------------------------------------------------------------------------------
// Harness "application kernel": after a touch sub-op is serviced, every block with a
// UM_ACC_WRITE access receives the content stamp s = (seq << 32) | block as the
// 16-byte pattern {s, ~s}, written through its frame (G or GL blocks are mapped).
// ------------------------------------------------------------------------------------
// TPB = 256 on the paging stream; TPB = 128 at one CTA per SM when it overlaps paging
// work (UM_F_OVERLAP): its grid-stride CTAs live for the whole kernel, and a small
// footprint leaves room on every SM for the 1024-thread planning CTAs.
template <int TPB>
__global__ void __launch_bounds__(TPB) k_app_stamp(Tables T, const __grid_constant__ OpIv iv, uint32_t g0, uint32_t n, uint32_t seq) {
  pdl_enter();
  __shared__ char* s_dst;
  __shared__ uint32_t s_q;
  // segments never straddle a page (P = B at single level), so a segment has one stamp
  const uint32_t SEG = T.P < kFillSeg ? T.P : kFillSeg;
  const uint32_t spb = T.B / SEG, spp = T.P / SEG;
  const unsigned long long units = (unsigned long long)n * spb;
  for (unsigned long long u = blockIdx.x; u < units; u += gridDim.x) {
    if (threadIdx.x == 0) {
      uint32_t g = g0 + (uint32_t)(u / spb);
      const uint32_t sg = (uint32_t)(u % spb), pg = sg / spp;
      char* d = nullptr;
      uint32_t bb, wr;
      if (iv.blist) {
        const uint32_t e = iv.blist[g];
        bb = e & 0x7fffffffu;
        wr = iv.pw ? (iv.pw[g] >> pg) & 1u : e >> 31;   // two-level: the pages it writes
      } else {
        const uint32_t j = iv_find(iv, g);
        bb = iv_lo(iv, j) + (g - iv_pre(iv, j));
        wr = iv_w(iv, j);
      }
      if (wr) {
        uint32_t fr = T.frame_of[bb];
        if (fr != UM_NONE) d = T.frames + (size_t)fr * T.B + (size_t)sg * SEG;
      }
      s_dst = d;
      s_q = bb * T.ppc + pg;   // content stamps are per page (= per block at single level)
    }
    __syncthreads();
    char* d = s_dst;
    const unsigned long long sv = ((unsigned long long)seq << 32) | s_q;
    __syncthreads();
    if (d) fill_segment<TPB>(reinterpret_cast<uint4*>(d), SEG / 16,
                             make_uint4((uint32_t)sv, (uint32_t)(sv >> 32), ~(uint32_t)sv, ~(uint32_t)(sv >> 32)));
  }
}

// ------------------------------------------------------------------------------------
// Two-level page masks (oracle/chunks.py).  Chunks stay the
// residency / eviction unit; pages discarded while their chunk is not are tracked in
// pdead (plazy: the lazily discarded subset) and skipped by the transfer engine.
// ------------------------------------------------------------------------------------
// After a GPU sub-op: a touch revives the eagerly discarded pages it covers ("skip the
// memory transfers ... until it gets accessed again", L196); a lazily discarded page
// needs the prefetch (L186-190, A8).  After a whole prefetch: it revives every page it
// covers (A17).
__global__ void __launch_bounds__(256) k_page_revive(Tables T, const __grid_constant__ OpIv iv, uint32_t g0, uint32_t n,
                                                     int touch) {
  pdl_enter();
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const uint32_t g = g0 + i, c = iv.blist[g] & 0x7fffffffu, cm = iv.pcov[g];
    const uint32_t d = T.pdead[c];
    if (!(d & cm)) continue;
    if (touch) {
      T.pdead[c] = d & ~(cm & ~T.plazy[c]);
    } else {
      T.pdead[c] = d & ~cm;
      T.plazy[c] &= ~cm;
      // a chunk an earlier sub-op of this prefetch brought in and a later one evicted is
      // on the host without its dead pages: revived, they read as zero
      if (ld_st(T, c) == ST_H) T.phz[c] |= d & cm;
    }
  }
}

// After a prefetch(HOST) of chunks [lo, lo + n) covering global pages [p0, p1): every
// chunk is now H; the pages covered are revalidated (A17), and a revalidated dead page
// holds no data on the host (it was never written back, or its host copy was released:
// R1), so it reads as zero and migrates from the zero page.
__global__ void __launch_bounds__(256) k_page_host_revive(Tables T, uint32_t lo, uint32_t n, unsigned long long p0,
                                                          unsigned long long p1) {
  pdl_enter();
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const uint32_t c = lo + i;
    const unsigned long long c0 = (unsigned long long)c * T.ppc;
    const uint32_t a = p0 > c0 ? (uint32_t)(p0 - c0) : 0u;
    const uint32_t e = p1 < c0 + T.ppc ? (uint32_t)(p1 - c0) : T.ppc;
    const uint32_t cm = (e >= 32 ? 0xffffffffu : ((1u << e) - 1u)) & ~((1u << a) - 1u);
    const uint32_t d = T.pdead[c];
    if (!(d & cm)) continue;
    T.pdead[c] = d & ~cm;
    T.plazy[c] &= ~cm;
    T.phz[c] |= d & cm;
  }
}

// A discard covering only pages m of chunk c (its edge chunks; whole chunks are
// handled at chunk level by k_directive): G or H chunks mark the pages dead without
// unmapping or re-queueing ("avoid splitting 2MB GPU mappings", §5.4).
__global__ void k_page_discard(Tables T, uint32_t c0, uint32_t m0, uint32_t c1, uint32_t m1, int lazy) {
  pdl_enter();
  const uint32_t c = threadIdx.x == 0 ? c0 : c1, m = threadIdx.x == 0 ? m0 : m1;
  if (threadIdx.x > 1 || c == UM_NONE || !m) return;
  const uint8_t ss = ld_st(T, c);
  if (ss != ST_G && ss != ST_H) return;
  const uint32_t d = T.pdead[c];
  if (lazy) T.plazy[c] |= m & ~d;
  else T.plazy[c] &= ~m;
  T.pdead[c] = d | m;
}

// ------------------------------------------------------------------------------------
// K8: directives over a contiguous block range (discard: fully covered blocks only,
// PAPER L211; prefetch HOST: every overlapping block).
//   discard      G -> GE (unmap, DISC append), GL -> GE, H -> HD
//   discard_lazy G -> GL (DISC append, mapping kept), H -> HD
//   prefetch HOST G -> H (D2H), GE/GL -> H (no transfer), HD/U -> H
// Streaming: block lo + idx owns DISC slot disc_tail + idx (entry (seq, b)); the slot
// is live only if the block turns GE/GL with dkey = seq here, so the ring stays sorted
// by (dkey, block) without ranking.  Frame / host-frame stack traffic and the D2H list
// take one atomic per CTA (their order is not observable).  The last CTA publishes
// disc_tail and the counters.
// ------------------------------------------------------------------------------------
template <int IPT>
__device__ __forceinline__ void directive_body(const Tables& T, int kind, uint32_t lo, uint32_t n, uint32_t seq,
                                               int discard_off, unsigned long long tail0) {
  constexpr int TPB = kStTPB, TILE = TPB * IPT;
  __shared__ unsigned long long s_sc[TPB / 32];
  __shared__ int s_hb, s_fb;
  __shared__ uint32_t s_db, s_hav;
  __shared__ uint32_t s_cnt[8];
  Ctl* c = T.ctl;
  const bool disc = kind == DIR_DISCARD || kind == DIR_DISCARD_LAZY;
  const bool active = !discard_off || kind == DIR_PREFETCH_HOST;
  const unsigned long long kseq = (unsigned long long)seq << 32;
  uint32_t nUnmap = 0, nD2H = 0, nAv = 0;
  // persistent grid (resident CTAs) striding over tiles of TILE blocks
  const uint32_t ntiles = (n + TILE - 1) / TILE;
  for (uint32_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
  const uint32_t tbase = tile * TILE;
  uint8_t s[IPT];
  uint32_t hasf = 0;   // bit k: item k is an H block holding a host frame (discard)
  // per-thread counts of stack / list traffic: A = host frames (released by a discard
  // of an H block holding one, taken by a prefetch HOST of G), F = GPU frames freed
  // (prefetch HOST)
  uint32_t nA = 0, nF = 0;
  // all state loads first (one basic block: IPT gathers in flight), then the
  // dependent host-frame loads of H blocks (predicated, again all in flight)
#pragma unroll
  for (int k = 0; k < IPT; ++k) {
    const uint32_t idx = tbase + k * TPB + threadIdx.x;   // coalesced
    s[k] = idx < n ? ld_st(T, lo + idx) : (uint8_t)0xff;
  }
  uint32_t hfv[IPT];
#pragma unroll
  for (int k = 0; k < IPT; ++k) hfv[k] = (disc && s[k] == ST_H) ? T.hframe[lo + tbase + k * TPB + threadIdx.x] : UM_NONE;
#pragma unroll
  for (int k = 0; k < IPT; ++k) {
    if (disc) {
      if (hfv[k] != UM_NONE) {
        hasf |= 1u << k;
        ++nA;
      }
    } else {
      nA += s[k] == ST_G;
      nF += s[k] == ST_G || s[k] == ST_GE || s[k] == ST_GL;
    }
  }
  // frame / host-frame stack traffic in this tile: ranked by a block scan, based by one
  // atomic per CTA -- skipped (one predicated barrier) when the tile has none, e.g. a
  // discard of GPU-resident data
  unsigned long long pre = 0ull;
  if (__syncthreads_or(active && (nA | nF))) {
  unsigned long long tot;
  pre = block_excl_scan<TPB>(active ? pack2(nA, nF) : 0ull, tot, s_sc);
  if (threadIdx.x == 0) {
    const uint32_t tA = unpackA(tot), tF = unpackB(tot);
    s_hb = 0; s_fb = 0; s_db = 0; s_hav = tA;
    if (disc) {
      if (tA) s_hb = atomicAdd(&c->hfree_top, (int)tA);            // release: push
    } else {
      if (tA) {                                                     // take: pop
        const int old = atomicSub(&c->hfree_top, (int)tA);
        const int avail = old < 0 ? 0 : (old < (int)tA ? old : (int)tA);
        if (avail < (int)tA) {
          atomicAdd(&c->hfree_top, (int)tA - avail);
          atomicExch(&c->err, 2u);                                  // -> UM_ENOMEM
        }
        s_hb = old;          // this CTA owns hfree_stack[old - avail, old)
        s_hav = (uint32_t)avail;
        s_db = atomicAdd(&c->n_d2h, tA);
      }
      if (tF) s_fb = atomicAdd(&c->free_top, (int)tF);
    }
  }
  __syncthreads();
  }
  uint32_t rA = unpackA(pre), rF = unpackB(pre);
  if (active) {
#pragma unroll
    for (int k = 0; k < IPT; ++k) {
      const uint32_t idx = tbase + k * TPB + threadIdx.x;
      if (idx >= n) continue;
      const uint32_t bb = lo + idx;
      const uint8_t ss = s[k];
      if (disc) {
        // only a G block enters DISC here (GL -> GE keeps its slot, A6; H -> HD has none)
        T.disc_ring[(tail0 + idx) & T.cap_mask] = ss == ST_G ? (kseq | bb) : kDeadSlot;
        if (T.pdead) T.pdead[bb] = T.plazy[bb] = T.phz[bb] = 0u;   // whole chunk: chunk level
        if (ss == ST_G) {
          T.sk[bb] = mk_sk(kind == DIR_DISCARD ? ST_GE : ST_GL, seq);
          if (kind == DIR_DISCARD) {
            T.map[bb] = UM_NONE;
            ++nUnmap;
          }
        } else if (ss == ST_GL && kind == DIR_DISCARD) {
          T.sk[bb] = (T.sk[bb] & ~7u) | ST_GE;   // keeps its dkey (A6)
          T.map[bb] = UM_NONE;
          ++nUnmap;
        } else if (ss == ST_H) {
          T.sk[bb] = mk_sk(ST_HD, 0);
          if ((hasf >> k) & 1u) {   // the host copy is released (reading R1)
            T.hfree_stack[s_hb + rA] = hfv[k];
            T.hframe[bb] = UM_NONE;
            ++rA;
          }
        }
      } else {  // prefetch to HOST
        if (ss == ST_G || ss == ST_GE || ss == ST_GL) {
          const uint32_t fr = T.frame_of[bb];
          if (ss == ST_G) {
            const uint32_t hf = rA < s_hav ? T.hfree_stack[s_hb - 1 - (int)rA] : UM_NONE;
            T.d2h_frame[s_db + rA] = fr;
            T.d2h_hf[s_db + rA] = hf;
            T.hframe[bb] = hf;
            d2h_listed(T, seq, bb, s_db + rA, ss);
            ++rA;
            ++nD2H;
          } else {
            ++nAv;
            if (ss == ST_GL) ++nUnmap;
          }
          T.free_stack[s_fb + rF] = fr;
          ++rF;
          T.frame_of[bb] = UM_NONE;
          T.map[bb] = UM_NONE;
        }
        if (ss != ST_H) {
          T.sk[bb] = mk_sk(ST_H, 0);
          if (T.phz) T.phz[bb] = 0u;   // revived pages are marked by k_page_host_revive
        }
      }
    }
  }
  __syncthreads();   // s_hb / s_fb / s_db are rewritten by the next tile
  }
  uint32_t v[3] = {nUnmap, nD2H, nAv};
  const int slots[3] = {S_UNMAPS, S_D2H, S_D2H_AV};
  const long long mul[3] = {1, (long long)T.B, (long long)T.B};
  block_counts_to<3>(T, v, s_cnt, slots, mul);
  // the host passes the exact tail; nothing in this launch reads c->disc_tail
  if (blockIdx.x == 0 && threadIdx.x == 0 && disc && active) c->disc_tail = tail0 + n;
}

// 8 blocks per thread, 6 CTAs/SM (A/B on B200: 16 per thread at 4 CTAs/SM, one round of
// 512 tiles for 2^21 blocks, measured the same 14.3 us)
template <int MINB>
__global__ void __launch_bounds__(kStTPB, MINB) k_directive(Tables T, int kind, uint32_t lo, uint32_t n, uint32_t seq,
                                                            int discard_off, unsigned long long tail0) {
  pdl_enter();
  directive_body<8>(T, kind, lo, n, seq, discard_off, tail0);
}

// ------------------------------------------------------------------------------------
// K7: stable compaction of a ring's live entries [head, tail) into `dst`, right-aligned:
// the live entries keep their order and end at the same tail, so ring tails only ever
// grow by appends and the host knows them exactly (it passes them to the appending
// kernels).  Entries are ranked from the tail backwards (tile 0 holds the newest).
// ------------------------------------------------------------------------------------
__global__ void __launch_bounds__(kScanTPB) k_ring_compact(Tables T, int ring, uint64_t* dst) {
  pdl_enter();
  constexpr int NW = kScanTPB / 32;
  __shared__ uint32_t s_off[kScanIPT * NW + 1];
  __shared__ unsigned long long s_excl, s_tail, s_n;
  Ctl* c = T.ctl;
  if (threadIdx.x == 0) {
    const unsigned long long hd = ring == RING_USED ? c->used_head : c->disc_head;
    s_tail = ring == RING_USED ? c->used_tail : c->disc_tail;
    s_n = s_tail - hd;
  }
  __syncthreads();
  const uint32_t tile = blockIdx.x;
  const uint32_t ntiles = gridDim.x;
  const uint64_t* R = ring == RING_USED ? T.used_ring : T.disc_ring;
  const unsigned long long n = s_n, tail = s_tail;
  const unsigned long long tbase = (unsigned long long)tile * kScanTile;
  const int w = threadIdx.x >> 5;
  unsigned long long e[kScanIPT];
  unsigned bL[kScanIPT], bZ[kScanIPT];
#pragma unroll
  for (int k = 0; k < kScanIPT; ++k) {
    const unsigned long long ri = tbase + k * kScanTPB + threadIdx.x;   // rank from the tail
    e[k] = 0;
    bool live = false;
    if (ri < n) {
      e[k] = R[(tail - 1 - ri) & T.cap_mask];
      const uint32_t blk = (uint32_t)e[k], kk = (uint32_t)(e[k] >> 32);
      live = entry_live(T, ring == RING_DISC, blk, kk);
    }
    bL[k] = __ballot_sync(FULL, live);
    bZ[k] = 0;
  }
  const uint32_t tt = ordered_offsets<kScanTPB, kScanIPT>(bL, bZ, s_off);
  const unsigned long long tot = pack2(tt & 0xffffu, 0);
  if (threadIdx.x < 32) {
    unsigned long long ex = lookback_warp(T, tile, tot);
    if (threadIdx.x == 0) s_excl = ex;
  }
  __syncthreads();
  const uint32_t eA = unpackA(s_excl);
  const unsigned lt = lanemask_lt();
#pragma unroll
  for (int k = 0; k < kScanIPT; ++k)
    if ((bL[k] >> (threadIdx.x & 31)) & 1)
      dst[(tail - 1 - (eA + (s_off[k * NW + w] & 0xffffu) + __popc(bL[k] & lt))) & T.cap_mask] = e[k];
  if (tile == ntiles - 1 && threadIdx.x == 0) {
    const unsigned long long total = unpackA(s_excl + tot);
    if (ring == RING_USED) c->used_head = tail - total;
    else c->disc_head = tail - total;
  }
  scan_finish(T, ntiles);
}

// ------------------------------------------------------------------------------------
// Device intake ("dedupe with the op bitmap"): a batch of accesses that is
// not already sorted and disjoint is deduplicated here, not on the host.
//   k_mark        every (split) record ORs its block range into obits (and wbits for a
//                 WRITE access): the union, duplicates and overlaps collapse for free
//   k_runs        one ordered scan over the bitmap words turns set-bit runs into sorted
//                 disjoint intervals (a run also breaks where the write flag changes):
//                 interval j = (first block, rank of that block among all set bits, W),
//                 ranked by block scan + decoupled look-back over word tiles
//   k_intake_clear zeroes the words again for the next batch
// ------------------------------------------------------------------------------------
__global__ void __launch_bounds__(256) k_mark(Tables T, const MarkRec* rec, uint32_t n) {
  pdl_enter();
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const MarkRec r = rec[i];
    const uint32_t lo = r.lo, hi = r.lo + r.cnt;   // blocks [lo, hi), cnt <= kMarkMaxBlocks
    for (uint32_t w = lo >> 5; w <= (hi - 1) >> 5; ++w) {
      const uint32_t a = max(lo, w << 5) - (w << 5), b = min(hi, (w + 1) << 5) - (w << 5);   // bits [a, b)
      const uint32_t mask = (b - a == 32) ? FULL : (((1u << (b - a)) - 1u) << a);
      atomicOr(&T.obits[w], mask);
      if (r.w) atomicOr(&T.wbits[w], mask);
    }
  }
}

constexpr int kRunTPB = 512, kRunIPT = 8, kRunTile = kRunTPB * kRunIPT;   // words per tile

__global__ void __launch_bounds__(kRunTPB) k_runs(Tables T, uint32_t w0, uint32_t w1) {
  pdl_enter();
  __shared__ unsigned long long s_sc[kRunTPB / 32];
  __shared__ unsigned long long s_excl;
  const uint32_t tile = blockIdx.x, ntiles = gridDim.x;
  const uint32_t first = w0 + tile * kRunTile + threadIdx.x * kRunIPT;   // this thread's words
  uint32_t o[kRunIPT], wb[kRunIPT], st[kRunIPT];
  uint32_t co = 0, cw = 0;   // carry: top bit of the previous word
  if (first < w1 && first > w0) {
    co = T.obits[first - 1] >> 31;
    cw = T.wbits[first - 1] >> 31;
  }
  uint32_t nS = 0, nB = 0;
#pragma unroll
  for (int q = 0; q < kRunIPT; ++q) {
    const uint32_t w = first + q;
    o[q] = w < w1 ? T.obits[w] : 0u;
    wb[q] = w < w1 ? T.wbits[w] : 0u;
  }
#pragma unroll
  for (int q = 0; q < kRunIPT; ++q) {
    // bit i starts an interval if it is set and (bit i-1 is clear or has the other W)
    const uint32_t P = (o[q] << 1) | co, PW = (wb[q] << 1) | cw;
    st[q] = o[q] & (~P | (wb[q] ^ PW));
    co = o[q] >> 31;
    cw = wb[q] >> 31;
    nS += __popc(st[q]);
    nB += __popc(o[q]);
  }
  unsigned long long tot;
  const unsigned long long pre = block_excl_scan<kRunTPB>(pack2(nS, nB), tot, s_sc);
  if (threadIdx.x < 32) {
    const unsigned long long ex = lookback_warp(T, tile, tot);
    if (threadIdx.x == 0) s_excl = ex;
  }
  __syncthreads();
  uint32_t J = unpackA(s_excl) + unpackA(pre), R = unpackB(s_excl) + unpackB(pre);
#pragma unroll
  for (int q = 0; q < kRunIPT; ++q) {
    uint32_t m = st[q];
    while (m) {
      const int i = __ffs(m) - 1;
      m &= m - 1;
      const uint32_t below = (1u << i) - 1u;
      T.dlo[J] = (first + q) * 32u + (uint32_t)i;
      T.dpre[J] = R + __popc(o[q] & below);
      T.dw[J] = (uint8_t)((wb[q] >> i) & 1u);
      ++J;
    }
    R += __popc(o[q]);
  }
  if (tile == ntiles - 1 && threadIdx.x == 0) {
    const unsigned long long all = s_excl + tot;
    T.ctl->iv_m = unpackA(all);
    T.ctl->iv_d = unpackB(all);
    T.dpre[unpackA(all)] = unpackB(all);
  }
  scan_finish(T, ntiles);
}

__global__ void __launch_bounds__(256) k_intake_clear(Tables T, uint32_t w0, uint32_t w1) {
  pdl_enter();
  for (uint32_t w = w0 + blockIdx.x * blockDim.x + threadIdx.x; w < w1; w += gridDim.x * blockDim.x) {
    T.obits[w] = 0u;
    T.wbits[w] = 0u;
  }
}

// ------------------------------------------------------------------------------------
// Device-resident access records (um_touch_batch_dev; SURVEY A0/A1 on the device): the
// GPU's own fault buffer analogue.  The records never visit the host.
//   k_mark_acc  one thread per 16-byte record: the API's range check (a record outside
//               the arena sets ctl->iv_err; the host then rejects the op), blocks
//               [off/B, (off+len-1)/B] ORed into obits (and wbits for a WRITE access)
//   k_list      one ordered pass over the bitmap words: the set bits, ascending, become
//               the distinct block list (bit 31 = write) that the LIST classify reads
//               (dlo), ranked by block scan + decoupled look-back; every word is zeroed
//               once read (the bitmaps are clean for the next batch); the last tile
//               publishes the block count (ctl->iv_d) and the write count (ctl->iv_m)
// ------------------------------------------------------------------------------------
constexpr int kMarkIPT = 8;   // consecutive records per thread, all loads in flight

// Each thread takes kMarkIPT CONSECUTIVE records: in a sorted fault batch they fall in
// one or two bitmap words, so the thread ORs their bits in a register and issues one
// atomic per word it leaves (no cross-lane work; the ALU cost per record is a few
// integer ops).  Unsorted records just flush more often.
__global__ void __launch_bounds__(256) k_mark_acc(Tables T, const ulonglong2* acc, uint32_t n, uint32_t lg) {
  pdl_enter();
  const unsigned long long arena = (unsigned long long)T.nblocks << lg;
  const uint32_t stride = gridDim.x * blockDim.x * kMarkIPT;
  for (uint32_t i0 = (blockIdx.x * blockDim.x + threadIdx.x) * kMarkIPT; i0 < n; i0 += stride) {
    ulonglong2 r[kMarkIPT];
#pragma unroll
    for (int q = 0; q < kMarkIPT; ++q)   // {off, len | kind << 32} (um_access); len 0 = nothing
      r[q] = i0 + q < n ? __ldg(acc + i0 + q) : make_ulonglong2(0ull, 0ull);
    uint32_t cw = UM_NONE, cm = 0u, cmw = 0u;   // the word being accumulated
#pragma unroll
    for (int q = 0; q < kMarkIPT; ++q) {
      const unsigned long long off = r[q].x, len = (uint32_t)r[q].y;
      const bool w = ((uint32_t)(r[q].y >> 32) & 2u) != 0;   // UM_ACC_WRITE (include/um.h)
      if (off > arena || len > arena - off) {
        T.ctl->iv_err = 1u;
        continue;
      }
      if (!len) continue;
      const uint32_t lo = (uint32_t)(off >> lg), hi = (uint32_t)((off + len - 1) >> lg) + 1u;
      if ((lo >> 5) == ((hi - 1) >> 5)) {
        const uint32_t wd = lo >> 5, a = lo & 31u, c = hi - lo;
        const uint32_t m = (c == 32) ? FULL : (((1u << c) - 1u) << a);
        if (wd != cw) {
          if (cw != UM_NONE) {
            atomicOr(&T.obits[cw], cm);
            if (cmw) atomicOr(&T.wbits[cw], cmw);
          }
          cw = wd;
          cm = cmw = 0u;
        }
        cm |= m;
        if (w) cmw |= m;
      } else {
        for (uint32_t x = lo >> 5; x <= (hi - 1) >> 5; ++x) {
          const uint32_t a = max(lo, x << 5) - (x << 5), b = min(hi, (x + 1) << 5) - (x << 5);   // bits [a, b)
          const uint32_t mask = (b - a == 32) ? FULL : (((1u << (b - a)) - 1u) << a);
          atomicOr(&T.obits[x], mask);
          if (w) atomicOr(&T.wbits[x], mask);
        }
      }
    }
    if (cw != UM_NONE) {
      atomicOr(&T.obits[cw], cm);
      if (cmw) atomicOr(&T.wbits[cw], cmw);
    }
  }
}

// one bitmap word per thread, 1024 words per tile (few tiles: a short look-back); a
// tile's list entries are staged in shared memory (<= 32 per word, 128 KB) and written
// out coalesced
constexpr int kListTPB = 1024, kListTile = kListTPB;   // words per tile
constexpr int kListSmem = kListTile * 32 * 4;

__global__ void __launch_bounds__(kListTPB) k_list(Tables T, uint32_t nwords) {
  pdl_enter();
  __shared__ unsigned long long s_sc[kListTPB / 32];
  __shared__ unsigned long long s_excl;
  extern __shared__ uint32_t s_ent[];
  const uint32_t tile = blockIdx.x, ntiles = gridDim.x;
  const uint32_t wd = tile * kListTile + threadIdx.x;
  const uint32_t o = wd < nwords ? T.obits[wd] : 0u;
  const uint32_t wb = (wd < nwords ? T.wbits[wd] : 0u) & o;
  const uint32_t nB = __popc(o), nW = __popc(wb);
  unsigned long long tot;
  const unsigned long long pre = block_excl_scan<kListTPB>(pack2(nB, nW), tot, s_sc);
  if (threadIdx.x < 32) {
    const unsigned long long ex = lookback_warp(T, tile, tot);
    if (threadIdx.x == 0) s_excl = ex;
  }
  uint32_t r = unpackA(pre), m = o;
  while (m) {
    const int i = __ffs(m) - 1;
    m &= m - 1;
    s_ent[r++] = (wd * 32u + (uint32_t)i) | (((wb >> i) & 1u) << 31);
  }
  // clear the words read (each is read by this thread only)
  if (wd < nwords) {
    if (o) T.obits[wd] = 0u;
    if (wb) T.wbits[wd] = 0u;   // write bits are only ever set with their obits bit
  }
  __syncthreads();
  const uint32_t base = unpackA(s_excl), cnt = unpackA(tot);
  for (uint32_t k = threadIdx.x; k < cnt; k += kListTPB) T.dlo[base + k] = s_ent[k];
  if (tile == ntiles - 1 && threadIdx.x == 0) {
    const unsigned long long all = s_excl + tot;
    T.ctl->iv_d = unpackA(all);
    T.ctl->iv_m = unpackB(all);
  }
  scan_finish(T, ntiles);
}

// ------------------------------------------------------------------------------------
// Harness: host writes (Listing 6 "Generate data, labels").
// ------------------------------------------------------------------------------------
// um_free (reading R9): blocks [lo, lo + n) return to U with no transfer.  A GPU frame
// goes back to the free pool (the paper's unused queue is reclaimed before the
// discarded one and without a transfer, §5.5; frames are anonymous), a host
// copy is released; the block's ring entries go stale by the liveness rule.
__global__ void __launch_bounds__(256) k_free(Tables T, uint32_t lo, uint32_t n) {
  pdl_enter();
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const uint32_t bb = lo + i;
    const uint8_t ss = ld_st(T, bb);
    if (ss == ST_U) continue;
    if (ss == ST_G || ss == ST_GE || ss == ST_GL) {
      const int idx = atomicAdd(&T.ctl->free_top, 1);
      T.free_stack[idx] = T.frame_of[bb];
      T.frame_of[bb] = UM_NONE;
      T.map[bb] = UM_NONE;
    } else if (T.hframe[bb] != UM_NONE) {   // H (HD holds none, R1)
      const int idx = atomicAdd(&T.ctl->hfree_top, 1);
      T.hfree_stack[idx] = T.hframe[bb];
      T.hframe[bb] = UM_NONE;
    }
    T.sk[bb] = mk_sk(ST_U, 0);
    if (T.pdead) T.pdead[bb] = T.plazy[bb] = T.phz[bb] = 0u;
  }
}

// Pages [p0, p1) of chunk c (global page indices) as a mask of the chunk's pages.
__device__ __forceinline__ uint32_t chunk_mask(const Tables& T, uint32_t c, unsigned long long p0, unsigned long long p1) {
  const unsigned long long c0 = (unsigned long long)c * T.ppc;
  const uint32_t a = p0 > c0 ? (uint32_t)(p0 - c0) : 0u;
  const uint32_t e = p1 < c0 + T.ppc ? (uint32_t)(p1 - c0) : T.ppc;
  return (e >= 32 ? 0xffffffffu : ((1u << e) - 1u)) & ~((1u << a) - 1u);
}

// Host write of pages [p0, p1): chunks [lo, lo + n) must be H; a chunk without a host
// frame (zero content) gets one, and its pages the write does not cover stay logically
// zero (phz).  The written pages become live (not dead, not zero).
__global__ void k_hw_alloc(Tables T, uint32_t lo, uint32_t n, unsigned long long p0, unsigned long long p1) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    uint32_t bb = lo + i;
    if (ld_st(T, bb) != ST_H) {
      atomicExch(&T.ctl->err, 1u);
      continue;
    }
    const uint32_t m = T.pdead ? chunk_mask(T, bb, p0, p1) : 0u;
    bool fresh = false;
    if (T.hframe[bb] == UM_NONE) {
      int idx = atomicSub(&T.ctl->hfree_top, 1) - 1;
      if (idx >= 0) {
        T.hframe[bb] = T.hfree_stack[idx];
        fresh = true;
      } else {
        atomicAdd(&T.ctl->hfree_top, 1);
        atomicExch(&T.ctl->err, 2u);
      }
    }
    if (T.pdead) {
      const uint32_t full = T.ppc >= 32 ? 0xffffffffu : ((1u << T.ppc) - 1u);
      T.phz[bb] = fresh ? (full & ~m) : (T.phz[bb] & ~m);
      T.pdead[bb] &= ~m;
      T.plazy[bb] &= ~m;
    }
  }
}

__global__ void __launch_bounds__(256) k_hw_fill(Tables T, unsigned long long p0, unsigned long long p1, uint32_t seq) {
  const uint32_t CH = T.P < kXferChunk ? T.P : kXferChunk;
  const uint32_t cpp = T.P / CH;
  const unsigned long long units = (p1 - p0) * cpp;
  for (unsigned long long u = blockIdx.x; u < units; u += gridDim.x) {
    const unsigned long long q = p0 + u / cpp;   // global page
    const uint32_t bb = (uint32_t)(q / T.ppc), pg = (uint32_t)(q % T.ppc), ch = (uint32_t)(u % cpp);
    uint32_t hf = T.hframe[bb];
    if (hf == UM_NONE || ld_st(T, bb) != ST_H) continue;
    unsigned long long sv = ((unsigned long long)seq << 32) | (uint32_t)q;
    uint4 pat = make_uint4((uint32_t)sv, (uint32_t)(sv >> 32), ~(uint32_t)sv, ~(uint32_t)(sv >> 32));
    uint4* dst = reinterpret_cast<uint4*>(hptr(T, hf) + (size_t)pg * T.P + (size_t)ch * CH);
    for (uint32_t t = threadIdx.x; t < CH / 16; t += blockDim.x) dst[t] = pat;
  }
}

// ------------------------------------------------------------------------------------
// Harness: content tag of every block (0 = zeros, s = uniform {s,~s}, ~0 = corrupt).
// ------------------------------------------------------------------------------------
__global__ void __launch_bounds__(256) k_tags(Tables T) {
  // one tag per page (= per block at single level); dead pages and zero-content pages
  // of an H chunk hold no data on the host and read as zero (R1)
  const unsigned long long npages = (unsigned long long)T.nblocks * T.ppc;
  for (unsigned long long q = blockIdx.x; q < npages; q += gridDim.x) {
    const uint32_t bb = (uint32_t)(q / T.ppc), pg = (uint32_t)(q % T.ppc);
    uint8_t ss = ld_st(T, bb);
    const uint4* src = nullptr;
    if (ss == ST_G || ss == ST_GE || ss == ST_GL) {
      uint32_t fr = T.frame_of[bb];
      if (fr != UM_NONE) src = reinterpret_cast<const uint4*>(T.frames + (size_t)fr * T.B + (size_t)pg * T.P);
    } else if (ss == ST_H) {
      uint32_t hf = T.hframe[bb];
      const bool nodata = T.pdead && (((T.pdead[bb] | T.phz[bb]) >> pg) & 1u);
      if (hf != UM_NONE && !nodata) src = reinterpret_cast<const uint4*>(hptr(T, hf) + (size_t)pg * T.P);
    }
    if (!src) {
      if (threadIdx.x == 0) T.tags[q] = (ss == ST_G || ss == ST_GE || ss == ST_GL) ? ~0ull : 0ull;
      continue;
    }
    uint4 v0 = src[0];
    bool ok = true;
    for (uint32_t t = threadIdx.x; t < T.P / 16; t += blockDim.x) {
      uint4 v = src[t];
      ok &= (v.x == v0.x) & (v.y == v0.y) & (v.z == v0.z) & (v.w == v0.w);
    }
    ok = __syncthreads_and(ok);
    if (threadIdx.x == 0) {
      unsigned long long s = (unsigned long long)v0.x | ((unsigned long long)v0.y << 32);
      unsigned long long ns = (unsigned long long)v0.z | ((unsigned long long)v0.w << 32);
      unsigned long long tag;
      if (!ok) tag = ~0ull;
      else if (s == 0 && ns == 0) tag = 0;
      else if (ns == ~s && s != 0) tag = s;
      else tag = ~0ull;
      T.tags[q] = tag;
    }
    __syncthreads();
  }
}

// ------------------------------------------------------------------------------------
// launch wrappers
// ------------------------------------------------------------------------------------
static int g_nsm = 0;
// k_classify CTA size: 256 threads x 4 items (UM_CLS_TPB=512: 512 x 4, half the CTAs,
// need-list atomics and counter reductions; A/B)
static int g_cls_tpb = 256;
static int g_vscan_occ = 1;   // resident k_victims_scan CTAs per SM
static bool g_pdl = true;     // UM_PDL=0 disables programmatic dependent launch (A/B)
static int g_dir_occ = 8;     // resident k_directive CTAs per SM (persistent grid)
static int g_dir_minb = 6;    // k_directive CTAs/SM the registers allow: 6 (40 regs); UM_DIR_MINB=7/8 (36/32 regs: one wave for 2^21 blocks) for A/B
static int g_vs_ctas = 0;     // UM_VS_CTAS=n caps the victim scan grid at n CTAs (test hook: small tables then take tiles by ticket and skip past the k-th candidate)
static int g_vs_prefetch = 0; // UM_VS_PREFETCH=1: the wide victim scan fetches its next ticket a tile ahead (A/B on B200: 79 vs 73 us pressured touch -- the earlier snapshot reads more tiles past the k-th candidate)

cudaError_t setup_kernels() {
  int dev;
  cudaError_t e = cudaGetDevice(&dev);
  if (e) return e;
  e = cudaDeviceGetAttribute(&g_nsm, cudaDevAttrMultiProcessorCount, dev);
  if (e) return e;
  if (const char* v = getenv("UM_PDL")) g_pdl = atoi(v) != 0;
  if (const char* v = getenv("UM_VS_PREFETCH")) g_vs_prefetch = atoi(v) != 0;
  if (const char* v = getenv("UM_VS_CTAS")) g_vs_ctas = atoi(v) > 0 ? atoi(v) : 0;
  if (const char* v = getenv("UM_CLS_TPB")) g_cls_tpb = atoi(v) == 512 ? 512 : 256;
  // Optionally one L1/shared carveout for every paging kernel (k_service needs 144 KB of
  // shared memory; a carveout change between consecutive kernels can force an SM drain).
  // UM_CARVEOUT=1 turns it on (A/B; off by default).
  bool carve = false;   // measured: no effect on the C1 small-op rate (B200, r01)
  if (const char* v = getenv("UM_CARVEOUT")) carve = atoi(v) != 0;
  if (carve) {
    const void* ks[] = {(const void*)k_classify<false, 256>, (const void*)k_classify<true, 256>,
                        (const void*)k_classify<false, 512>, (const void*)k_classify<true, 512>, (const void*)k_victims, (const void*)k_plan_small,
                        (const void*)k_victims_scan, (const void*)k_victims_apply, (const void*)k_service,
                        (const void*)k_app_stamp<256>, (const void*)k_app_stamp<128>, (const void*)k_directive<6>, (const void*)k_directive<7>, (const void*)k_directive<8>,
                        (const void*)k_ring_compact,
                        (const void*)k_plan_commit, (const void*)k_zero_items, (const void*)k_mark,
                        (const void*)k_runs, (const void*)k_intake_clear};
    for (const void* k : ks) {
      e = cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, (int)cudaSharedmemCarveoutMaxShared);
      if (e) return e;
    }
  }
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&g_vscan_occ, k_victims_scan, kVsTPB, 0);
  if (e) return e;
  if (g_vscan_occ < 1) g_vscan_occ = 1;
  if (const char* v = getenv("UM_DIR_MINB")) g_dir_minb = std::min(8, std::max(6, atoi(v)));
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(
      &g_dir_occ,
      g_dir_minb == 8 ? (const void*)k_directive<8> : g_dir_minb == 7 ? (const void*)k_directive<7> : (const void*)k_directive<6>,
      kStTPB, 0);
  if (e) return e;
  if (g_dir_occ < 1) g_dir_occ = 1;
  if (const char* v = getenv("UM_DIR_OCC")) g_dir_occ = std::max(1, atoi(v));
  e = cudaFuncSetAttribute(k_list, cudaFuncAttributeMaxDynamicSharedMemorySize, kListSmem);
  if (e) return e;
  int smem = (int)(kXferChunk * (1 + 2 * kXferStages));
  return cudaFuncSetAttribute(k_service, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
}


// Launch on `s` with programmatic stream serialization (see pdl_enter).
template <typename... KArgs, typename... Args>
static cudaError_t launch_pdl(void (*k)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                              Args... args) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = g_pdl ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, k, static_cast<KArgs>(args)...);
}

static inline unsigned ceil_div(unsigned long long a, unsigned long long b) { return (unsigned)((a + b - 1) / b); }

cudaError_t launch_init(const Tables& T, int nh, cudaStream_t s) {
  k_init<<<g_nsm * 4, 256, 0, s>>>(T, nh);
  return cudaGetLastError();
}

cudaError_t launch_poison(const Tables& T, cudaStream_t s) {
  k_poison<<<g_nsm * 4, 512, 0, s>>>(T.frames, (size_t)T.nframes * T.B);
  return cudaGetLastError();
}

uint32_t classify_tile() { return (uint32_t)g_cls_tpb * 4u; }

cudaError_t launch_classify(const Tables& T, OpIv iv, uint32_t g0, uint32_t n, uint32_t seq, int touch,
                            unsigned long long tail0, int npar, int k0, cudaStream_t s) {
  unsigned nt = n ? ceil_div(n, classify_tile()) : 1;
  cudaError_t le__;
  if (g_cls_tpb == 512)
    le__ = iv.blist ? launch_pdl(k_classify<true, 512>, dim3(nt), dim3(512), 0, s, T, iv, g0, n, seq, touch, tail0, npar, k0)
                    : launch_pdl(k_classify<false, 512>, dim3(nt), dim3(512), 0, s, T, iv, g0, n, seq, touch, tail0, npar, k0);
  else
    le__ = iv.blist ? launch_pdl(k_classify<true, 256>, dim3(nt), dim3(256), 0, s, T, iv, g0, n, seq, touch, tail0, npar, k0)
                    : launch_pdl(k_classify<false, 256>, dim3(nt), dim3(256), 0, s, T, iv, g0, n, seq, touch, tail0, npar, k0);
  if (le__) return le__;
  return cudaGetLastError();
}

cudaError_t launch_victims(const Tables& T, uint32_t seq, int evict_mode, uint32_t want, int npar, cudaStream_t s) {
  cudaError_t le__ = launch_pdl(k_victims, dim3(1), dim3(kVictTPB), 0, s, T, seq, evict_mode, want, npar);
  if (le__) return le__;
  return cudaGetLastError();
}

cudaError_t launch_plan_small(const Tables& T, const OpIv& iv, uint32_t g0, uint32_t n, uint32_t seq, int touch,
                              unsigned long long tail0, cudaStream_t s) {
  cudaError_t le__ = launch_pdl(k_plan_small, dim3(1), dim3(kVictTPB), 0, s, T, iv, g0, n, seq, touch, tail0);
  if (le__) return le__;
  return cudaGetLastError();
}

cudaError_t launch_victims_wide(const Tables& T, uint32_t seq, int evict_mode, uint32_t want, uint64_t scan_bound,
                                uint32_t max_victims, int npar, cudaStream_t s) {
  // persistent scan grid: never more CTAs than can be resident (tiles are taken from a
  // ticket in order and a tile may wait on its predecessors' status)
  unsigned nt = ceil_div(scan_bound ? scan_bound : 1, kVsTile);
  const unsigned cap = g_vs_ctas ? (unsigned)g_vs_ctas : (unsigned)(g_nsm * g_vscan_occ);
  cudaError_t le__ = launch_pdl(k_victims_scan, dim3(nt < cap ? nt : cap), dim3(kVsTPB), 0, s, T, seq, evict_mode, want, npar, g_vs_prefetch);
  if (le__) return le__;
  cudaError_t e = cudaGetLastError();
  if (e) return e;
  // one warp per pass of <= kVaPass victims (<= max_victims / kVaPass + tiles passes)
  unsigned grid = ceil_div((unsigned long long)ceil_div(max_victims ? max_victims : 1, kVaPass) + nt, kVaTPB / 32);
  if (grid > (unsigned)g_nsm * 2) grid = g_nsm * 2;
  le__ = launch_pdl(k_victims_apply, dim3(grid), dim3(kVaTPB), 0, s, T, evict_mode, seq);
  if (le__) return le__;
  return cudaGetLastError();
}

cudaError_t launch_service(const Tables& T, int mode, uint32_t seq, uint32_t max_items, cudaStream_t s) {
  const uint32_t CH = T.B < kXferChunk ? T.B : kXferChunk;
  unsigned long long units = (unsigned long long)max_items * (T.B / CH);
  unsigned grid = (unsigned)(units < (unsigned long long)g_nsm ? units : (unsigned long long)g_nsm);
  if (grid == 0) grid = 1;
  size_t smem = (size_t)CH * (1 + 2 * kXferStages);
  cudaError_t le__ = launch_pdl(k_service, dim3(grid), dim3(32 * kSvcWarps), smem, s, T, mode, seq);
  if (le__) return le__;
  return cudaGetLastError();
}

cudaError_t launch_app_stamp(const Tables& T, OpIv iv, uint32_t g0, uint32_t n, uint32_t seq, int ctas_per_sm,
                             cudaStream_t s) {
  const uint32_t SEG = T.P < kFillSeg ? T.P : kFillSeg;
  unsigned long long units = (unsigned long long)n * (T.B / SEG);
  // ctas_per_sm < 0: a grid of -ctas_per_sm CTAs in total (a bandwidth-capped background kernel)
  const unsigned long long cap = ctas_per_sm < 0 ? (unsigned long long)(-ctas_per_sm)
                                                 : (unsigned long long)g_nsm * ctas_per_sm;
  unsigned grid = (unsigned)(units < cap ? units : cap);
  if (!grid) return cudaSuccess;
  cudaError_t le__ = ctas_per_sm >= 8 ? launch_pdl(k_app_stamp<256>, dim3(grid), dim3(256), 0, s, T, iv, g0, n, seq)
                                      : launch_pdl(k_app_stamp<128>, dim3(grid), dim3(128), 0, s, T, iv, g0, n, seq);
  if (le__) return le__;
  return cudaGetLastError();
}

cudaError_t launch_directive(const Tables& T, int kind, uint32_t lo, uint32_t n, uint32_t seq, int discard_off,
                             unsigned long long tail0, cudaStream_t s) {
  unsigned nt = n ? ceil_div(n, kStTPB * 8) : 1;
  if (nt > (unsigned)(g_nsm * g_dir_occ)) nt = (unsigned)(g_nsm * g_dir_occ);   // persistent
  cudaError_t le__ =
      g_dir_minb == 8   ? launch_pdl(k_directive<8>, dim3(nt), dim3(kStTPB), 0, s, T, kind, lo, n, seq, discard_off, tail0)
      : g_dir_minb == 7 ? launch_pdl(k_directive<7>, dim3(nt), dim3(kStTPB), 0, s, T, kind, lo, n, seq, discard_off, tail0)
                        : launch_pdl(k_directive<6>, dim3(nt), dim3(kStTPB), 0, s, T, kind, lo, n, seq, discard_off, tail0);
  if (le__) return le__;
  return cudaGetLastError();
}

cudaError_t launch_ring_compact(const Tables& T, int ring, uint64_t* dst, uint64_t cap_bound, cudaStream_t s) {
  unsigned nt = ceil_div(cap_bound ? cap_bound : 1, kScanTile);
  cudaError_t le__ = launch_pdl(k_ring_compact, dim3(nt), dim3(kScanTPB), 0, s, T, ring, dst);
  if (le__) return le__;
  return cudaGetLastError();
}

cudaError_t launch_host_write(const Tables& T, uint64_t p0, uint64_t p1, uint32_t seq, cudaStream_t s) {
  if (p1 <= p0) return cudaSuccess;
  const uint32_t lo = (uint32_t)(p0 / T.ppc), n = (uint32_t)((p1 - 1) / T.ppc + 1 - lo);
  k_hw_alloc<<<ceil_div(n, 256), 256, 0, s>>>(T, lo, n, p0, p1);
  const uint32_t CH = T.P < kXferChunk ? T.P : kXferChunk;
  unsigned long long units = (p1 - p0) * (T.P / CH);
  unsigned grid = (unsigned)(units < (unsigned long long)g_nsm * 8 ? units : (unsigned long long)g_nsm * 8);
  k_hw_fill<<<grid, 256, 0, s>>>(T, p0, p1, seq);
  return cudaGetLastError();
}

cudaError_t launch_free(const Tables& T, uint32_t lo, uint32_t n, cudaStream_t s) {
  if (!n) return cudaSuccess;
  unsigned grid = ceil_div(n, 256);
  if (grid > (unsigned)g_nsm * 8) grid = g_nsm * 8;
  cudaError_t e = launch_pdl(k_free, dim3(grid), dim3(256), 0, s, T, lo, n);
  if (e) return e;
  return cudaGetLastError();
}

cudaError_t launch_page_revive(const Tables& T, const OpIv& iv, uint32_t g0, uint32_t n, int touch, cudaStream_t s) {
  if (!n) return cudaSuccess;
  unsigned grid = ceil_div(n, 256);
  if (grid > (unsigned)g_nsm * 4) grid = g_nsm * 4;
  cudaError_t e = launch_pdl(k_page_revive, dim3(grid), dim3(256), 0, s, T, iv, g0, n, touch);
  if (e) return e;
  return cudaGetLastError();
}

cudaError_t launch_page_host_revive(const Tables& T, uint32_t lo, uint32_t n, uint64_t p0, uint64_t p1,
                                    cudaStream_t s) {
  if (!n) return cudaSuccess;
  unsigned grid = ceil_div(n, 256);
  if (grid > (unsigned)g_nsm * 4) grid = g_nsm * 4;
  cudaError_t e = launch_pdl(k_page_host_revive, dim3(grid), dim3(256), 0, s, T, lo, n,
                             (unsigned long long)p0, (unsigned long long)p1);
  if (e) return e;
  return cudaGetLastError();
}

cudaError_t launch_page_discard(const Tables& T, uint32_t c0, uint32_t m0, uint32_t c1, uint32_t m1, int lazy,
                                cudaStream_t s) {
  cudaError_t e = launch_pdl(k_page_discard, dim3(1), dim3(32), 0, s, T, c0, m0, c1, m1, lazy);
  if (e) return e;
  return cudaGetLastError();
}

cudaError_t launch_plan_commit(const Tables& T, uint32_t seq, uint32_t max_items, cudaStream_t s) {
  unsigned grid = ceil_div(max_items ? max_items : 1, 256);
  cudaError_t le__ = launch_pdl(k_plan_commit, dim3(grid), dim3(256), 0, s, T, seq);
  if (le__) return le__;
  return cudaGetLastError();
}

cudaError_t launch_zero_items(const Tables& T, uint32_t i0, uint32_t i1, cudaStream_t s) {
  const uint32_t SEG = T.B < kFillSeg ? T.B : kFillSeg;
  unsigned long long units = (unsigned long long)(i1 - i0) * (T.B / SEG);
  unsigned grid = (unsigned)(units < (unsigned long long)g_nsm * 8 ? units : (unsigned long long)g_nsm * 8);
  if (!grid) return cudaSuccess;
  k_zero_items<<<grid, 256, 0, s>>>(T, i0, i1);
  return cudaGetLastError();
}

cudaError_t launch_tags(const Tables& T, cudaStream_t s) {
  const unsigned long long np = (unsigned long long)T.nblocks * T.ppc;
  unsigned grid = np < (unsigned long long)g_nsm * 16 ? (unsigned)np : (unsigned)g_nsm * 16;
  if (!grid) grid = 1;
  k_tags<<<grid, 256, 0, s>>>(T);
  return cudaGetLastError();
}

cudaError_t launch_mark(const Tables& T, const MarkRec* rec, uint32_t n, cudaStream_t s) {
  if (!n) return cudaSuccess;
  unsigned grid = ceil_div(n, 256);
  if (grid > (unsigned)g_nsm * 8) grid = g_nsm * 8;
  cudaError_t e = launch_pdl(k_mark, dim3(grid), dim3(256), 0, s, T, rec, n);
  if (e) return e;
  return cudaGetLastError();
}

cudaError_t launch_runs(const Tables& T, uint32_t w0, uint32_t w1, cudaStream_t s) {
  unsigned nt = w1 > w0 ? ceil_div(w1 - w0, kRunTile) : 1;
  cudaError_t e = launch_pdl(k_runs, dim3(nt), dim3(kRunTPB), 0, s, T, w0, w1);
  if (e) return e;
  return cudaGetLastError();
}

cudaError_t launch_intake_clear(const Tables& T, uint32_t w0, uint32_t w1, cudaStream_t s) {
  if (w1 <= w0) return cudaSuccess;
  unsigned grid = ceil_div(w1 - w0, 256);
  if (grid > (unsigned)g_nsm * 8) grid = g_nsm * 8;
  cudaError_t e = launch_pdl(k_intake_clear, dim3(grid), dim3(256), 0, s, T, w0, w1);
  if (e) return e;
  return cudaGetLastError();
}

cudaError_t launch_mark_acc(const Tables& T, const void* acc, uint32_t n, uint32_t lg, cudaStream_t s) {
  if (!n) return cudaSuccess;
  unsigned grid = ceil_div(n, 256 * kMarkIPT);
  if (grid > (unsigned)g_nsm * 8) grid = g_nsm * 8;
  cudaError_t e = launch_pdl(k_mark_acc, dim3(grid), dim3(256), 0, s, T, (const ulonglong2*)acc, n, lg);
  if (e) return e;
  return cudaGetLastError();
}

cudaError_t launch_list(const Tables& T, uint32_t nwords, cudaStream_t s) {
  unsigned nt = nwords ? ceil_div(nwords, kListTile) : 1;
  cudaError_t e = launch_pdl(k_list, dim3(nt), dim3(kListTPB), (size_t)kListSmem, s, T, nwords);
  if (e) return e;
  return cudaGetLastError();
}

}  // namespace um

#ifdef UM_VS_TRACE
extern "C" __attribute__((visibility("default"))) int um_debug_vs_trace(void* host, unsigned long long bytes) {
  return (int)cudaMemcpyFromSymbol(host, um::g_vs_tr, bytes);
}
#endif
