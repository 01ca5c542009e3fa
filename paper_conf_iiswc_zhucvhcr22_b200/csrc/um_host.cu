// Host runtime and C ABI of libum (include/um.h).
//
// The host side never inspects block states: it validates arguments, turns a batch of
// accesses into sorted disjoint block intervals, splits GPU-destination ops into
// sub-ops of <= nframes blocks (reading A3 of DESIGN.md), assigns sequence numbers,
// stages the interval lists to the device and enqueues the kernel chain of
// um_kernels.cu on the arena's paging stream.  All planning is on the device, so the
// kernel-driven transfer path never round-trips to the host inside an op.
#include "um_internal.h"

#include <algorithm>
#include <atomic>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <deque>
#include <new>
#include <chrono>
#include <vector>

#include "../../include/um.h"

#define UM_API extern "C" __attribute__((visibility("default")))

using namespace um;

namespace {

constexpr uint64_t kAlign = 256;

struct Layout {
  uint64_t sk, frame_of, map, hframe, pin, free_stack, hfree_stack;
  uint64_t used[2], disc[2];
  uint64_t need, needk, needhf, victim, vframe, vhf, vkind, d2h_frame, d2h_hf;
  uint64_t tile_status, tile_cnt, tags, ctl, hchunks, stage, xitems, bounce;
  uint64_t obits, wbits, dlo, dpre, dw, vscratch, vpass;
  uint64_t pdead, plazy, phz, d2h_dmask;
  uint64_t stage_bytes, max_tiles, cap, total, ce_group, bounce_bytes;
};

static uint64_t pow2_ceil(uint64_t x) {
  uint64_t p = 1;
  while (p < x) p <<= 1;
  return p;
}

static bool is_pow2(uint64_t x) { return x && !(x & (x - 1)); }

// Pages per chunk: 1 at single level (page_bytes 0 or = block_bytes).
static uint32_t cfg_ppc(const um_config* c) {
  return (c->page_bytes == 0 || c->page_bytes == c->block_bytes) ? 1u : c->block_bytes / c->page_bytes;
}

static um_status check_cfg(const um_config* c) {
  if (!c) return UM_EINVAL;
  if (c->page_bytes && c->page_bytes != c->block_bytes) {   // two-level granularity (NEXT-1)
    if (!is_pow2(c->page_bytes) || c->page_bytes < kXferChunk || c->page_bytes > c->block_bytes ||
        c->block_bytes / c->page_bytes > 32)
      return UM_EINVAL;
    if (c->flags & (UM_F_COPY_CE | UM_F_OVERLAP)) return UM_EINVAL;
    if (c->reserve_blocks) return UM_EINVAL;
  }
  if (!is_pow2(c->block_bytes) || c->block_bytes < 4096) return UM_EINVAL;
  if (c->arena_bytes == 0 || c->arena_bytes % c->block_bytes) return UM_EINVAL;
  // block ids < 2^31: bit 31 of a staged list entry is the write flag (fault-list and
  // two-level chunk-list forms)
  if (c->arena_bytes / c->block_bytes >= 0x80000000ull) return UM_EINVAL;
  if (c->budget_bytes < c->block_bytes) return UM_EINVAL;
  if (c->budget_bytes / c->block_bytes >= 0x7fffffffull) return UM_EINVAL;
  if (c->reserve_blocks > c->budget_bytes / c->block_bytes) return UM_EINVAL;
  if (c->host_chunk_bytes == 0 || c->host_chunk_bytes % c->block_bytes) return UM_EINVAL;
  if (c->n_host_chunks == 0) return UM_EINVAL;
  if ((uint64_t)c->n_host_chunks * (c->host_chunk_bytes / c->block_bytes) < 2) return UM_EINVAL;
  return UM_OK;
}

static Layout make_layout(const um_config* c) {
  Layout L{};
  const uint64_t nb = c->arena_bytes / c->block_bytes;
  const uint64_t nf = c->budget_bytes / c->block_bytes;
  const uint64_t nh = (uint64_t)c->n_host_chunks * (c->host_chunk_bytes / c->block_bytes);
  L.cap = pow2_ceil(std::max<uint64_t>(1024, 4 * nf));
  // tiles: classify/directive scan <= nblocks items, compaction <= cap, the wide victim
  // scan <= |DISC| + |USED| <= 2 * cap (its bound is also clamped to 2 * cap)
  L.max_tiles = (std::max(nb, 2 * L.cap) + 2048 - 1) / 2048 + 1;   // smallest scan tile: 2048 items
  const uint64_t ppc = cfg_ppc(c);
  // staged touch lists: 12 B per distinct block at two levels (chunk, cover, write masks)
  L.stage_bytes = std::min<uint64_t>(64ull << 20, (ppc > 1 ? 24 : 12) * nb + (1 << 20));
  uint64_t o = 0;
  auto take = [&](uint64_t bytes) {
    uint64_t r = o;
    o += (bytes + kAlign - 1) / kAlign * kAlign;
    return r;
  };
  L.sk = take(4 * nb);
  L.frame_of = take(4 * nb);
  L.map = take(4 * nb);
  L.hframe = take(4 * nb);
  L.pin = take(4 * nb);
  L.free_stack = take(4 * nf);
  L.hfree_stack = take(4 * nh);
  for (int i = 0; i < 2; ++i) L.used[i] = take(8 * L.cap);
  for (int i = 0; i < 2; ++i) L.disc[i] = take(8 * L.cap);
  L.need = take(4 * nf);
  L.needk = take(nf);
  L.needhf = take(4 * nf);
  L.victim = take(4 * nf);
  L.vscratch = take(4 * (2 * L.cap + 2048));   // wide victim scan: candidates per tile
  L.vpass = take(16 * (nf / 128 + L.max_tiles + 2));   // wide victim apply: work table
  L.vframe = take(4 * nf);
  L.vhf = take(4 * nf);
  L.vkind = take(nf);
  L.d2h_frame = take(4 * nf);
  L.d2h_hf = take(4 * nf);
  L.tile_status = take(8 * L.max_tiles);
  L.tile_cnt = take(32 * L.max_tiles);
  L.tags = take(8 * nb * ppc);   // content tags: per page
  L.ctl = take(sizeof(Ctl));
  L.hchunks = take(8ull * c->n_host_chunks);
  L.stage = take(L.stage_bytes);
  L.xitems = take(sizeof(XItem) * nf);
  // K4-CE: groups of ce_group items alternate between two copy streams; fused swaps
  // bounce the victim's bytes through HBM (one slot per item per stream)
  L.ce_group = std::max<uint64_t>(1, std::min<uint64_t>(1024, (64ull << 20) / c->block_bytes));
  L.bounce_bytes = 2 * L.ce_group * c->block_bytes;
  L.bounce = take(L.bounce_bytes);
  const uint64_t nw = (nb + 31) / 32;
  L.obits = take(4 * nw);
  L.wbits = take(4 * nw);
  L.dlo = take(4 * nb);
  L.dpre = take(4 * (nb + 1));
  L.dw = take(nb);
  L.d2h_dmask = take(4 * nf);
  if (ppc > 1) {
    L.pdead = take(4 * nb);
    L.plazy = take(4 * nb);
    L.phz = take(4 * nb);
  }
  L.total = o;
  return L;
}

// Pinned host staging ring for interval lists, with events guarding in-flight copies.
struct Stager {
  uint8_t* host = nullptr;
  uint8_t* dev = nullptr;
  uint64_t cap = 0, pos = 0;
  struct Fly { uint64_t lo, hi; cudaEvent_t ev; };
  std::deque<Fly> fly;
  std::vector<cudaEvent_t> pool;

  cudaError_t init(uint8_t* d, uint64_t bytes) {
    dev = d;
    cap = bytes;
    return cudaHostAlloc((void**)&host, bytes, cudaHostAllocDefault);
  }
  void destroy() {
    for (auto& f : fly) cudaEventDestroy(f.ev);
    for (auto e : pool) cudaEventDestroy(e);
    fly.clear();
    pool.clear();
    if (host) cudaFreeHost(host);
    host = nullptr;
  }
  // Reserve [off, off+bytes) of the ring; waits for copies still reading it.
  cudaError_t reserve(uint64_t bytes, uint64_t* off) {
    bytes = (bytes + 15) & ~15ull;
    if (bytes > cap) return cudaErrorInvalidValue;
    if (pos + bytes > cap) pos = 0;
    uint64_t lo = pos, hi = pos + bytes;
    while (!fly.empty()) {
      Fly& f = fly.front();
      bool overlap = f.lo < hi && lo < f.hi;
      if (!overlap && cudaEventQuery(f.ev) != cudaSuccess) break;
      cudaError_t e = cudaEventSynchronize(f.ev);
      if (e) return e;
      pool.push_back(f.ev);
      fly.pop_front();
    }
    for (auto& f : fly)
      if (f.lo < hi && lo < f.hi) {
        cudaError_t e = cudaEventSynchronize(f.ev);
        if (e) return e;
      }
    *off = lo;
    pos = hi;
    return cudaSuccess;
  }
  // Keep [off, off+bytes) reserved until the work enqueued on stream s so far is done
  // (an application kernel on another stream still reading staged intervals, R7).
  cudaError_t fence(uint64_t off, uint64_t bytes, cudaStream_t s) {
    cudaEvent_t ev;
    cudaError_t e;
    if (pool.empty()) {
      e = cudaEventCreateWithFlags(&ev, cudaEventDisableTiming);
      if (e) return e;
    } else {
      ev = pool.back();
      pool.pop_back();
    }
    e = cudaEventRecord(ev, s);
    fly.push_back({off, off + bytes, ev});
    return e;
  }
  cudaError_t push(uint64_t off, uint64_t bytes, cudaStream_t s) {
    cudaError_t e = cudaMemcpyAsync(dev + off, host + off, bytes, cudaMemcpyHostToDevice, s);
    if (e) return e;
    cudaEvent_t ev;
    if (pool.empty()) {
      e = cudaEventCreateWithFlags(&ev, cudaEventDisableTiming);
      if (e) return e;
    } else {
      ev = pool.back();
      pool.pop_back();
    }
    e = cudaEventRecord(ev, s);
    fly.push_back({off, off + bytes, ev});
    return e;
  }
};

struct Iv {
  uint32_t lo, cnt;
  uint8_t w;
};

// Two-level touch / prefetch list item: a chunk, the pages the op covers and writes.
struct CItem {
  uint32_t c, cm, wm;
};

}  // namespace

struct um_arena {
  um_config cfg{};
  Layout L{};
  Tables T{};
  uint64_t* ring_buf[2][2] = {{nullptr, nullptr}, {nullptr, nullptr}};  // [ring][buffer]
  int ring_cur[2] = {0, 0};
  uint64_t ub[2] = {0, 0};  // upper bound of (tail - head) per ring
  // exact ring tails: rings only grow by appends (every block of a GPU sub-op or of a
  // discard range takes a slot) and compaction keeps the tail, so the host passes the
  // tail to the appending kernels instead of having them read and publish it
  uint64_t tail[2] = {0, 0};
  // upper bound of the frames held (G, GE, GL blocks): every GPU sub-op of n blocks may
  // take n more; nothing is subtracted.  While bound + n <= nframes a sub-op cannot need
  // a victim, and its victim kernels are not launched.
  uint64_t used_ub = 0;
  int npar = 0;             // parity slot of the multi-CTA classify's need counter
  // device intake result for the current op (intervals in T.dlo/dpre/dw)
  bool dev_iv = false, dev_anyw = false;
  uint32_t dev_m = 0;
  uint64_t dev_total = 0;
  std::vector<uint32_t> hpre;   // interval prefix of the current op (host copy, for tile tables)
  std::vector<MarkRec> mark;    // scratch: split records
  uint32_t B = 0, nblocks = 0, nframes = 0, nhframes = 0;
  cudaStream_t ps = nullptr;
  cudaEvent_t ev_in = nullptr, ev_out = nullptr;
  uint32_t clock = 0;
  uint64_t bump = 0;
  int64_t ops = 0, subops = 0;
  um_status sticky = UM_OK;
  std::atomic<int> busy{0};
  Stager stage;
  Ctl* hctl = nullptr;  // pinned mirror for reads
  std::vector<Iv> ivs;
  uint64_t iv_total = 0;       // blocks in ivs, and whether any interval is written
  bool iv_anyw = false;
  // sparse sorted batch, scanned once: the fault list (block | write << 31) ready to stage
  std::vector<uint32_t> flist;
  bool fl_ready = false;
  uint32_t fl_m = 0;           // the batch's merged intervals (what decides the form)
  std::vector<CItem> citems;   // two-level: the op's chunks with page masks
  uint32_t ppc = 1, P = 0;     // pages per chunk, page bytes (single level: 1, B)
  uint32_t lgB = 0, lgP = 0;   // log2 of block and page bytes (record -> block by shifts)
  bool dev_list = false;       // run_gpu_op: the sorted block list is in T.dlo (um_touch_batch_dev)
  bool host_prof = false;      // UM_HOST_PROFILE (diagnostic): host phases of a touch batch to stderr
  // UM_F_TIMING: event pairs around planning / transfer launches
  struct Span { cudaEvent_t a, b; int xfer; uint32_t seq; };
  std::vector<Span> spans;
  std::vector<cudaEvent_t> evpool;
  double ms_plan = 0, ms_xfer = 0;
  uint64_t n_xfer = 0, n_launch = 0;
  // K4-CE path
  cudaStream_t cs[2] = {nullptr, nullptr};
  cudaEvent_t ev_cs[2] = {nullptr, nullptr};
  XItem* hitems = nullptr;              // pinned mirror of xitems (written by k_plan_commit)
  uint32_t* hflag = nullptr;            // pinned {seq, n_need} published by k_plan_commit
  uint32_t* hd2h = nullptr;             // pinned mirror of d2h_frame / d2h_hf
  std::vector<char*> hhost;             // host chunk pointers
  char* bounce = nullptr;
  uint64_t ce_min_bytes = ~0ull;  // diagnostic auto mode (UM_CE_MIN_BYTES): sub-ops moving >= this use the copy engines
  uint64_t n_ce = 0;
  // UM_F_OVERLAP (reading R7): application kernels run on their own stream `as`; the
  // last kOverlapW GPU sub-ops form the victim-exclusion window; `pend` holds the app
  // kernels the paging stream has not waited for yet (ascending seq)
  cudaStream_t as = nullptr;
  cudaEvent_t ev_app_in = nullptr;
  // the app kernel's CTAs per SM while it overlaps paging work: its grid-stride CTAs
  // live for the whole kernel, so a full-occupancy grid would keep the paging and
  // zero-fill kernels off the SMs until it ends (UM_APP_CTAS overrides)
  int app_ctas = 1;
  bool app_serial = false;   // UM_OVERLAP_SERIAL (diagnostic): window rule, app kernel on ps
  struct WinE { uint32_t seq, n; };
  WinE win[kOverlapWMax] = {};
  int ovw = kOverlapW;      // window length (UM_OVERLAP_W overrides, 1..kOverlapWMax)
  int nwin = 0;
  struct Pend { uint32_t seq; cudaEvent_t ev; };
  std::deque<Pend> pend;
  std::vector<cudaEvent_t> apool;
};

namespace {

struct Guard {
  um_arena* a;
  bool ok;
  explicit Guard(um_arena* x) : a(x), ok(false) {
    int z = 0;
    ok = a && a->busy.compare_exchange_strong(z, 1);
  }
  ~Guard() {
    if (ok) a->busy.store(0);
  }
};

#define CK(x)                                         \
  do {                                                \
    cudaError_t e__ = (x);                            \
    if (e__ != cudaSuccess) {                         \
      a->sticky = UM_ECUDA;                           \
      if (getenv("UM_DEBUG"))                         \
        fprintf(stderr, "libum: %s at %s:%d\n", cudaGetErrorString(e__), __FILE__, __LINE__); \
      return UM_ECUDA;                                \
    }                                                 \
  } while (0)

#define ENTER(a)                           \
  Guard g__(a);                            \
  if (!a) return UM_EINVAL;                \
  if (!g__.ok) return UM_EBUSY;            \
  if (a->sticky != UM_OK) return a->sticky

static um_status hand_in(um_arena* a, void* stream) {
  cudaStream_t cs = (cudaStream_t)stream;
  if (cs != a->ps) {
    CK(cudaEventRecord(a->ev_in, cs));
    CK(cudaStreamWaitEvent(a->ps, a->ev_in, 0));
  }
  return UM_OK;
}

static um_status hand_out(um_arena* a, void* stream) {
  cudaStream_t cs = (cudaStream_t)stream;
  if (cs != a->ps) {
    CK(cudaEventRecord(a->ev_out, a->ps));
    CK(cudaStreamWaitEvent(cs, a->ev_out, 0));
  }
  return UM_OK;
}

static void set_ring_ptrs(um_arena* a) {
  a->T.used_ring = a->ring_buf[RING_USED][a->ring_cur[RING_USED]];
  a->T.disc_ring = a->ring_buf[RING_DISC][a->ring_cur[RING_DISC]];
}

static cudaEvent_t tev(um_arena* a) {
  if (!a->evpool.empty()) {
    cudaEvent_t e = a->evpool.back();
    a->evpool.pop_back();
    return e;
  }
  cudaEvent_t e = nullptr;
  cudaEventCreate(&e);
  return e;
}

// Open / close a timed span on the paging stream (no-ops without UM_F_TIMING).
static cudaEvent_t span_open(um_arena* a) {
  if (!(a->cfg.flags & UM_F_TIMING)) return nullptr;
  cudaEvent_t e = tev(a);
  cudaEventRecord(e, a->ps);
  return e;
}
static void span_close(um_arena* a, cudaEvent_t open, int xfer) {
  if (!open) return;
  cudaEvent_t e = tev(a);
  cudaEventRecord(e, a->ps);
  a->spans.push_back({open, e, xfer, a->clock});
}

// ---- UM_F_OVERLAP (reading R7) ----------------------------------------------------
static inline bool overlap_on(const um_arena* a) { return (a->cfg.flags & UM_F_OVERLAP) != 0; }

// The paging stream waits for every application kernel of a sub-op with seq < floor
// (the app stream runs them in order, so waiting for the newest of them suffices).
static um_status app_wait_below(um_arena* a, uint32_t floor) {
  cudaEvent_t last = nullptr;
  while (!a->pend.empty() && a->pend.front().seq < floor) {
    if (last) a->apool.push_back(last);
    last = a->pend.front().ev;
    a->pend.pop_front();
  }
  if (last) {
    CK(cudaStreamWaitEvent(a->ps, last, 0));
    a->apool.push_back(last);
  }
  return UM_OK;
}
static um_status app_wait_all(um_arena* a) { return app_wait_below(a, UM_NONE); }

// Victim floor of GPU sub-op `seq` with n distinct blocks: the longest suffix of the last
// kOverlapW GPU sub-ops whose block counts, added to n, stay <= nframes is protected
// (so k = need - free stays satisfiable); the floor is the seq of its oldest member, or
// seq itself when nothing is protected.  Identical to oracle.sim's window rule.
static uint32_t window_floor(um_arena* a, uint32_t seq, uint32_t n) {
  uint64_t tot = n;
  uint32_t floor = seq;
  for (int i = a->nwin - 1; i >= 0; --i) {
    if (tot + a->win[i].n > a->nframes) break;
    tot += a->win[i].n;
    floor = a->win[i].seq;
  }
  if (a->nwin == a->ovw) {
    for (int i = 1; i < a->ovw; ++i) a->win[i - 1] = a->win[i];
    a->nwin--;
  }
  a->win[a->nwin++] = {seq, n};
  return floor;
}

// K7 trigger: the host keeps an upper bound of each ring's occupancy (appends are
// bounded by the op's block count; live entries never exceed nframes).
static um_status ensure_ring_room(um_arena* a, int ring, uint64_t appends) {
  if (a->ub[ring] + appends <= a->L.cap) {
    a->ub[ring] += appends;
    return UM_OK;
  }
  int nxt = a->ring_cur[ring] ^ 1;
  cudaEvent_t sp = span_open(a);
  CK(launch_ring_compact(a->T, ring, a->ring_buf[ring][nxt], a->L.cap, a->ps));
  span_close(a, sp, 0);
  a->n_launch++;
  a->ring_cur[ring] = nxt;
  set_ring_ptrs(a);
  a->ub[ring] = std::min<uint64_t>(a->nframes, a->L.cap) + appends;
  return UM_OK;
}

// Keys live in the upper 29 bits of the packed state word, so an arena has 2^29 - 1
// sequence numbers; an op that would need more fails with UM_ENOMEM (sticky).
constexpr uint64_t kSeqLimit = (1ull << 29) - 1;
static um_status seq_room(um_arena* a, uint64_t k) {
  if ((uint64_t)a->clock + k > kSeqLimit) {
    a->sticky = UM_ENOMEM;
    return UM_ENOMEM;
  }
  return UM_OK;
}

static bool range_ok(um_arena* a, uint64_t off, uint64_t len) {
  return off <= a->cfg.arena_bytes && len <= a->cfg.arena_bytes - off;
}

// Records already in ascending, non-overlapping block order -- e.g. a fault batch sorted
// by address -- are the intervals (adjacent equal-W records merge): one linear pass with
// shifts (blocks are powers of two).  Returns false, with a->ivs unspecified, otherwise.
static bool sorted_intervals(um_arena* a, const um_access* acc, uint32_t n) {
  const uint32_t lg = a->lgB;
  auto& v = a->ivs;
  v.clear();
  v.reserve(n);
  uint64_t prev_hi = 0, total = 0;
  bool anyw = false;
  for (uint32_t i = 0; i < n; ++i) {
    if (!acc[i].len) continue;
    const uint64_t lo = acc[i].off >> lg, hi = ((acc[i].off + acc[i].len - 1) >> lg) + 1;
    const uint8_t w = (acc[i].kind & UM_ACC_WRITE) ? 1 : 0;
    total += hi - lo;
    anyw |= w != 0;
    if (!v.empty()) {
      if (lo < prev_hi) return false;
      if (prev_hi == lo && v.back().w == w) {
        v.back().cnt += (uint32_t)(hi - lo);
        prev_hi = hi;
        continue;
      }
    }
    v.push_back({(uint32_t)lo, (uint32_t)(hi - lo), w});
    prev_hi = hi;
  }
  a->iv_total = total;
  a->iv_anyw = anyw;
  return true;
}

// One pass over a batch that is already in ascending, non-overlapping block order (the
// usual shape of a large fault batch): totals, the merged-interval count, and the fault
// list itself (one u32 per block, bit 31 = write) -- no interval list is built.  Returns
// false (nothing decided) if the records are not sorted and disjoint.
static bool scan_sorted(um_arena* a, const um_access* acc, uint32_t n, bool* out_of_range) {
  const uint32_t lg = a->lgB;
  const uint64_t arena = a->cfg.arena_bytes;
  bool oor = false;
  auto& fl = a->flist;
  size_t cap = (size_t)n + 1024, k = 0;
  if (fl.size() < cap) fl.resize(cap);
  uint32_t* out = fl.data();
  uint64_t prev_hi = 0, total = 0, lim = 3ull * n;
  uint32_t m = 0, prev_w = 2;
  bool anyw = false, bad = false;
  for (uint32_t i = 0; i < n; ++i) {
    const uint64_t off = acc[i].off, len = acc[i].len;
    oor |= (off > arena) | (len > arena - off);   // the API's range check, same pass
    if (!len) continue;
    const uint64_t lo = off >> lg, hi = ((off + len - 1) >> lg) + 1, cnt = hi - lo;
    const uint32_t w = (acc[i].kind & UM_ACC_WRITE) ? 1u : 0u;
    // branch-free on the data: order violations are collected and decided after the pass
    bad |= (m != 0) & (lo < prev_hi);
    m += 1u - (uint32_t)((m != 0) & (prev_hi == lo) & (prev_w == w));
    total += cnt;
    anyw |= w != 0;
    prev_hi = hi;
    prev_w = w;
    if (total > lim) continue;   // past 3 blocks per record the list form cannot be chosen
    const uint32_t wbit = w << 31;
    if (k + cnt > cap) {
      cap = std::max<size_t>(2 * cap, k + cnt);
      fl.resize(cap);
      out = fl.data();
    }
    for (uint64_t x = 0; x < cnt; ++x) out[k++] = (uint32_t)(lo + x) | wbit;
  }
  *out_of_range = oor;
  if (bad) return false;
  a->iv_total = total;
  a->iv_anyw = anyw;
  a->fl_m = m;
  return true;
}

// Sorted disjoint intervals with constant write flag from any access records (the
// <= kIvInline-record case that is not already sorted): a 2n-event sweep.
static void build_intervals(um_arena* a, const um_access* acc, uint32_t n) {
  if (sorted_intervals(a, acc, n)) return;
  const uint32_t lg = a->lgB;
  struct Ev { uint64_t x; int dc, dw; };
  std::vector<Ev> ev;
  ev.reserve(2 * (size_t)n);
  for (uint32_t i = 0; i < n; ++i) {
    if (!acc[i].len) continue;
    uint64_t lo = acc[i].off >> lg, hi = ((acc[i].off + acc[i].len - 1) >> lg) + 1;
    int w = (acc[i].kind & UM_ACC_WRITE) ? 1 : 0;
    ev.push_back({lo, +1, w});
    ev.push_back({hi, -1, -w});
  }
  std::sort(ev.begin(), ev.end(), [](const Ev& p, const Ev& q) { return p.x < q.x; });
  a->ivs.clear();
  int cov = 0, wr = 0;
  for (size_t i = 0; i < ev.size();) {
    uint64_t x = ev[i].x;
    while (i < ev.size() && ev[i].x == x) {
      cov += ev[i].dc;
      wr += ev[i].dw;
      ++i;
    }
    if (i < ev.size() && cov > 0) {
      uint64_t nx = ev[i].x;
      uint8_t w = wr > 0;
      if (!a->ivs.empty() && (uint64_t)a->ivs.back().lo + a->ivs.back().cnt == x && a->ivs.back().w == w)
        a->ivs.back().cnt += (uint32_t)(nx - x);
      else
        a->ivs.push_back({(uint32_t)x, (uint32_t)(nx - x), w});
    }
  }
  a->iv_total = 0;
  a->iv_anyw = false;
  for (const Iv& x : a->ivs) {
    a->iv_total += x.cnt;
    a->iv_anyw |= x.w != 0;
  }
}

// The TMA kernel (K4) is the transfer engine; the copy engines (K4-CE) are the
// comparison arm, selected with UM_F_COPY_CE (or, for A/B runs only, for sub-ops of at
// least UM_CE_MIN_BYTES).
static bool use_ce(um_arena* a, uint64_t n) {
  if (a->ppc > 1) return false;   // two-level: page-granular transfers run in K4 only
  if (a->cfg.flags & UM_F_COPY_CE) return true;
  if (a->cfg.flags & UM_F_COPY_KERNEL) return false;
  return n * a->B >= a->ce_min_bytes;
}

static inline char* hframe_ptr(um_arena* a, uint32_t h) {
  return a->hhost[h / a->T.hpc] + (size_t)(h % a->T.hpc) * a->B;
}
static inline char* frame_ptr(um_arena* a, uint32_t f) { return a->T.frames + (size_t)f * a->B; }

// A copy list with run coalescing (adjacent items whose source and destination are
// both contiguous AND inside the same host chunk allocation become one copy — a copy
// may not span two pinned allocations even if they happen to be adjacent), issued as
// one copy call per run.
struct CopyList {
  std::vector<void*> dst, src;
  std::vector<size_t> size;
  std::vector<uint32_t> seg;
  void clear() { dst.clear(); src.clear(); size.clear(); seg.clear(); }
  void add(void* d, const void* s_, size_t n, uint32_t chunk) {
    if (!dst.empty() && seg.back() == chunk && (char*)dst.back() + size.back() == (char*)d &&
        (const char*)src.back() + size.back() == (const char*)s_) {
      size.back() += n;
      return;
    }
    dst.push_back(d);
    src.push_back(const_cast<void*>(s_));
    size.push_back(n);
    seg.push_back(chunk);
  }
  // one cudaMemcpyAsync per coalesced run (the copy engines take 2 MiB+ runs at link rate)
  cudaError_t issue(cudaStream_t st) {
    for (size_t i = 0; i < dst.size(); ++i) {
      cudaError_t e = cudaMemcpyAsync(dst[i], src[i], size[i], cudaMemcpyDefault, st);
      if (e) return e;
    }
    return cudaSuccess;
  }
};

// K4-CE: the plan is on the device (K1-K3 + K6 in k_plan_commit); one host sync reads
// it, then groups of items alternate between two copy-engine streams:
//   D2D victim->bounce (fused swaps) ; D2H write-backs ; H2D migrations ; zero-fill
//   kernel ; D2H bounce->host (fused swaps).
// Stream order gives every frame its write-after-read order; alternating streams keep
// both PCIe directions busy.  The paging stream waits for both copy streams.
// Spin until k_plan_commit of sub-op `seq` has published its plan in mapped host memory
// (no stream sync, no read-back copies).  Bounded: if the paging stream reports an error,
// or goes idle without the flag, the op fails with UM_ECUDA instead of hanging.
static um_status wait_plan(um_arena* a, uint32_t seq) {
  volatile uint32_t* f = a->hflag;
  for (uint64_t it = 1;; ++it) {
    if (f[0] == seq) break;
    if ((it & 255) == 0) {
      const cudaError_t q = cudaStreamQuery(a->ps);
      if (q == cudaSuccess) {
        if (f[0] == seq) break;
        a->sticky = UM_ECUDA;
        return UM_ECUDA;
      }
      if (q != cudaErrorNotReady) CK(q);
    }
  }
  std::atomic_thread_fence(std::memory_order_acquire);
  return UM_OK;
}

static um_status ce_subop(um_arena* a, uint32_t seq, uint32_t n) {
  CK(launch_plan_commit(a->T, seq, n, a->ps));
  a->n_launch++;
  um_status ws = wait_plan(a, seq);
  if (ws) return ws;
  const uint32_t nn = std::min<uint32_t>((uint32_t)((volatile uint32_t*)a->hflag)[1], n);
  const uint64_t G = a->L.ce_group, B = a->B;
  CopyList d2d, wb, h2d, sw;
  // consecutive groups of zero-fill items only (no copy to order against) share one
  // zero kernel instead of one launch per group
  uint32_t zr0 = 0, zr1 = 0;
  cudaStream_t zst = a->cs[0];
  auto flush_zero = [&]() -> cudaError_t {
    if (zr1 <= zr0) return cudaSuccess;
    cudaError_t e = launch_zero_items(a->T, zr0, zr1, zst);
    a->n_launch++;
    zr0 = zr1 = 0;
    return e;
  };
  for (uint32_t g0 = 0, gi = 0; g0 < nn; g0 += (uint32_t)G, ++gi) {
    const uint32_t g1 = (uint32_t)std::min<uint64_t>(nn, g0 + G);
    cudaStream_t st = a->cs[gi & 1];
    char* bnc = a->bounce + (gi & 1) * G * B;
    bool pure = true;
    for (uint32_t i = g0; i < g1 && pure; ++i) pure = a->hitems[i].flags == XI_ZF;
    if (pure) {
      if (zr1 != g0 || zr1 <= zr0) {
        CK(flush_zero());
        zr0 = g0;
        zst = st;
      }
      zr1 = g1;
      continue;
    }
    CK(flush_zero());
    d2d.clear(); wb.clear(); h2d.clear(); sw.clear();
    bool anyzf = false;
    uint32_t k = 0;
    for (uint32_t i = g0; i < g1; ++i) {
      const XItem& x = a->hitems[i];
      char* fr = frame_ptr(a, x.fr);
      if (x.flags & XI_SWAP) {
        d2d.add(bnc + (size_t)k * B, fr, B, UM_NONE);
        sw.add(hframe_ptr(a, x.dst_hf), bnc + (size_t)k * B, B, x.dst_hf / a->T.hpc);
        ++k;
      } else if (x.flags & XI_D2H) {
        wb.add(hframe_ptr(a, x.dst_hf), fr, B, x.dst_hf / a->T.hpc);
      }
      if (x.flags & XI_H2D) h2d.add(fr, hframe_ptr(a, x.src_hf), B, x.src_hf / a->T.hpc);
      anyzf |= (x.flags & XI_ZF) != 0;
    }
    CK(d2d.issue(st));
    CK(wb.issue(st));
    CK(h2d.issue(st));
    if (anyzf) {
      CK(launch_zero_items(a->T, g0, g1, st));
      a->n_launch++;
    }
    CK(sw.issue(st));
  }
  CK(flush_zero());
  for (int i = 0; i < 2; ++i) {
    CK(cudaEventRecord(a->ev_cs[i], a->cs[i]));
    CK(cudaStreamWaitEvent(a->ps, a->ev_cs[i], 0));
  }
  a->n_ce++;
  return UM_OK;
}

// D2H-only list (prefetch HOST, evict) through the copy engines.
static um_status ce_d2h_only(um_arena* a, uint32_t nmax) {
  CK(cudaMemcpyAsync(a->hctl, a->T.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, a->ps));
  CK(cudaMemcpyAsync(a->hd2h, a->T.d2h_frame, 4ull * nmax, cudaMemcpyDeviceToHost, a->ps));
  CK(cudaMemcpyAsync(a->hd2h + a->nframes, a->T.d2h_hf, 4ull * nmax, cudaMemcpyDeviceToHost, a->ps));
  CK(cudaMemsetAsync(&a->T.ctl->n_d2h, 0, sizeof(unsigned int), a->ps));
  CK(cudaStreamSynchronize(a->ps));
  const uint32_t nd = std::min<uint32_t>(a->hctl->n_d2h, nmax);
  CopyList wb;
  for (uint32_t i = 0; i < nd; ++i)
    if (a->hd2h[a->nframes + i] != UM_NONE)
      wb.add(hframe_ptr(a, a->hd2h[a->nframes + i]), frame_ptr(a, a->hd2h[i]), a->B, a->hd2h[a->nframes + i] / a->T.hpc);
  CK(wb.issue(a->cs[0]));
  CK(cudaEventRecord(a->ev_cs[0], a->cs[0]));
  CK(cudaStreamWaitEvent(a->ps, a->ev_cs[0], 0));
  a->n_ce++;
  return UM_OK;
}

// Device intake: dedupe a batch of accesses on the GPU.  The host converts
// each record to blocks and splits it into pieces of <= kMarkMaxBlocks (argument
// marshalling), stages the pieces, and the kernels build the sorted disjoint interval
// list in HBM.  One sync reads the interval count and the prefix array back: the host
// needs them to number the sub-ops and index tiles, not to compute anything.
static um_status device_intake(um_arena* a, const um_access* acc, uint32_t n) {
  const uint32_t lg = a->lgB;
  uint64_t bmin = ~0ull, bmax = 0;
  bool anyw = false;
  auto& mk = a->mark;
  mk.clear();
  for (uint32_t i = 0; i < n; ++i) {
    if (!acc[i].len) continue;
    const uint64_t lo = acc[i].off >> lg, hi = ((acc[i].off + acc[i].len - 1) >> lg) + 1;
    const uint32_t w = (acc[i].kind & UM_ACC_WRITE) ? 1u : 0u;
    anyw |= w != 0;
    bmin = std::min(bmin, lo);
    bmax = std::max(bmax, hi);
    for (uint64_t x = lo; x < hi; x += kMarkMaxBlocks)
      mk.push_back({(uint32_t)x, (uint32_t)std::min<uint64_t>(kMarkMaxBlocks, hi - x), w, 0u});
  }
  if (mk.empty()) {
    a->dev_iv = true;
    a->dev_m = 0;
    a->dev_total = 0;
    a->dev_anyw = false;
    a->hpre.assign(1, 0u);
    return UM_OK;
  }
  const uint64_t per = std::max<uint64_t>(1, (a->L.stage_bytes / 2) / sizeof(MarkRec));
  for (size_t c0 = 0; c0 < mk.size(); c0 += per) {
    const size_t cn = std::min<size_t>(per, mk.size() - c0);
    uint64_t off;
    CK(a->stage.reserve(cn * sizeof(MarkRec), &off));
    memcpy(a->stage.host + off, mk.data() + c0, cn * sizeof(MarkRec));
    CK(a->stage.push(off, (cn * sizeof(MarkRec) + 15) & ~15ull, a->ps));
    CK(launch_mark(a->T, (const MarkRec*)(a->stage.dev + off), (uint32_t)cn, a->ps));
  }
  const uint32_t w0 = (uint32_t)(bmin >> 5), w1 = (uint32_t)((bmax + 31) >> 5);
  CK(launch_runs(a->T, w0, w1, a->ps));
  CK(launch_intake_clear(a->T, w0, w1, a->ps));
  a->n_launch += 2 + (mk.size() + per - 1) / per;
  CK(cudaMemcpyAsync(a->hctl, a->T.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, a->ps));
  CK(cudaStreamSynchronize(a->ps));
  const uint32_t m = a->hctl->iv_m;
  a->hpre.resize((size_t)m + 1);
  CK(cudaMemcpyAsync(a->hpre.data(), a->T.dpre, 4ull * (m + 1), cudaMemcpyDeviceToHost, a->ps));
  CK(cudaStreamSynchronize(a->ps));
  a->dev_iv = true;
  a->dev_m = m;
  a->dev_total = a->hctl->iv_d;
  a->dev_anyw = anyw;
  return UM_OK;
}

// Evict mode of K3 (k = want - free on the device, clamped to the candidates: blocks
// with pin >= T.pfloor are skipped), then the D2H-only list through the engine.  Used by
// um_evict (R4) and by the proactive eviction after a GPU sub-op (R12).
static um_status evict_enqueue(um_arena* a, uint32_t seq, uint32_t want) {
  cudaEvent_t sp = span_open(a);
  if (want > kVictWideMin)
    CK(launch_victims_wide(a->T, seq, 1, want, std::min<uint64_t>(a->ub[RING_DISC] + a->ub[RING_USED], 2 * a->L.cap),
                           want, a->npar, a->ps));
  else
    CK(launch_victims(a->T, seq, 1, want, a->npar, a->ps));
  a->n_launch += want > kVictWideMin ? 1 : 0;
  span_close(a, sp, 0);
  sp = span_open(a);
  if (use_ce(a, want)) {
    um_status s = ce_d2h_only(a, want);
    if (s) return s;
  } else {
    CK(launch_service(a->T, SVC_D2H_ONLY, seq, want, a->ps));
  }
  span_close(a, sp, 1);
  a->n_launch += 2;
  a->n_xfer++;
  return UM_OK;
}

// R12 proactive eviction after GPU sub-op `seq` (n >= 1 blocks): keep reserve_blocks
// frames free, best effort.  Protected: the sub-op's blocks (pin == seq) and, with
// UM_F_OVERLAP, every block of the window (the last ovw GPU sub-ops, this one included:
// their application kernels may still run), i.e. pin >= the oldest member's seq; older
// application kernels finish first (they wrote frames that may now be written back).
static um_status evict_ahead(um_arena* a, uint32_t seq) {
  const uint32_t R = a->cfg.reserve_blocks;
  if (!R) return UM_OK;
  uint32_t floor = seq;
  if (overlap_on(a)) {
    floor = a->nwin ? a->win[0].seq : seq;
    um_status st = app_wait_below(a, floor);
    if (st) return st;
  }
  a->T.pfloor = floor;
  return evict_enqueue(a, seq, R);
}

// Enqueue the K1/K2 -> K3 -> K4/K5/K6 (-> K9) chain for every sub-op of a GPU op.
static um_status run_gpu_op(um_arena* a, int touch) {
  uint64_t total = 0;
  bool anyw = false;
  const bool dev = a->dev_iv, devl = a->dev_list;
  a->dev_iv = false;
  a->dev_list = false;
  if (dev || devl) {
    total = a->dev_total;
    anyw = a->dev_anyw;
  } else {
    total = a->iv_total;   // from the interval builder (hpre is made below only if needed)
    anyw = a->iv_anyw;
  }
  {
    um_status sr = seq_room(a, total ? (total + a->nframes - 1) / a->nframes : 1);
    if (sr) return sr;
  }
  a->ops++;
  if (total == 0) {
    a->clock++;
    a->subops++;
    if (overlap_on(a)) window_floor(a, a->clock, 0);
    return UM_OK;
  }
  const bool fl = a->fl_ready;
  a->fl_ready = false;
  const uint32_t m = dev ? a->dev_m : (fl ? a->fl_m : (devl ? 0u : (uint32_t)a->ivs.size()));
  uint64_t iv_off = 0, iv_bytes = 0;   // staged interval arrays (read by the app kernels)
  OpIv iv{};
  iv.m = m;
  if (fl) {
    // sparse sorted batch: the fault list made while scanning the records
    const uint64_t bytes = 4ull * total;
    uint64_t off;
    CK(a->stage.reserve(bytes, &off));
    iv_off = off;
    iv_bytes = (bytes + 15) & ~15ull;
    memcpy(a->stage.host + off, a->flist.data(), bytes);   // flist holds exactly `total` entries
    CK(a->stage.push(off, iv_bytes, a->ps));
    iv.blist = (const uint32_t*)(a->stage.dev + off);
  } else if (devl) {
    // the distinct block list made on the device from device-resident records (HBM)
    iv.blist = a->T.dlo;
  } else if (dev) {
    // intervals made on the device by the intake kernels (already in HBM)
    iv.lo = a->T.dlo;
    iv.pre = a->T.dpre;
    iv.wflag = a->T.dw;
  } else if (m <= kIvInline) {
    // small list: pass it inline in the kernel parameters (no staging copy)
    iv.inl = 1;
    uint32_t acc = 0;
    for (uint32_t j = 0; j < m; ++j) {
      iv.ilo[j] = a->ivs[j].lo;
      iv.ipre[j] = acc;
      iv.iw[j] = a->ivs[j].w;
      acc += a->ivs[j].cnt;
    }
    iv.ipre[m] = acc;
  } else if (total <= 3ull * m && 4ull * total <= a->L.stage_bytes / 2) {
    // sparse batch (intervals average <= 3 blocks, e.g. a fault buffer of scattered
    // pages): stage the distinct blocks themselves, bit 31 = write (argument marshalling;
    // <= 12 B per interval against 9 B + the tile table, and the kernels then need no
    // interval lookup)
    const uint64_t bytes = 4ull * total;
    uint64_t off;
    CK(a->stage.reserve(bytes, &off));
    iv_off = off;
    iv_bytes = (bytes + 15) & ~15ull;
    uint32_t* hb = (uint32_t*)(a->stage.host + off);
    uint64_t g = 0;
    for (uint32_t j = 0; j < m; ++j) {
      const uint32_t wbit = a->ivs[j].w ? 0x80000000u : 0u;
      for (uint32_t x = 0; x < a->ivs[j].cnt; ++x) hb[g++] = (a->ivs[j].lo + x) | wbit;
    }
    CK(a->stage.push(off, iv_bytes, a->ps));
    iv.blist = (const uint32_t*)(a->stage.dev + off);
  } else {
    // stage lo[m], pre[m+1], w[m] through the pinned ring
    const uint64_t bytes_lo = 4ull * m, bytes_pre = 4ull * (m + 1), bytes_w = m;
    const uint64_t o_lo = 0, o_pre = (bytes_lo + 15) & ~15ull, o_w = o_pre + ((bytes_pre + 15) & ~15ull);
    const uint64_t bytes = o_w + bytes_w;
    uint64_t off;
    CK(a->stage.reserve(bytes, &off));
    iv_off = off;
    iv_bytes = (bytes + 15) & ~15ull;
    uint32_t* hlo = (uint32_t*)(a->stage.host + off + o_lo);
    uint32_t* hpre = (uint32_t*)(a->stage.host + off + o_pre);
    uint8_t* hw = a->stage.host + off + o_w;
    uint32_t acc = 0;
    a->hpre.resize((size_t)m + 1);   // host copy for the per-tile interval index below
    for (uint32_t j = 0; j < m; ++j) {
      hlo[j] = a->ivs[j].lo;
      hpre[j] = acc;
      a->hpre[j] = acc;
      hw[j] = a->ivs[j].w;
      acc += a->ivs[j].cnt;
    }
    hpre[m] = acc;
    a->hpre[m] = acc;
    CK(a->stage.push(off, (bytes + 15) & ~15ull, a->ps));
    iv.lo = (const uint32_t*)(a->stage.dev + off + o_lo);
    iv.pre = (const uint32_t*)(a->stage.dev + off + o_pre);
    iv.wflag = a->stage.dev + off + o_w;
  }
  const uint32_t F = a->nframes;
  uint32_t jcur = 0;   // interval holding the current item (items ascend across sub-ops)
  const uint32_t* hp = a->hpre.data();
  for (uint64_t g0 = 0; g0 < total; g0 += F) {
    const uint32_t n = (uint32_t)std::min<uint64_t>(F, total - g0);
    const uint32_t seq = ++a->clock;
    a->subops++;
    um_status st = ensure_ring_room(a, RING_USED, n);
    if (st) return st;
    if (overlap_on(a)) {
      a->T.pfloor = window_floor(a, seq, n);
      st = app_wait_below(a, a->T.pfloor);   // app kernels outside the window finish first
      if (st) return st;
    } else {
      a->T.pfloor = seq;
    }
    uint64_t tj_off = 0, tj_bytes = 0;
    if (!iv.inl && !iv.blist) {
      // per tile of this sub-op, the interval slice its items fall in: an index the
      // kernels would otherwise find by a dependent binary search over the staged list
      const uint32_t tile = n <= kSmallPlan ? kSmallPlan : classify_tile();
      const uint32_t nt = (n + tile - 1) / tile;
      uint64_t off;
      CK(a->stage.reserve(8ull * nt, &off));
      tj_off = off;
      tj_bytes = (8ull * nt + 15) & ~15ull;
      uint32_t* tj = (uint32_t*)(a->stage.host + off);
      auto seek = [&](uint64_t g) {
        while (hp[jcur + 1] <= g) ++jcur;
        return jcur;
      };
      for (uint32_t t = 0; t < nt; ++t) {
        tj[2 * t] = seek(g0 + (uint64_t)t * tile);
        tj[2 * t + 1] = seek(g0 + std::min<uint64_t>(n, (uint64_t)(t + 1) * tile) - 1);
      }
      CK(a->stage.push(off, 8ull * nt, a->ps));
      iv.tj = (const uint32_t*)(a->stage.dev + off);
    }
    cudaEvent_t sp = span_open(a);
    const uint64_t tail0 = a->tail[RING_USED];
    a->tail[RING_USED] += n;
    const uint64_t used_before = a->used_ub;
    a->used_ub = std::min<uint64_t>(a->nframes, a->used_ub + n);
    if (n <= kSmallPlan) {
      CK(launch_plan_small(a->T, iv, (uint32_t)g0, n, seq, touch, tail0, a->ps));
      a->n_launch += 1;
    } else {
      const int k0 = used_before + n <= a->nframes;   // no victim possible: skip the victim kernels
      CK(launch_classify(a->T, iv, (uint32_t)g0, n, seq, touch, tail0, a->npar, k0, a->ps));
      if (!k0) {
        if (n > kVictWideMin)
          CK(launch_victims_wide(a->T, seq, 0, 0, std::min<uint64_t>(a->ub[RING_DISC] + a->ub[RING_USED], 2 * a->L.cap),
                                 n, a->npar, a->ps));
        else
          CK(launch_victims(a->T, seq, 0, 0, a->npar, a->ps));
      }
      a->npar ^= 1;
      a->n_launch += k0 ? 1 : (n > kVictWideMin ? 3 : 2);
    }
    span_close(a, sp, 0);
    if (use_ce(a, n)) {
      sp = span_open(a);
      um_status st = ce_subop(a, seq, n);   // counts its own launches
      if (st) return st;
      span_close(a, sp, 1);
    } else {
      sp = span_open(a);
      CK(launch_service(a->T, SVC_SUBOP, seq, n, a->ps));
      span_close(a, sp, 1);
      a->n_launch += 1;
    }
    a->n_xfer++;
    if (touch && anyw && (a->cfg.flags & UM_F_APP_STAMP)) {
      if (overlap_on(a) && !a->app_serial) {
        // R7: the application kernel runs on its own stream after this sub-op's
        // transfers and overlaps the next sub-ops' planning and transfers
        CK(cudaEventRecord(a->ev_app_in, a->ps));
        CK(cudaStreamWaitEvent(a->as, a->ev_app_in, 0));
        CK(launch_app_stamp(a->T, iv, (uint32_t)g0, n, seq, a->app_ctas, a->as));
        cudaEvent_t e;
        if (a->apool.empty()) {
          CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
        } else {
          e = a->apool.back();
          a->apool.pop_back();
        }
        CK(cudaEventRecord(e, a->as));
        a->pend.push_back({seq, e});
        if (iv_bytes) CK(a->stage.fence(iv_off, iv_bytes, a->as));
        if (tj_bytes) CK(a->stage.fence(tj_off, tj_bytes, a->as));
      } else {
        CK(launch_app_stamp(a->T, iv, (uint32_t)g0, n, seq, 8, a->ps));
      }
      a->n_launch++;
    }
    um_status ea = evict_ahead(a, seq);
    if (ea) return ea;
  }
  return UM_OK;
}

// ---- two-level granularity ------------------------------------------
// Pages [p0, p1) (global page indices) of chunk c as the chunk's page mask.
static uint32_t chunk_mask(const um_arena* a, uint64_t c, uint64_t p0, uint64_t p1) {
  const uint64_t c0 = c * a->ppc;
  const uint32_t lo = p0 > c0 ? (uint32_t)(p0 - c0) : 0u;
  const uint32_t hi = p1 < c0 + a->ppc ? (uint32_t)(p1 - c0) : a->ppc;
  return (hi >= 32 ? 0xffffffffu : ((1u << hi) - 1u)) & ~((1u << lo) - 1u);
}

// Append the chunks overlapping byte range [off, off+len) with their page masks.
static void add_range(um_arena* a, uint64_t off, uint64_t len, bool w) {
  if (!len) return;
  const uint64_t p0 = off >> a->lgP, p1 = ((off + len - 1) >> a->lgP) + 1;
  for (uint64_t c = p0 / a->ppc; c <= (p1 - 1) / a->ppc; ++c) {
    const uint32_t m = chunk_mask(a, c, p0, p1);
    a->citems.push_back({(uint32_t)c, m, w ? m : 0u});
  }
}

// Sort by chunk and merge duplicates (argument marshalling: which pages the op names).
static void finish_citems(um_arena* a) {
  auto& v = a->citems;
  std::sort(v.begin(), v.end(), [](const CItem& x, const CItem& y) { return x.c < y.c; });
  size_t k = 0;
  for (size_t i = 0; i < v.size(); ++i) {
    if (k && v[k - 1].c == v[i].c) {
      v[k - 1].cm |= v[i].cm;
      v[k - 1].wm |= v[i].wm;
    } else {
      v[k++] = v[i];
    }
  }
  v.resize(k);
}

// Two-level GPU-destination op over a->citems: the chunk-level chain of run_gpu_op in the
// list form (classify / victims unchanged), the page-aware transfer kernel, then the page
// revive of the op's cover masks, then the application kernel on the written pages.
static um_status run_gpu_op2(um_arena* a, int touch) {
  const uint64_t total = a->citems.size();
  bool anyw = false;
  for (const CItem& x : a->citems) anyw |= x.wm != 0;
  {
    um_status sr = seq_room(a, total ? (total + a->nframes - 1) / a->nframes : 1);
    if (sr) return sr;
  }
  a->ops++;
  if (total == 0) {
    a->clock++;
    a->subops++;
    return UM_OK;
  }
  const uint64_t arr = (4 * total + 15) & ~15ull;
  uint64_t off;
  CK(a->stage.reserve(3 * arr, &off));
  uint32_t* hb = (uint32_t*)(a->stage.host + off);
  uint32_t* hc = (uint32_t*)(a->stage.host + off + arr);
  uint32_t* hw = (uint32_t*)(a->stage.host + off + 2 * arr);
  for (uint64_t g = 0; g < total; ++g) {
    const CItem& x = a->citems[g];
    hb[g] = x.c | (x.wm ? 0x80000000u : 0u);
    hc[g] = x.cm;
    hw[g] = x.wm;
  }
  CK(a->stage.push(off, 3 * arr, a->ps));
  OpIv iv{};
  iv.m = (uint32_t)total;
  iv.blist = (const uint32_t*)(a->stage.dev + off);
  iv.pcov = (const uint32_t*)(a->stage.dev + off + arr);
  iv.pw = (const uint32_t*)(a->stage.dev + off + 2 * arr);
  const uint32_t F = a->nframes;
  for (uint64_t g0 = 0; g0 < total; g0 += F) {
    const uint32_t n = (uint32_t)std::min<uint64_t>(F, total - g0);
    const uint32_t seq = ++a->clock;
    a->subops++;
    um_status st = ensure_ring_room(a, RING_USED, n);
    if (st) return st;
    a->T.pfloor = seq;
    cudaEvent_t sp = span_open(a);
    const uint64_t tail0 = a->tail[RING_USED];
    a->tail[RING_USED] += n;
    const uint64_t used_before = a->used_ub;
    a->used_ub = std::min<uint64_t>(a->nframes, a->used_ub + n);
    if (n <= kSmallPlan) {
      CK(launch_plan_small(a->T, iv, (uint32_t)g0, n, seq, touch, tail0, a->ps));
      a->n_launch += 1;
    } else {
      const int k0 = used_before + n <= a->nframes;   // no victim possible: skip the victim kernels
      CK(launch_classify(a->T, iv, (uint32_t)g0, n, seq, touch, tail0, a->npar, k0, a->ps));
      if (!k0) {
        if (n > kVictWideMin)
          CK(launch_victims_wide(a->T, seq, 0, 0, std::min<uint64_t>(a->ub[RING_DISC] + a->ub[RING_USED], 2 * a->L.cap),
                                 n, a->npar, a->ps));
        else
          CK(launch_victims(a->T, seq, 0, 0, a->npar, a->ps));
      }
      a->npar ^= 1;
      a->n_launch += k0 ? 1 : (n > kVictWideMin ? 3 : 2);
    }
    span_close(a, sp, 0);
    sp = span_open(a);
    CK(launch_service(a->T, SVC_SUBOP, seq, n, a->ps));
    span_close(a, sp, 1);
    if (touch) {   // a touch revives the pages of each sub-op once it is serviced
      CK(launch_page_revive(a->T, iv, (uint32_t)g0, n, 1, a->ps));
      a->n_launch++;
    }
    a->n_launch++;
    a->n_xfer++;
    if (touch && anyw && (a->cfg.flags & UM_F_APP_STAMP)) {
      CK(launch_app_stamp(a->T, iv, (uint32_t)g0, n, seq, 8, a->ps));
      a->n_launch++;
    }
  }
  if (!touch) {   // a prefetch revalidates its pages when the whole op is done (oracle.chunks)
    CK(launch_page_revive(a->T, iv, 0, (uint32_t)total, 0, a->ps));
    a->n_launch++;
  }
  return UM_OK;
}

}  // namespace

// =====================================================================================
// C ABI
// =====================================================================================
UM_API const char* um_strerror(um_status s) {
  switch (s) {
    case UM_OK: return "ok";
    case UM_EINVAL: return "invalid argument";
    case UM_ENOMEM: return "out of memory (arena or host-frame pool)";
    case UM_ECUDA: return "CUDA error";
    case UM_EBUSY: return "arena busy (concurrent call)";
  }
  return "unknown";
}

UM_API um_status um_workspace_size(const um_config* cfg, uint64_t* bytes) {
  if (check_cfg(cfg) || !bytes) return UM_EINVAL;
  *bytes = make_layout(cfg).total;
  return UM_OK;
}

UM_API um_status um_arena_create(const um_config* cfg, um_arena** out) {
  if (check_cfg(cfg) || !out || !cfg->frames || !cfg->workspace || !cfg->host_chunks) return UM_EINVAL;
  Layout L = make_layout(cfg);
  if (cfg->workspace_bytes < L.total) return UM_EINVAL;
  if ((cfg->flags & UM_F_COPY_CE) && (cfg->flags & UM_F_COPY_KERNEL)) return UM_EINVAL;
  um_arena* a = new (std::nothrow) um_arena();
  if (!a) return UM_ENOMEM;
  a->cfg = *cfg;
  a->L = L;
  a->B = cfg->block_bytes;
  a->nblocks = (uint32_t)(cfg->arena_bytes / cfg->block_bytes);
  a->nframes = (uint32_t)(cfg->budget_bytes / cfg->block_bytes);
  const uint32_t hpc = (uint32_t)(cfg->host_chunk_bytes / cfg->block_bytes);
  a->nhframes = cfg->n_host_chunks * hpc;
  auto fail = [&](cudaError_t e) {
    if (getenv("UM_DEBUG")) fprintf(stderr, "libum create: %s\n", cudaGetErrorString(e));
    a->stage.destroy();
    delete a;
    return UM_ECUDA;
  };
  cudaError_t e;
  if ((e = cudaSetDevice(cfg->device))) return fail(e);
  if ((e = setup_kernels())) return fail(e);
  char* ws = (char*)cfg->workspace;
  Tables& T = a->T;
  T.sk = (uint32_t*)(ws + L.sk);
  T.frame_of = (uint32_t*)(ws + L.frame_of);
  T.map = (uint32_t*)(ws + L.map);
  T.hframe = (uint32_t*)(ws + L.hframe);
  T.pin = (uint32_t*)(ws + L.pin);
  T.free_stack = (uint32_t*)(ws + L.free_stack);
  T.hfree_stack = (uint32_t*)(ws + L.hfree_stack);
  for (int i = 0; i < 2; ++i) {
    a->ring_buf[RING_USED][i] = (uint64_t*)(ws + L.used[i]);
    a->ring_buf[RING_DISC][i] = (uint64_t*)(ws + L.disc[i]);
  }
  T.cap_mask = L.cap - 1;
  T.need = (uint32_t*)(ws + L.need);
  T.needk = (uint8_t*)(ws + L.needk);
  T.needhf = (uint32_t*)(ws + L.needhf);
  T.victim = (uint32_t*)(ws + L.victim);
  T.vscratch = (uint32_t*)(ws + L.vscratch);
  T.vpass = (ulonglong2*)(ws + L.vpass);
  T.vframe = (uint32_t*)(ws + L.vframe);
  T.vhf = (uint32_t*)(ws + L.vhf);
  T.vkind = (uint8_t*)(ws + L.vkind);
  T.d2h_frame = (uint32_t*)(ws + L.d2h_frame);
  T.d2h_hf = (uint32_t*)(ws + L.d2h_hf);
  T.tile_status = (unsigned long long*)(ws + L.tile_status);
  T.tile_cnt = (uint32_t*)(ws + L.tile_cnt);
  T.tags = (uint64_t*)(ws + L.tags);
  T.ctl = (Ctl*)(ws + L.ctl);
  T.xitems = (XItem*)(ws + L.xitems);
  T.obits = (uint32_t*)(ws + L.obits);
  T.wbits = (uint32_t*)(ws + L.wbits);
  T.dlo = (uint32_t*)(ws + L.dlo);
  T.dpre = (uint32_t*)(ws + L.dpre);
  T.dw = (uint8_t*)(ws + L.dw);
  T.d2h_dmask = (uint32_t*)(ws + L.d2h_dmask);
  a->ppc = cfg_ppc(cfg);
  a->P = cfg->block_bytes / a->ppc;
  a->lgB = 31 - __builtin_clz(a->B);
  a->lgP = 31 - __builtin_clz(a->P);
  T.ppc = a->ppc;
  T.P = a->P;
  if (a->ppc > 1) {
    T.pdead = (uint32_t*)(ws + L.pdead);
    T.plazy = (uint32_t*)(ws + L.plazy);
    T.phz = (uint32_t*)(ws + L.phz);
  }
  a->bounce = ws + L.bounce;
  T.frames = (char*)cfg->frames;
  T.hpc = hpc;
  T.B = a->B;
  T.nblocks = a->nblocks;
  T.nframes = a->nframes;
  T.nhframes = a->nhframes;
  T.zero_hf = a->nhframes - 1;  // last host frame: the shared zero page
  set_ring_ptrs(a);
  // host chunk table (device pointers of the mapped pinned chunks)
  std::vector<char*> hc(cfg->n_host_chunks);
  for (uint32_t i = 0; i < cfg->n_host_chunks; ++i) {
    void* dp = nullptr;
    if (cudaHostGetDevicePointer(&dp, cfg->host_chunks[i], 0) != cudaSuccess) {
      cudaGetLastError();
      dp = cfg->host_chunks[i];  // UVA: the host pointer is the device pointer
    }
    hc[i] = (char*)dp;
  }
  char** dhc = (char**)(ws + L.hchunks);
  T.hchunks = dhc;
  // zero page
  {
    uint32_t z = T.zero_hf;
    memset((char*)cfg->host_chunks[z / hpc] + (size_t)(z % hpc) * a->B, 0, a->B);
  }
  // UM_F_OVERLAP: the paging and copy streams take the highest priority and the app
  // stream the lowest, so queued paging CTAs are scheduled ahead of app CTAs
  int prio_lo = 0, prio_hi = 0;
  if ((cfg->flags & UM_F_OVERLAP) && !getenv("UM_NO_PRIO")) cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi);
  if ((e = cudaStreamCreateWithPriority(&a->ps, cudaStreamNonBlocking, prio_hi))) return fail(e);
  if (cfg->flags & UM_F_OVERLAP) {
    if ((e = cudaStreamCreateWithPriority(&a->as, cudaStreamNonBlocking, prio_lo))) return fail(e);
    if ((e = cudaEventCreateWithFlags(&a->ev_app_in, cudaEventDisableTiming))) return fail(e);
    if (const char* v = getenv("UM_APP_CTAS")) a->app_ctas = std::max(1, atoi(v));
    if (const char* v = getenv("UM_APP_GRID")) a->app_ctas = -std::max(1, atoi(v));
    a->app_serial = getenv("UM_OVERLAP_SERIAL") != nullptr;
    if (const char* v = getenv("UM_OVERLAP_W")) a->ovw = std::min(kOverlapWMax, std::max(1, atoi(v)));
  }
  if ((e = cudaEventCreateWithFlags(&a->ev_in, cudaEventDisableTiming))) return fail(e);
  if ((e = cudaEventCreateWithFlags(&a->ev_out, cudaEventDisableTiming))) return fail(e);
  if ((e = cudaHostAlloc((void**)&a->hctl, sizeof(Ctl), cudaHostAllocDefault))) return fail(e);
  if ((e = cudaHostAlloc((void**)&a->hitems, sizeof(XItem) * a->nframes, cudaHostAllocMapped))) return fail(e);
  if ((e = cudaHostAlloc((void**)&a->hflag, 16, cudaHostAllocMapped))) return fail(e);
  memset(a->hflag, 0, 16);
  if ((e = cudaHostGetDevicePointer((void**)&a->T.hx, a->hitems, 0))) return fail(e);
  if ((e = cudaHostGetDevicePointer((void**)&a->T.hflag, a->hflag, 0))) return fail(e);
  if ((e = cudaHostAlloc((void**)&a->hd2h, 8ull * a->nframes, cudaHostAllocDefault))) return fail(e);
  for (int i = 0; i < 2; ++i) {
    if ((e = cudaStreamCreateWithPriority(&a->cs[i], cudaStreamNonBlocking, prio_hi))) return fail(e);
    if ((e = cudaEventCreateWithFlags(&a->ev_cs[i], cudaEventDisableTiming))) return fail(e);
  }
  for (uint32_t i = 0; i < cfg->n_host_chunks; ++i) a->hhost.push_back((char*)cfg->host_chunks[i]);
  if (const char* v = getenv("UM_CE_MIN_BYTES")) a->ce_min_bytes = strtoull(v, nullptr, 10);
  a->host_prof = getenv("UM_HOST_PROFILE") != nullptr;
  if ((e = a->stage.init((uint8_t*)(ws + L.stage), L.stage_bytes))) return fail(e);
  // zero the whole workspace once: every table, ring slot and list starts defined (the
  // parity exports copy whole rings / lists; compute-sanitizer initcheck stays clean)
  if ((e = cudaMemsetAsync(ws, 0, L.total, a->ps))) return fail(e);
  if ((e = cudaMemcpyAsync(dhc, hc.data(), 8ull * cfg->n_host_chunks, cudaMemcpyHostToDevice, a->ps))) return fail(e);
  if ((e = launch_init(T, (int)(a->nhframes - 1), a->ps))) return fail(e);
  if (cfg->flags & UM_F_CHECK)
    if ((e = launch_poison(T, a->ps))) return fail(e);
  if ((e = cudaStreamSynchronize(a->ps))) return fail(e);
  *out = a;
  return UM_OK;
}

UM_API um_status um_arena_destroy(um_arena* a) {
  if (!a) return UM_EINVAL;
  if (a->ps) cudaStreamSynchronize(a->ps);
  if (a->as) cudaStreamSynchronize(a->as);
  a->stage.destroy();
  for (auto& p : a->pend) cudaEventDestroy(p.ev);
  for (auto e : a->apool) cudaEventDestroy(e);
  if (a->ev_app_in) cudaEventDestroy(a->ev_app_in);
  if (a->as) cudaStreamDestroy(a->as);
  for (auto& sp : a->spans) { cudaEventDestroy(sp.a); cudaEventDestroy(sp.b); }
  for (auto e : a->evpool) cudaEventDestroy(e);
  if (a->hctl) cudaFreeHost(a->hctl);
  if (a->hitems) cudaFreeHost(a->hitems);
  if (a->hflag) cudaFreeHost(a->hflag);
  if (a->hd2h) cudaFreeHost(a->hd2h);
  for (int i = 0; i < 2; ++i) {
    if (a->ev_cs[i]) cudaEventDestroy(a->ev_cs[i]);
    if (a->cs[i]) cudaStreamDestroy(a->cs[i]);
  }
  if (a->ev_in) cudaEventDestroy(a->ev_in);
  if (a->ev_out) cudaEventDestroy(a->ev_out);
  if (a->ps) cudaStreamDestroy(a->ps);
  delete a;
  return UM_OK;
}

UM_API um_status um_alloc(um_arena* a, uint64_t bytes, uint64_t* off) {
  ENTER(a);
  if (!off) return UM_EINVAL;
  uint64_t r = (bytes + a->B - 1) / a->B * a->B;
  if (a->bump + r > a->cfg.arena_bytes || r < bytes) return UM_ENOMEM;
  *off = a->bump;
  a->bump += r;
  return UM_OK;
}

UM_API um_status um_touch_batch(um_arena* a, const um_access* acc, uint32_t n, void* stream) {
  ENTER(a);
  if (n && !acc) return UM_EINVAL;
  using clk = std::chrono::steady_clock;
  const auto t0 = clk::now();
  // a large single-level batch is scanned once here: range check, order check and (for a
  // sorted one) totals and the fault list; anything else is range-checked on its own
  bool scanned = false;
  if (a->ppc == 1 && n > kIvInline) {
    bool oor = false;
    scanned = scan_sorted(a, acc, n, &oor);
    if (oor) return UM_EINVAL;
  } else {
    for (uint32_t i = 0; i < n; ++i)
      if (!range_ok(a, acc[i].off, acc[i].len)) return UM_EINVAL;
  }
  const auto t1 = clk::now();
  um_status s = hand_in(a, stream);
  if (s) return s;
  if (a->ppc > 1) {   // two-level: the chunks with the pages each record covers / writes
    a->citems.clear();
    for (uint32_t i = 0; i < n; ++i) add_range(a, acc[i].off, acc[i].len, (acc[i].kind & UM_ACC_WRITE) != 0);
    finish_citems(a);
    s = run_gpu_op2(a, 1);
    if (s) return s;
    return hand_out(a, stream);
  }
  // a batch of more records than fit inline that is not already sorted and disjoint is
  // deduplicated on the device; otherwise the records (one linear pass), or the <=
  // kIvInline records after a 2n-event merge, are the intervals
  if (n > kIvInline && !scanned) {
    // the intake rewrites the device interval list that in-flight app kernels may read
    if (overlap_on(a) && (s = app_wait_all(a))) return s;
    s = device_intake(a, acc, n);
    if (s) return s;
  } else if (n > kIvInline && a->fl_m > kIvInline && a->iv_total <= 3ull * a->fl_m &&
             4ull * a->iv_total <= a->L.stage_bytes / 2) {
    a->fl_ready = true;   // sparse batch: the fault list is already made
  } else if (n > kIvInline) {
    sorted_intervals(a, acc, n);   // sorted, but the interval forms fit it better
  } else {
    build_intervals(a, acc, n);
  }
  const auto t2 = clk::now();
  s = run_gpu_op(a, 1);
  if (s) return s;
  if (a->host_prof) {
    const auto t3 = clk::now();
    auto us = [](clk::duration d) { return std::chrono::duration<double, std::micro>(d).count(); };
    fprintf(stderr, "libum touch_batch n=%u: scan %.1f us, intervals %.1f us, stage + launch %.1f us\n", n,
            us(t1 - t0), us(t2 - t1), us(t3 - t2));
  }
  return hand_out(a, stream);
}

UM_API um_status um_touch_batch_dev(um_arena* a, const um_access* acc, uint32_t n, void* stream) {
  ENTER(a);
  if ((n && !acc) || ((uintptr_t)acc & 15) || a->ppc > 1) return UM_EINVAL;
  using clk = std::chrono::steady_clock;
  const auto t0 = clk::now();
  um_status s = hand_in(a, stream);
  if (s) return s;
  // the list rewrites T.dlo, which in-flight application kernels of earlier sub-ops may
  // read (their block list)
  if (overlap_on(a) && (s = app_wait_all(a))) return s;
  cudaEvent_t sp = span_open(a);
  CK(launch_mark_acc(a->T, acc, n, a->lgB, a->ps));
  CK(launch_list(a->T, (a->nblocks + 31) / 32, a->ps));
  span_close(a, sp, 0);
  a->n_launch += (n ? 1 : 0) + 1;
  // the host needs the distinct-block count to number the sub-ops (and learns of a
  // range error before anything that changes state is enqueued)
  CK(cudaMemcpyAsync(a->hctl, a->T.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, a->ps));
  CK(cudaStreamSynchronize(a->ps));
  const auto t1 = clk::now();
  if (a->hctl->iv_err) {
    CK(cudaMemsetAsync(&a->T.ctl->iv_err, 0, sizeof(unsigned int), a->ps));
    return UM_EINVAL;
  }
  a->dev_list = true;
  a->dev_total = a->hctl->iv_d;
  a->dev_anyw = a->hctl->iv_m != 0;
  s = run_gpu_op(a, 1);
  if (s) return s;
  if (a->host_prof) {
    const auto t2 = clk::now();
    auto us = [](clk::duration d) { return std::chrono::duration<double, std::micro>(d).count(); };
    fprintf(stderr, "libum touch_batch_dev n=%u: intake + count read-back %.1f us, launch %.1f us\n", n,
            us(t1 - t0), us(t2 - t1));
  }
  return hand_out(a, stream);
}

UM_API um_status um_prefetch(um_arena* a, uint64_t off, uint64_t len, int dst, void* stream) {
  ENTER(a);
  if (!range_ok(a, off, len) || (dst != UM_DST_GPU && dst != UM_DST_HOST)) return UM_EINVAL;
  um_status s = hand_in(a, stream);
  if (s) return s;
  if (dst == UM_DST_GPU && a->ppc > 1) {
    a->citems.clear();
    add_range(a, off, len, false);
    s = run_gpu_op2(a, 0);
    if (s) return s;
  } else if (dst == UM_DST_GPU) {
    a->ivs.clear();
    a->iv_total = 0;
    a->iv_anyw = false;
    if (len) {
      uint64_t lo = off >> a->lgB, hi = ((off + len - 1) >> a->lgB) + 1;
      a->ivs.push_back({(uint32_t)lo, (uint32_t)(hi - lo), 0});
      a->iv_total = hi - lo;
    }
    s = run_gpu_op(a, 0);
    if (s) return s;
  } else {
    if ((s = seq_room(a, 1))) return s;
    // moves data and frees frames: every in-flight application kernel finishes first (R7)
    if (overlap_on(a) && (s = app_wait_all(a))) return s;
    a->ops++;
    a->subops++;
    const uint32_t seq = ++a->clock;
    if (len) {
      uint32_t lo = (uint32_t)(off / a->B), hi = (uint32_t)((off + len - 1) / a->B + 1);
      cudaEvent_t sp = span_open(a);
      CK(launch_directive(a->T, DIR_PREFETCH_HOST, lo, hi - lo, seq, 0, a->tail[RING_DISC], a->ps));
      span_close(a, sp, 0);
      const uint32_t nmax = std::min<uint32_t>(hi - lo, a->nframes);
      sp = span_open(a);
      if (use_ce(a, nmax)) {
        s = ce_d2h_only(a, nmax);
        if (s) return s;
      } else {
        CK(launch_service(a->T, SVC_D2H_ONLY, seq, nmax, a->ps));
      }
      span_close(a, sp, 1);
      a->n_launch += 2;
      a->n_xfer++;
      if (a->ppc > 1) {   // revalidate the covered pages (A17); revived dead pages read zero
        CK(launch_page_host_revive(a->T, lo, hi - lo, off / a->P, (off + len - 1) / a->P + 1, a->ps));
        a->n_launch++;
      }
    }
  }
  return hand_out(a, stream);
}

static um_status discard_common(um_arena* a, uint64_t off, uint64_t len, void* stream, int kind) {
  ENTER(a);
  if (!range_ok(a, off, len)) return UM_EINVAL;
  um_status s = hand_in(a, stream);
  if (s) return s;
  if ((s = seq_room(a, 1))) return s;
  a->ops++;
  a->subops++;
  const uint32_t seq = ++a->clock;
  const uint64_t lo = (off + a->B - 1) / a->B, hi = (off + len) / a->B;  // fully covered blocks
  if (hi > lo && !(a->cfg.flags & UM_F_DISCARD_OFF)) {
    // every block of the range takes a DISC slot (k_directive), so a range larger than
    // the ring's free space after compaction (cap - nframes live entries) is applied in
    // ascending chunks with the same seq: the ring stays sorted by (dkey, block)
    const uint64_t chunk = a->L.cap - std::min<uint64_t>(a->nframes, a->L.cap / 2);
    for (uint64_t c0 = lo; c0 < hi; c0 += chunk) {
      const uint32_t n = (uint32_t)std::min<uint64_t>(chunk, hi - c0);
      s = ensure_ring_room(a, RING_DISC, n);
      if (s) return s;
      const uint64_t tail0 = a->tail[RING_DISC];
      a->tail[RING_DISC] += n;
      cudaEvent_t sp = span_open(a);
      CK(launch_directive(a->T, kind, (uint32_t)c0, n, seq, 0, tail0, a->ps));
      span_close(a, sp, 0);
      a->n_launch++;
    }
  }
  if (a->ppc > 1 && !(a->cfg.flags & UM_F_DISCARD_OFF)) {
    // pages fully inside the range whose chunk is not (at most the two edge chunks):
    // marked dead without unmapping (§5.4)
    const uint64_t pp0 = (off + a->P - 1) / a->P, pp1 = (off + len) / a->P;
    if (pp1 > pp0) {
      uint32_t ce[2] = {UM_NONE, UM_NONE}, me[2] = {0u, 0u};
      int k = 0;
      const uint64_t cand[2] = {pp0 / a->ppc, (pp1 - 1) / a->ppc};
      for (int i = 0; i < 2; ++i) {
        const uint64_t c = cand[i];
        if ((i == 1 && c == cand[0]) || (c >= lo && c < hi)) continue;
        ce[k] = (uint32_t)c;
        me[k] = chunk_mask(a, c, pp0, pp1);
        ++k;
      }
      if (k) {
        CK(launch_page_discard(a->T, ce[0], me[0], ce[1], me[1], kind == DIR_DISCARD_LAZY, a->ps));
        a->n_launch++;
      }
    }
  }
  return hand_out(a, stream);
}

UM_API um_status um_discard(um_arena* a, uint64_t off, uint64_t len, void* stream) {
  return discard_common(a, off, len, stream, DIR_DISCARD);
}

UM_API um_status um_discard_lazy(um_arena* a, uint64_t off, uint64_t len, void* stream) {
  return discard_common(a, off, len, stream, DIR_DISCARD_LAZY);
}

UM_API um_status um_free(um_arena* a, uint64_t off, uint64_t len, void* stream) {
  ENTER(a);
  if (!range_ok(a, off, len)) return UM_EINVAL;
  um_status s = hand_in(a, stream);
  if (s) return s;
  if ((s = seq_room(a, 1))) return s;
  // frees frames an in-flight application kernel may still write: those finish first (R7)
  if (overlap_on(a) && (s = app_wait_all(a))) return s;
  a->ops++;
  a->subops++;
  ++a->clock;
  const uint64_t lo = (off + a->B - 1) / a->B, hi = (off + len) / a->B;   // fully covered blocks
  if (hi > lo) {
    cudaEvent_t sp = span_open(a);
    CK(launch_free(a->T, (uint32_t)lo, (uint32_t)(hi - lo), a->ps));
    span_close(a, sp, 0);
    a->n_launch++;
  }
  return hand_out(a, stream);
}

UM_API um_status um_evict(um_arena* a, uint64_t bytes, void* stream) {
  ENTER(a);
  um_status s = hand_in(a, stream);
  if (s) return s;
  if ((s = seq_room(a, 1))) return s;
  a->ops++;
  a->subops++;
  const uint32_t seq = ++a->clock;
  uint64_t want = (bytes + a->B - 1) / a->B;
  if (want > a->nframes) want = a->nframes;
  a->T.pfloor = seq;   // no pinned blocks: every in-flight application kernel finishes first
  if (overlap_on(a) && (s = app_wait_all(a))) return s;
  if (want && (s = evict_enqueue(a, seq, (uint32_t)want))) return s;
  return hand_out(a, stream);
}

UM_API um_status um_host_write(um_arena* a, uint64_t off, uint64_t len, void* stream) {
  ENTER(a);
  if (!range_ok(a, off, len)) return UM_EINVAL;
  um_status s = hand_in(a, stream);
  if (s) return s;
  if ((s = seq_room(a, 1))) return s;
  a->ops++;
  a->subops++;
  const uint32_t seq = ++a->clock;
  if (len) {   // pages (= blocks at single level) overlapping the range
    CK(launch_host_write(a->T, off / a->P, (off + len - 1) / a->P + 1, seq, a->ps));
    a->n_launch += 2;
  }
  return hand_out(a, stream);
}

UM_API um_status um_block_table(um_arena* a, const uint32_t** dev_map) {
  if (!a || !dev_map) return UM_EINVAL;
  *dev_map = a->T.map;
  return UM_OK;
}

UM_API um_status um_join(um_arena* a, void* stream) {
  ENTER(a);
  if (overlap_on(a)) {
    um_status s = app_wait_all(a);
    if (s) return s;
  }
  return hand_out(a, stream);
}

UM_API um_status um_stream(um_arena* a, void** stream) {
  if (!a || !stream) return UM_EINVAL;
  *stream = (void*)a->ps;
  return UM_OK;
}

static um_status sync_ctl(um_arena* a) {
  if (a->as) CK(cudaStreamSynchronize(a->as));
  CK(cudaMemcpyAsync(a->hctl, a->T.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, a->ps));
  CK(cudaStreamSynchronize(a->ps));
  if (a->hctl->err == 1u) a->sticky = UM_EINVAL;
  if (a->hctl->err == 2u) a->sticky = UM_ENOMEM;
  return a->sticky;
}

UM_API um_status um_get_stats(um_arena* a, um_stats* out) {
  ENTER(a);
  if (!out) return UM_EINVAL;
  um_status s = sync_ctl(a);
  int64_t v[16];
  for (int i = 0; i < 16; ++i) {
    v[i] = 0;
    for (int j = 0; j < 8; ++j) v[i] += a->hctl->stats[j][i];
  }
  v[S_OPS] = a->ops;
  v[S_SUBOPS] = a->subops;
  memcpy(out, v, sizeof(um_stats));
  return s;
}

UM_API um_status um_dump(um_arena* a, uint8_t* st, uint32_t* used_order, uint32_t* n_used, uint32_t* disc_order,
                         uint32_t* n_disc) {
  ENTER(a);
  um_status s = sync_ctl(a);
  if (s) return s;
  std::vector<uint32_t> hsk(a->nblocks);
  CK(cudaMemcpy(hsk.data(), a->T.sk, 4ull * a->nblocks, cudaMemcpyDeviceToHost));
  std::vector<uint8_t> hst(a->nblocks);
  for (uint32_t b = 0; b < a->nblocks; ++b) hst[b] = (uint8_t)(hsk[b] & 7u);
  if (st) memcpy(st, hst.data(), a->nblocks);
  std::vector<uint64_t> ring(a->L.cap);
  for (int r = 0; r < 2; ++r) {
    uint32_t* outp = r == RING_USED ? used_order : disc_order;
    uint32_t* outn = r == RING_USED ? n_used : n_disc;
    if (!outp && !outn) continue;
    CK(cudaMemcpy(ring.data(), r == RING_USED ? a->T.used_ring : a->T.disc_ring, 8 * a->L.cap, cudaMemcpyDeviceToHost));
    unsigned long long head = r == RING_USED ? a->hctl->used_head : a->hctl->disc_head;
    unsigned long long tail = r == RING_USED ? a->hctl->used_tail : a->hctl->disc_tail;
    uint32_t cnt = 0;
    for (unsigned long long p = head; p < tail; ++p) {
      uint64_t e = ring[p & (a->L.cap - 1)];
      uint32_t b = (uint32_t)e, k = (uint32_t)(e >> 32);
      if (b == UM_NONE) continue;   // a slot whose block did not enter the ring
      uint8_t x = hst[b];
      bool live = (r == RING_USED ? x == ST_G : (x == ST_GE || x == ST_GL)) && (hsk[b] >> 3) == k;
      if (live) {
        if (outp && cnt < a->nframes) outp[cnt] = b;
        ++cnt;
      }
    }
    if (outn) *outn = cnt;
  }
  return UM_OK;
}

UM_API um_status um_content_tags(um_arena* a, uint64_t* tags) {
  ENTER(a);
  if (!tags) return UM_EINVAL;
  if (overlap_on(a)) {
    um_status s = app_wait_all(a);
    if (s) return s;
  }
  CK(launch_tags(a->T, a->ps));
  CK(cudaMemcpyAsync(tags, a->T.tags, 8ull * a->nblocks * a->ppc, cudaMemcpyDeviceToHost, a->ps));
  CK(cudaStreamSynchronize(a->ps));
  return UM_OK;
}

UM_API um_status um_page_masks(um_arena* a, uint32_t* dead, uint32_t* lazy) {
  ENTER(a);
  if (a->ppc <= 1) return UM_EINVAL;
  um_status s = sync_ctl(a);
  if (s) return s;
  if (dead) CK(cudaMemcpy(dead, a->T.pdead, 4ull * a->nblocks, cudaMemcpyDeviceToHost));
  if (lazy) CK(cudaMemcpy(lazy, a->T.plazy, 4ull * a->nblocks, cudaMemcpyDeviceToHost));
  return UM_OK;
}

UM_API um_status um_xlog_attach(um_arena* a, void* buf, uint64_t cap_entries) {
  ENTER(a);
  if (buf && cap_entries == 0) return UM_EINVAL;
  // launches already enqueued carry their own copy of the tables: the reset is stream-ordered
  CK(cudaMemsetAsync(&a->T.ctl->xlog_n, 0, sizeof(unsigned long long), a->ps));
  a->T.xlog = (uint4*)buf;
  a->T.xlog_cap = buf ? cap_entries : 0;
  return UM_OK;
}

UM_API um_status um_xlog_count(um_arena* a, uint64_t* n) {
  ENTER(a);
  if (!n) return UM_EINVAL;
  um_status s = sync_ctl(a);
  if (s) return s;
  *n = a->hctl->xlog_n;
  return UM_OK;
}

UM_API um_status um_timing(um_arena* a, double* ms_plan, double* ms_xfer, uint64_t* xfer_launches,
                           uint64_t* launches, int reset) {
  ENTER(a);
  CK(cudaStreamSynchronize(a->ps));
  if (a->as) CK(cudaStreamSynchronize(a->as));
  FILE* lg = nullptr;
  if (const char* p = getenv("UM_SPAN_LOG")) lg = fopen(p, "a");   // diagnostics: one line per span
  for (auto& sp : a->spans) {
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, sp.a, sp.b));
    if (lg) fprintf(lg, "%u %d %.4f\n", sp.seq, sp.xfer, ms);
    (sp.xfer ? a->ms_xfer : a->ms_plan) += ms;
    a->evpool.push_back(sp.a);
    a->evpool.push_back(sp.b);
  }
  a->spans.clear();
  if (lg) fclose(lg);
  if (ms_plan) *ms_plan = a->ms_plan;
  if (ms_xfer) *ms_xfer = a->ms_xfer;
  if (xfer_launches) *xfer_launches = a->n_xfer;
  if (launches) *launches = a->n_launch;
  if (reset) {
    a->ms_plan = a->ms_xfer = 0;
    a->n_xfer = a->n_launch = 0;
  }
  return UM_OK;
}
