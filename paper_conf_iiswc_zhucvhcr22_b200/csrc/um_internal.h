// Internal layout shared by the host runtime (um_host.cu) and the kernels
// (um_kernels.cu).  Not part of the ABI.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#define UM_NONE 0xffffffffu

namespace um {

// Block states (same values as UM_ST_* in include/um.h).
enum : uint8_t { ST_U = 0, ST_H = 1, ST_HD = 2, ST_G = 3, ST_GE = 4, ST_GL = 5 };

// Stats slots (order of um_stats).
enum {
  S_H2D = 0, S_D2H, S_ZF, S_H2D_AV, S_D2H_AV, S_FAULTS, S_HITS, S_REMAPS, S_UNMAPS,
  S_REVAL, S_REFRESH, S_EVICT, S_OPS, S_SUBOPS, S_N = 16
};

// Device control block: ring cursors, free-stack tops, the current sub-op's plan
// sizes, counters and the self-cleaning scan state.
struct Ctl {
  unsigned long long used_head, used_tail, disc_head, disc_tail;
  int free_top;          // free GPU frames: free_stack[0, free_top)
  int hfree_top;         // free host frames: hfree_stack[0, hfree_top)
  unsigned int n_need;   // current sub-op: blocks needing a frame (need list length)
  unsigned int n_rekey;  // current sub-op: USED appends staged at used_tail
  unsigned int f0;       // free_top when the sub-op's victims were chosen
  unsigned int n_vict;   // victims chosen
  unsigned int n_d2h;    // D2H-only work-list length (prefetch HOST / evict)
  unsigned int err;      // sticky device error (0 or -um_status)
  unsigned int scan_ticket, scan_done;  // decoupled look-back tile ticket / completion
  unsigned int app_units;               // D2H-only service completion counter
  unsigned int vict_done;               // wide victim apply completion counter
  unsigned int need_acc;                // streaming classify: need-list slots taken so far
  unsigned int reach_tile;              // wide victim scan: first tile whose inclusive count >= k
  unsigned int iv_m, iv_d;              // device intake: intervals produced (list form: write blocks), distinct blocks
  unsigned int iv_err;                  // device records: a record outside the arena (read and cleared by the host)
  unsigned long long minkeep[2];        // wide victim scan: first kept ring position
  unsigned int k_want;                  // wide victim scan: victims wanted
  unsigned int need_cnt[2];             // streaming classify: need-list slots, by sub-op parity
  unsigned int k0_take, k0_pend;        // wide victim scan with k = 0: frames to take, pending flag
  unsigned long long vs_combo;          // wide victim scan: (candidates of finished tiles << 32) | next ticket
  unsigned int first_skip;              // wide victim scan: first ticket not examined
  unsigned int vs_fin;                  // wide victim scan: tiles finished (ticket pacing)
  unsigned int vt_reach;                // wide victim scan: passes in the apply work table (vpass)
  unsigned int pc_done;                 // k_plan_commit completion ticket (host read-back flag)
  unsigned long long xlog_n;            // transfer log: records appended (may exceed the capacity)
  unsigned long long need_tk;           // k_classify with k = 0 certain: (need count << 32) | tickets
  // counters, striped over 8 cache lines by CTA index (fire-and-forget atomics from
  // thousands of CTAs do not serialise on one address); the host sums the stripes
  long long stats[8][S_N];
};

// One need item's transfer plan (K4-CE path exports these to the host).
struct XItem {
  uint32_t fr;      // destination GPU frame
  uint32_t src_hf;  // host frame to migrate from (XI_H2D), else NONE
  uint32_t dst_hf;  // host frame receiving the victim's write-back (XI_D2H), else NONE
  uint32_t flags;
};
enum { XI_H2D = 1u, XI_ZF = 2u, XI_D2H = 4u, XI_SWAP = 8u };

// Transfer log record (um_xlog_attach): one per block moved or zero-filled, appended
// where the work list that the transfer engine executes is fixed.
enum { XL_H2D = 0u, XL_D2H = 1u, XL_ZF = 2u };

// Everything a kernel needs, passed by value.
struct Tables {
  uint32_t* sk;         // [nblocks] packed state word (key << 3) | state, key = ukey or
                        // dkey (a seq < 2^29): one load decides whether a ring entry is live
  uint32_t* frame_of;   // [nblocks] GPU frame (G/GE/GL) or NONE
  uint32_t* map;        // [nblocks] app-visible table: frame if mapped (G/GL) else NONE
  uint32_t* hframe;     // [nblocks] host frame holding the block's data (H only) or NONE
  uint32_t* pin;        // [nblocks] seq of the sub-op that pinned the block
  uint32_t* free_stack; // [nframes]
  uint32_t* hfree_stack;// [nhframes]
  uint64_t* used_ring;  // [cap] (key<<32)|block, current buffer
  uint64_t* disc_ring;  // [cap]
  uint64_t cap_mask;
  uint32_t* need;       // [nframes] blocks needing a frame, ascending
  uint8_t* needk;       // [nframes] their state at classification
  uint32_t* needhf;     // [nframes] their host frame at classification (H) or NONE
  uint32_t* victim;     // [nframes] victims, in eviction order
  uint32_t* vscratch;   // [2 cap + 2048] wide victim scan: the candidates of tile t at [t * 2048, ...), in ring order
  ulonglong2* vpass;    // [nframes / 128 + tiles] wide victim apply work table, one entry per pass of <= 128 victims: {first victim index | tile << 32, offset in the tile's candidates | victims << 32}
  uint32_t* vframe;     // [nframes] victim's frame
  uint32_t* vhf;        // [nframes] host frame receiving a G victim's write-back, else NONE
  uint8_t* vkind;       // [nframes] victim's state when chosen
  uint32_t* d2h_frame;  // [nframes] D2H-only list (prefetch HOST, evict)
  uint32_t* d2h_hf;     // [nframes]
  unsigned long long* tile_status;  // [max tiles] decoupled look-back
  uint32_t* tile_cnt;   // [max tiles * 8] per-tile counter partials
  uint64_t* tags;       // [nblocks] content tags (harness)
  XItem* xitems;        // [nframes] exported plan of the current sub-op (K4-CE path)
  // device intake (dedupe of unsorted / overlapping access batches, SURVEY A1 "op bitmap")
  uint32_t* obits;      // [nwords] blocks touched by the batch (cleared after each batch)
  uint32_t* wbits;      // [nwords] ... with a WRITE access
  uint32_t* dlo;        // [nblocks] produced intervals: first block
  uint32_t* dpre;       // [nblocks + 1] exclusive prefix of interval lengths (pre[m] = D)
  uint8_t* dw;          // [nblocks] write flag per interval
  Ctl* ctl;
  char* frames;             // device, nframes * B
  char* const* hchunks;     // device array of host-chunk device pointers
  uint32_t hpc;             // host frames per chunk
  uint32_t B;               // block bytes
  uint32_t nblocks, nframes, nhframes;
  uint32_t zero_hf;         // host frame id of the zero page (never allocated)
  // victim floor: a live ring entry is a candidate iff pin[b] < pfloor.  = seq of the
  // current sub-op (its own blocks are never victims, A3), or with UM_F_OVERLAP the seq
  // of the oldest GPU sub-op whose application kernel may still run (reading R7)
  uint32_t pfloor;
  // K4-CE read-back without a host stream sync: k_plan_commit also writes the plan into
  // the pinned host mirror `hx` and its last CTA publishes {seq, n_need} in `hflag`
  // (mapped pinned memory) after a system-scope fence; the host spins on hflag[0]
  XItem* hx;
  unsigned int* hflag;
  // transfer log (null = off): {seq, block, XL_* kind, state before the move}
  uint4* xlog;
  unsigned long long xlog_cap;
  // Two-level granularity (null = single level): a block is
  // a chunk of ppc pages of P bytes.  Per chunk, bit p = page p:
  //   pdead  pages discarded while the chunk itself is not (G or H only): not written
  //          back, zero-filled instead of migrated
  //   plazy  the subset discarded lazily (revived by a prefetch only, A8 / A17)
  //   phz    pages of an H chunk whose host content is logically zero (released or never
  //          written host pages that became live again): migrated from the zero page
  uint32_t* pdead;
  uint32_t* plazy;
  uint32_t* phz;
  uint32_t* d2h_dmask;  // [nframes] dead-page mask of each D2H-only item (when it was listed)
  uint32_t ppc;         // pages per chunk (1 = single level)
  uint32_t P;           // page bytes (= B at single level)
};

// A GPU-destination op's distinct blocks as sorted disjoint intervals.  Interval j
// covers blocks [lo[j], lo[j] + pre[j+1] - pre[j]); pre[] is the op-global exclusive
// prefix of block counts; wflag[j] = the interval holds UM_ACC_WRITE blocks.
// Small ops (m <= kIvInline) carry the list inline in the kernel parameters (no staging
// copy); larger ones point at a staged device copy.
constexpr uint32_t kIvInline = 24;
// UM_F_OVERLAP: number of previous GPU sub-ops whose application kernels may still run
// while a sub-op is serviced (reading R7; the oracle's `overlap` parameter)
constexpr int kOverlapW = 2;
constexpr int kOverlapWMax = 8;   // UM_OVERLAP_W (diagnostic A/B): another window length
struct OpIv {
  const uint32_t* lo;
  const uint32_t* pre;
  const uint8_t* wflag;
  const uint32_t* blist; // "fault list" form (staged; null otherwise): the op's distinct blocks
                         // in ascending order, one u32 per block, bit 31 = UM_ACC_WRITE.
                         // Chosen by the host when intervals average <= 3 blocks (a sparse
                         // batch): item g's block is one coalesced load, no interval lookup
  const uint32_t* tj;   // staged lists: per tile of the current sub-op, the interval slice
                        // [tj[2t], tj[2t+1]] its items fall in (host-computed, no search)
  const uint32_t* pcov; // two-level (with blist): per item, the chunk's pages the op covers
  const uint32_t* pw;   // two-level (with blist): per item, the chunk's pages it writes
  uint32_t m;
  uint32_t inl;
  uint32_t ilo[kIvInline];
  uint32_t ipre[kIvInline + 1];
  uint8_t iw[kIvInline];
};

constexpr int kScanTPB = 512;
constexpr int kScanIPT = 8;
constexpr int kScanTile = kScanTPB * kScanIPT;
// streaming state kernels (classify, directives): no inter-CTA ordering, one wave
constexpr int kStTPB = 256;
// multi-CTA classify: items per thread (4, or 8 with UM_CLS_IPT=8); its tile in items
uint32_t classify_tile();
constexpr int kVictTPB = 1024;
constexpr int kVaTPB = 512;   // k_victims_apply block size
constexpr int kVictIPT = 4;
constexpr int kXferStages = 4;
constexpr uint32_t kXferChunk = 16384;

enum SvcMode { SVC_SUBOP = 0, SVC_D2H_ONLY = 1 };
enum DirKind { DIR_DISCARD = 0, DIR_DISCARD_LAZY = 1, DIR_PREFETCH_HOST = 2 };
enum RingId { RING_USED = 0, RING_DISC = 1 };

// Launch wrappers (um_kernels.cu).  All enqueue on `s`; none synchronizes.
cudaError_t setup_kernels();
cudaError_t launch_init(const Tables& T, int nhframes_alloc, cudaStream_t s);
// tail0: the ring tail before this sub-op's appends (host-tracked, exact); npar: parity
// slot of the need counter for multi-CTA sub-ops (alternates per multi-CTA sub-op)
// k0 != 0: the host guarantees that the sub-op needs no victim (its blocks fit the free
// frames); classify then does the victim kernels' k = 0 bookkeeping and none is launched
cudaError_t launch_classify(const Tables& T, OpIv iv, uint32_t g0, uint32_t n, uint32_t seq, int touch,
                            unsigned long long tail0, int npar, int k0, cudaStream_t s);
cudaError_t launch_victims(const Tables& T, uint32_t seq, int evict_mode, uint32_t want, int npar, cudaStream_t s);
// K1+K2+K3 fused in one CTA for sub-ops of <= kSmallPlan blocks
constexpr uint32_t kSmallPlan = 4096;
cudaError_t launch_plan_small(const Tables& T, const OpIv& iv, uint32_t g0, uint32_t n, uint32_t seq, int touch,
                              unsigned long long tail0, cudaStream_t s);
// multi-CTA victim selection for large sub-ops (scan bound = max ring entries to scan)
cudaError_t launch_victims_wide(const Tables& T, uint32_t seq, int evict_mode, uint32_t want,
                                uint64_t scan_bound, uint32_t max_victims, int npar, cudaStream_t s);
constexpr uint32_t kVictWideMin = 8192;
cudaError_t launch_service(const Tables& T, int mode, uint32_t seq, uint32_t max_items, cudaStream_t s);
cudaError_t launch_app_stamp(const Tables& T, OpIv iv, uint32_t g0, uint32_t n, uint32_t seq, int ctas_per_sm,
                             cudaStream_t s);
cudaError_t launch_directive(const Tables& T, int kind, uint32_t lo, uint32_t n, uint32_t seq,
                             int discard_off, unsigned long long tail0, cudaStream_t s);
cudaError_t launch_ring_compact(const Tables& T, int ring, uint64_t* dst, uint64_t cap_bound, cudaStream_t s);
// um_free of blocks [lo, lo + n): back to U, frames and host frames released (R9).
cudaError_t launch_free(const Tables& T, uint32_t lo, uint32_t n, cudaStream_t s);
// Harness host write of pages [p0, p1) (global page indices; p = block at single level).
cudaError_t launch_host_write(const Tables& T, uint64_t p0, uint64_t p1, uint32_t seq, cudaStream_t s);
cudaError_t launch_tags(const Tables& T, cudaStream_t s);
cudaError_t launch_plan_commit(const Tables& T, uint32_t seq, uint32_t max_items, cudaStream_t s);
cudaError_t launch_zero_items(const Tables& T, uint32_t i0, uint32_t i1, cudaStream_t s);
cudaError_t launch_poison(const Tables& T, cudaStream_t s);
// Two-level page masks (NEXT-1).  After a GPU sub-op: revive the pages it covers
// (touch: eagerly discarded pages only; prefetch: all, clearing lazy).  After a
// prefetch(HOST) of chunks [lo, lo+n) covering pages [p0, p1) (global): revive, and mark
// revived pages of host chunks zero.  A discard's partial edge chunk c: pages m.
cudaError_t launch_page_revive(const Tables& T, const OpIv& iv, uint32_t g0, uint32_t n, int touch, cudaStream_t s);
cudaError_t launch_page_host_revive(const Tables& T, uint32_t lo, uint32_t n, uint64_t p0, uint64_t p1,
                                    cudaStream_t s);
cudaError_t launch_page_discard(const Tables& T, uint32_t c0, uint32_t m0, uint32_t c1, uint32_t m1, int lazy,
                                cudaStream_t s);
// Device intake: mark a staged record chunk into the op bitmaps; turn the bitmap words
// [w0, w1) into sorted disjoint intervals (dlo/dpre/dw, ctl->iv_m / iv_d); clear them.
// Records must not cover more than kMarkMaxBlocks blocks each (the host splits them).
constexpr uint32_t kMarkMaxBlocks = 1024;
struct MarkRec { uint32_t lo, cnt, w, pad; };   // one staged (split) record, in blocks
cudaError_t launch_mark(const Tables& T, const MarkRec* rec, uint32_t n, cudaStream_t s);
cudaError_t launch_runs(const Tables& T, uint32_t w0, uint32_t w1, cudaStream_t s);
cudaError_t launch_intake_clear(const Tables& T, uint32_t w0, uint32_t w1, cudaStream_t s);
// Device-resident records (um_touch_batch_dev): mark n um_access records (16-byte
// aligned, device-accessible) into the op bitmaps (range errors set ctl->iv_err); turn
// the bitmap's nwords words into the sorted distinct block list dlo (bit 31 = write),
// ctl->iv_d = blocks, ctl->iv_m = write blocks, and clear the bitmaps.
cudaError_t launch_mark_acc(const Tables& T, const void* acc, uint32_t n, uint32_t lg, cudaStream_t s);
cudaError_t launch_list(const Tables& T, uint32_t nwords, cudaStream_t s);

}  // namespace um
