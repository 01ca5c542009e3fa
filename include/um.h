/* um.h — C ABI of libum, a B200-native, discard-aware unified-memory paging layer.
 *
 * Method: "UVM Discard: Eliminating Redundant Memory Transfers for Accelerators"
 * (Zhu et al., IISWC'22).  Citations "PAPER L<n>" are lines of its text
 * (/root/reference/PAPER.md at build time); "A<n>"/"R<n>" are the readings listed in
 * DESIGN.md §3 where the paper is silent.
 *
 * Model.  An arena of nblocks = arena_bytes / block_bytes virtual blocks (64 KiB or
 * 2 MiB) is backed by nframes = budget_bytes / block_bytes GPU frames in HBM and by a
 * pool of pinned, mapped host frames.  Every block is in one state:
 *   U  never populated            H  valid on host              HD discarded, not on GPU
 *   G  valid, mapped, in USED     GE eager-discarded (unmapped), in DISC
 *   GL lazy-discarded (mapped, software dirty bit clear), in DISC
 * GPU accesses ("faults") and prefetches to the GPU give a block a frame; when no frame
 * is free a victim is reclaimed in the order discarded-FIFO, then used-LRU
 * (PAPER L217-221).  Valid victims are written back (D2H); discarded ones are dropped
 * (Fig. 2 (6)); a discarded-then-reclaimed block is zero-filled instead of
 * migrated when it is used again (Fig. 2 (7)).
 *
 * Execution.  All planning (state tables, victim selection, work-list compaction) runs
 * in sm_100a kernels on device-resident tables; data moves by a kernel-driven TMA copy
 * over mapped pinned host memory (K4, no host round trip) or, as the comparison arm
 * (UM_F_COPY_CE), by the copy engines from the device-made plan (K4-CE, one host round
 * trip per sub-op).  No CPU fallback: the host never computes a state, a victim or a
 * transfer list.
 *
 * Conventions (all functions):
 *  - Return um_status; UM_OK = 0.  No exceptions cross the ABI.
 *  - Pointers are plain host pointers unless documented as device pointers.
 *  - Streams are cudaStream_t values passed as void* (0 = legacy default stream).
 *    Each op is stream-ordered like a CUDA memory op: it runs after
 *    prior work on `stream`, and later work on `stream` sees its effects.  Ops of one
 *    arena execute in call order on the arena's internal paging stream.
 *  - Range errors (outside the arena, bad dst) return UM_EINVAL and enqueue nothing.
 *    len == 0 is valid: it consumes one sequence number and moves nothing.
 *  - A CUDA failure returns UM_ECUDA and is sticky: later calls return it too.
 *  - One host thread per arena; a concurrent call returns UM_EBUSY.
 *  - Every call that enqueues work consumes one sequence number per sub-op (A3).
 */
#ifndef UM_H
#define UM_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct um_arena um_arena; /* opaque; library-owned host bookkeeping */

typedef enum {
  UM_OK = 0,
  UM_EINVAL = -1, /* bad argument / range; nothing enqueued                              */
  UM_ENOMEM = -2, /* arena (um_alloc) or host-frame pool exhausted (sticky when on device), or
                     the arena's 2^29 - 1 sequence numbers (one per sub-op) used up (sticky) */
  UM_ECUDA = -3,  /* CUDA error; sticky                                                   */
  UM_EBUSY = -4   /* concurrent call on the same arena                                   */
} um_status;

enum { UM_DST_GPU = 0, UM_DST_HOST = 1 };
enum { UM_ACC_READ = 1u, UM_ACC_WRITE = 2u };
enum { UM_ST_U = 0, UM_ST_H = 1, UM_ST_HD = 2, UM_ST_G = 3, UM_ST_GE = 4, UM_ST_GL = 5 };

enum {
  UM_F_DISCARD_OFF = 1u, /* "UVM-opt" baseline: discards are accepted no-ops */
  UM_F_COPY_CE = 2u,     /* comparison arm: move data with the copy engines (K4-CE:
                            device plan, one host round trip per sub-op, one
                            cudaMemcpyAsync per coalesced run on 2 copy streams)      */
  UM_F_CHECK = 4u,       /* poison frames with 0xA5 at creation; extra validation       */
  UM_F_APP_STAMP = 8u,   /* harness: after each touch sub-op, write the content stamp of
                            every UM_ACC_WRITE block (simulated application kernel)    */
  UM_F_TIMING = 16u,     /* record CUDA events around the planning and transfer kernels
                            of every op (read with um_timing)                          */
  UM_F_COPY_KERNEL = 32u,/* move data with the TMA kernel (K4).  This is also the default
                            (neither flag); the flag only overrides the diagnostic
                            UM_CE_MIN_BYTES environment threshold                      */
  UM_F_OVERLAP = 64u     /* pipelined application kernels (reading R7; the
                            paper's async API calls overlap compute):
                            the UM_F_APP_STAMP kernel of a touch sub-op runs on an
                            arena-internal app stream and overlaps the next sub-ops;
                            victim selection skips the blocks of the last 2 GPU sub-ops
                            (the longest suffix that leaves k satisfiable).  Ops that
                            move data out or free frames (prefetch HOST, evict) wait for
                            every app kernel.  An op's completion on the caller's stream
                            covers the paging work only: use um_join for the app work. */
};

/* One GPU access record of a batch (16 bytes).  Covers every block overlapping
 * [off, off+len); kind = UM_ACC_READ | UM_ACC_WRITE.  len is u32 (< 4 GiB per record). */
typedef struct {
  uint64_t off;
  uint32_t len;
  uint32_t kind;
} um_access;

typedef struct {
  int device;                 /* CUDA device ordinal                                       */
  uint32_t block_bytes;       /* 65536 or 2097152 (any power of two >= 4096 is accepted)  */
  uint64_t arena_bytes;       /* multiple of block_bytes; nblocks = arena/block < 2^31     */
  uint64_t budget_bytes;      /* nframes = budget/block >= 1                               */
  void *frames;               /* DEVICE, >= nframes*block_bytes, caller-owned              */
  void *workspace;            /* DEVICE, >= um_workspace_size(), caller-owned              */
  uint64_t workspace_bytes;
  void *const *host_chunks;   /* HOST array of n_host_chunks pinned+mapped host pointers;
                                 caller-owned, alive until destroy.  Together they form the
                                 host-frame pool: n_host_chunks*host_chunk_bytes/block_bytes
                                 frames (+1 block reserved as the zero page).  Contents need
                                 not be zero: host frames are written before being read.   */
  uint32_t n_host_chunks;
  uint64_t host_chunk_bytes;  /* multiple of block_bytes                                   */
  uint32_t flags;             /* UM_F_*                                                    */
  uint32_t page_bytes;        /* 0 or block_bytes: single level.  Otherwise two-level
                                 granularity (PAPER §5.3-5.4): a
                                 block is a chunk of block_bytes/page_bytes <= 32 pages
                                 (page_bytes a power of two >= 16384).  Chunks stay the
                                 residency and eviction unit (L198, L209, L217-221); a
                                 discard covering only some pages of a chunk marks them
                                 dead without unmapping (L211); dead pages are not written
                                 back and are zero-filled instead of migrated (L196-200)
                                 until accessed again (a touch revives eagerly discarded
                                 pages, a prefetch any, A8/A17).  Byte counters and
                                 content tags are per page.  Not combinable with
                                 UM_F_COPY_CE or UM_F_OVERLAP (UM_EINVAL).                */
  uint32_t reserve_blocks;    /* 0: evict on demand only (PAPER §5.5: "The eviction
                                 process starts when the GPU's free page queue is empty").
                                 R > 0: proactive eviction (reading R12, SURVEY
                                 NEXT-2): after every GPU sub-op with >= 1 block, if fewer
                                 than R frames are free, R - free more are reclaimed (best
                                 effort) in the same order (discarded FIFO, then the LRU end
                                 of USED, L219-221), skipping the sub-op's blocks and, with
                                 UM_F_OVERLAP, the window's; valid victims are written back
                                 on the paging stream, where they overlap the sub-op's
                                 application kernel under UM_F_OVERLAP.  Same seq as the
                                 sub-op.  Must be <= nframes; single level only (UM_EINVAL
                                 with two-level page_bytes).                              */
} um_config;

/* Counters (int64, 16 slots).  Byte counters are multiples of block_bytes. */
typedef struct {
  int64_t h2d_bytes, d2h_bytes, zf_bytes, h2d_avoided_bytes, d2h_avoided_bytes,
      faults, hits, remaps, unmaps, revalidations, refreshes, evictions, ops, subops;
  int64_t pad[2];
} um_stats;

/* Bytes of device workspace the arena needs (state tables, rings, work lists). */
um_status um_workspace_size(const um_config *cfg, uint64_t *bytes);

/* Create an arena: all blocks start in U, all frames free.  Synchronizes. */
um_status um_arena_create(const um_config *cfg, um_arena **out);

/* Synchronize and free the library's host-side state (caller memory is not freed). */
um_status um_arena_destroy(um_arena *a);

/* Block-aligned bump allocation (layout rule: offset = previous end rounded up to
 * block_bytes).  UM_ENOMEM if it does not fit.  No device work. */
um_status um_alloc(um_arena *a, uint64_t bytes, uint64_t *off);

/* cudaMemPrefetchAsync analogue (PAPER §2.1).  dst GPU: every block overlapping
 * the range gets a frame (U/HD zero-filled, H migrated, G refreshed to MRU, GE
 * re-mapped, GL revalidated = software dirty bit set); ops with more
 * distinct blocks than frames are split into ascending sub-ops (A3).  dst HOST: G
 * migrates back (D2H), GE/GL/HD/U become H with no transfer (A9). */
um_status um_prefetch(um_arena *a, uint64_t off, uint64_t len, int dst, void *stream);

/* UvmDiscard (PAPER §5.1): for blocks FULLY inside the range (PAPER L211,
 * A4): G -> GE (unmap; appended to DISC), GL -> GE, H -> HD. */
um_status um_discard(um_arena *a, uint64_t off, uint64_t len, void *stream);

/* UvmDiscardLazy (PAPER §5.2): fully covered G -> GL (mapping kept, appended
 * to DISC), H -> HD.  The caller MUST um_prefetch the range before reusing it (either
 * destination, A17); an access without it does not revalidate (A8). */
um_status um_discard_lazy(um_arena *a, uint64_t off, uint64_t len, void *stream);

/* A batch of GPU accesses ("faults"): the distinct blocks of all
 * records are serviced in ascending sub-ops of <= nframes blocks.  `acc` is read before
 * return (the caller may reuse it). */
um_status um_touch_batch(um_arena *a, const um_access *acc, uint32_t n, void *stream);

/* The same batch with the records in DEVICE-accessible memory (the GPU's own fault
 * buffer: faults are raised by the GPU): `acc` = n records, 16-byte
 * aligned, written in stream order before this call on `stream`.  The GPU range-checks,
 * expands and deduplicates them (op bitmap -> sorted distinct block list); the host only
 * reads back the block count (one stream synchronization) to number the sub-ops, so the
 * records have been consumed when the call returns.  A record outside the arena:
 * UM_EINVAL with no state changed.  Single level only (UM_EINVAL with page_bytes). */
um_status um_touch_batch_dev(um_arena *a, const um_access *acc, uint32_t n, void *stream);

/* The application releases [off, off+len) (cudaFree of managed memory; reading R9 of
 * DESIGN.md).  Every block FULLY inside the range returns to U (never populated: it
 * reads as zeros) with no transfer: its GPU frame goes back to the pool the eviction
 * process takes before any discarded or used page (the paper's unused queue, §5.5
 * L217-221), a host copy is released.  The virtual range stays allocated (um_alloc is a
 * bump allocator).  Consumes one sequence number. */
um_status um_free(um_arena *a, uint64_t off, uint64_t len, void *stream);

/* Make >= bytes of frames free by the eviction policy (PAPER §5.5). */
um_status um_evict(um_arena *a, uint64_t bytes, void *stream);

/* Harness op (simulated CPU writes, Listing 6 "Generate data, labels" L330): every block
 * overlapping the range must be host-resident (H); its host frame receives the content
 * stamp of this op.  A block not in H sets a sticky device error (UM_EINVAL). */
um_status um_host_write(um_arena *a, uint64_t off, uint64_t len, void *stream);

/* DEVICE pointer to the block table map[nblocks] (u32 frame id, 0xffffffff = unmapped)
 * that application kernels translate through: addr = frames + map[b]*block + off%block.
 * G and GL blocks are mapped; U/H/HD/GE are not (an eager discard unmaps). */
um_status um_block_table(um_arena *a, const uint32_t **dev_map);

/* Make `stream` wait for all work the arena has enqueued so far, including the
 * UM_F_OVERLAP application kernels (without that flag it equals an empty op's
 * hand-off).  Enqueues only; never blocks the host. */
um_status um_join(um_arena *a, void *stream);

/* The arena's internal paging stream (work enqueued on it needs no event hand-off). */
um_status um_stream(um_arena *a, void **stream);

/* Synchronizes; copies the counters out. */
um_status um_get_stats(um_arena *a, um_stats *out);

/* Synchronizes; exports the observable result for parity: st[nblocks] (UM_ST_*),
 * USED order (LRU first) and DISC order (FIFO head first) as block ids.  Buffers
 * used_order/disc_order need room for nframes entries.  Any pointer may be NULL. */
um_status um_dump(um_arena *a, uint8_t *st, uint32_t *used_order, uint32_t *n_used,
                  uint32_t *disc_order, uint32_t *n_disc);

/* Harness: synchronizes; content tag of every block (u64 per block; per page, nblocks *
 * block_bytes/page_bytes entries, at two levels): 0 = all-zero, stamp s = filled with
 * the 16-byte pattern {s, ~s}, UINT64_MAX = anything else (corrupt).  Reads frames
 * (G/GE/GL) or host frames (H; HD/U and the dead pages of an H chunk read as zero). */
um_status um_content_tags(um_arena *a, uint64_t *tags);

/* Two-level arenas (page_bytes < block_bytes): synchronizes; per chunk, the dead-page
 * and lazily-discarded-page masks (bit p = page p).  Either pointer may be NULL.
 * UM_EINVAL on a single-level arena. */
um_status um_page_masks(um_arena *a, uint32_t *dead, uint32_t *lazy);

/* Synchronizes.  Device time (ms) spent since the last reset in planning kernels
 * (classify, victim selection, directives, ring compaction) and in the transfer engine
 * (fused swap / write-back / zero-fill kernel), summed per launch from CUDA events
 * (needs UM_F_TIMING, else 0), the number of transfer-kernel launches, and the number of
 * libum kernel launches enqueued.  reset != 0 clears all four afterwards. */
um_status um_timing(um_arena *a, double *ms_plan, double *ms_xfer, uint64_t *xfer_launches,
                    uint64_t *launches, int reset);

/* Transfer log (parity and redundant-transfer accounting; PAPER
 * L34 "overwritten before being read", Fig. 3 L125 required vs performed transfers).
 * Attaches a caller-owned DEVICE buffer of cap_entries records of 16 bytes
 * {uint32 seq, uint32 block, uint32 kind (0 = H2D, 1 = D2H, 2 = zero-fill), uint32
 * state of the block before the move (UM_ST_*)} and restarts the count at zero.  From
 * then on every block whose migration, write-back or zero-fill enters a work list the
 * transfer engine executes appends one record, in no particular order (sort by seq).
 * buf = NULL detaches.  The caller keeps the buffer alive until it detaches or
 * destroys the arena.  Enqueued on the paging stream; UM_EINVAL if buf != NULL and
 * cap_entries == 0. */
um_status um_xlog_attach(um_arena *a, void *buf, uint64_t cap_entries);

/* Synchronizes.  Number of records appended since the last attach; records beyond the
 * capacity were counted but not written (*n > cap_entries means the log overflowed). */
um_status um_xlog_count(um_arena *a, uint64_t *n);

const char *um_strerror(um_status s);

#ifdef __cplusplus
}
#endif
#endif /* UM_H */
