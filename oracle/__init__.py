"""CPU oracle for the discard-aware paging layer — TEST INFRASTRUCTURE ONLY.

Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s `cpu_baseline` / `--impl
reference` legs may import anything under `oracle/`.  The product path
(`paper_conf_iiswc_zhucvhcr22_b200/`) never imports it, and this package never imports
the product path: the two share no code, constants, tables or helpers.  The only shared
input is the trace from `tracegen/` (op records, no method arithmetic).

`oracle.sim` is a plain, slow, sequential simulator of the UVM model in the paper
(PAPER.md = "UVM Discard", Zhu et al., IISWC'22), following SURVEY.md §8(c) step by step:
fault-driven migration (Fig. 1, L87), prefetch (§2.1), the eviction order
free -> discarded FIFO -> used LRU (§5.5), eager UvmDiscard (§5.1),
UvmDiscardLazy with software dirty bits (§5.2), skipped transfers (§5.3,
L196-200), 2 MB-granular discard ignoring partial regions (§5.4), delayed
reclamation (§5.6) and access-after-discard revival (§5.7).

Pins (tests/test_oracle_*.py, `-m "not gpu"`): the hand-enumerated scenarios E1-E8,
the closed form of the C2 streaming trace, the textbook LRU/FIFO reductions, a second
independently written linked-list formulation on brute-forced inputs, and the
invariants (i)-(vii) of SURVEY §8(c).  Parity unpinned: the exact byte totals of the
C3 DNN trace (pinned only by the invariants), contents of GE/GL/HD blocks beyond
readings A7/A9, all timings.

`oracle.chunks.ChunkOracle` is the two-level model of SURVEY NEXT-1 (2 MiB chunks as the
residency / eviction unit, page-granular partial discards, reading R10), pinned
in tests/test_oracle_chunks.py (hand-derived scenarios, reduction to oracle.sim,
page-level invariants); the CUDA path's two-level mode is compared with it in
tests/test_gpu_pages.py.

`oracle.rmt` is the redundant-transfer accounting of SURVEY §8(c) item 7 (DESIGN.md
reading R8), pinned in tests/test_rmt.py (Fig. 2's two redundant transfers, the C2
closed form, a versioned flat-memory second formulation).

`Oracle.free_range` is um_free (reading R9), pinned by the hand-derived scenarios E13.
"""
from .sim import Oracle, replay, ST_NAMES, stamp  # noqa: F401
