"""CPU ORACLE — TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct NumPy/Python statement of what the Aegaeon data-movement hot
path computes (§5.2 "Unified KV cache" / "Quick model loading", §5.3 rules ❶❷❸,
Table 1, Fig. 9/10).  Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import it.  It shares no code with the CUDA
library (``paper_conf_sosp_xiang0qyzyzl0025_b200``) and imports nothing from it; the only
common dependency is the seeded input generator package ``aeg_inputs``.

Modules (each function cites the passage it follows):
  shape    O1  per-token / per-chunk / per-block byte arithmetic (Table 1)
  slab     O2  slab allocator with move-list quarantine and slab reclaim (§5.2, §5.3)
  kv       O3–O7 gather / scatter / swap-out / swap-in / migrate as byte copies
  weights  O8  Megatron TP shard extraction + bump allocation (§5.2)
  rules    O9/O10 layer readiness and the ❶❷❸ happens-before checker (§5.3)
  memmove  N1  on-device relocation of prefetched weights (§5.2 "3.b Copy")

Pins: see tests/test_oracle_*.py and DESIGN.md "Oracle pins".  Functions without an
independent pin say "parity unpinned" in their docstring (only timing-related parts of O9).
"""
