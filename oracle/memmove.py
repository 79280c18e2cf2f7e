"""N1 — on-device relocation of prefetched weights.  TEST INFRASTRUCTURE ONLY.

PAPER.md:1359-1364 (§5.2): "the prefetched model is allocated right after the running model in the
self-managed buffer, and moved to the start of the buffer during the actual scale-up with a cheap
on-device copy (step 3.b in Figure 9)."  The move may overlap (28 GB prefetched vs 14 GB running in
Fig. 9), so it has memmove semantics (reading 21): the destination receives the
bytes the source held BEFORE the move, as if copied through a temporary buffer.
"""
from __future__ import annotations

import numpy as np


def memmove(buf: np.ndarray, src: int, dst: int, n: int) -> np.ndarray:
    """Returns buf' with buf'[dst:dst+n] = buf[src:src+n] (pre-move bytes); all else unchanged."""
    assert 0 <= src and 0 <= dst and src + n <= buf.size and dst + n <= buf.size
    tmp = buf[src:src + n].copy()
    out = buf.copy()
    out[dst:dst + n] = tmp
    return out
