"""Pin for N1 (oracle/memmove.py): brute force over every (src, dst, n) in a 12-byte buffer against
the classic direction-aware byte loop (ascending when dst < src, descending otherwise) — a different
formulation from the oracle's copy-through-a-temporary — plus the non-overlapping special case."""
import numpy as np

from oracle.memmove import memmove


def byte_loop(buf, src, dst, n):
    out = buf.copy()
    rng = range(n) if dst < src else range(n - 1, -1, -1)
    for i in rng:
        out[dst + i] = out[src + i]
    return out


def test_memmove_bruteforce():
    buf = np.arange(12, dtype=np.uint8) * 7 + 3
    cases = 0
    for n in range(0, 13):
        for src in range(0, 13 - n):
            for dst in range(0, 13 - n):
                assert np.array_equal(memmove(buf, src, dst, n), byte_loop(buf, src, dst, n))
                cases += 1
    assert cases > 500


def test_disjoint_is_plain_copy():
    buf = np.arange(100, dtype=np.uint8)
    out = memmove(buf, 60, 0, 30)
    assert np.array_equal(out[:30], buf[60:90]) and np.array_equal(out[30:], buf[30:])
