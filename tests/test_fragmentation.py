"""N3 (CPU): the fragmentation study replays a seeded 6-shape trace through the library allocator;
fragmentation (unused / peak allocated) stays within [0, 1), grows with slab size on
average, and on this trace stays under the paper's 20% overall bound."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))


def test_fragmentation_trace_small():
    from paper_conf_sosp_xiang0qyzyzl0025_b200 import build
    build.build()
    import fragmentation as F
    pool = 64 * F.GIB
    ev = F.trace(4000, pool, seed=3001)
    small, big = F.run(ev, pool, F.GIB // 4), F.run(ev, pool, 2 * F.GIB)
    k = "frag_unused_over_peak_allocated_mean"
    for r in (small, big):
        assert 0 <= r[k] < 1 and r["peak_allocated_GiB"] > 0
        assert 0.3 < r["occupancy_used_over_pool_mean"] < 0.7
    assert small["oom_allocs"] == 0
    assert small[k] <= big[k]
    assert small[k] < 0.20
