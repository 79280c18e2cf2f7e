"""Pins for O2 (oracle/slab.py): the paper's slab prose checked
as properties, with brute-force enumeration of every admissible choice on tiny pools.

Nothing here re-types the allocator: each check is a property the paper's text fixes (or a
DESIGN.md reading), evaluated from the observable state before/after each call.
"""
import itertools
import random

import pytest

from oracle.shape import KVShape
from oracle.slab import AllocError, SlabPool, OOM, STATE, INVALID

# block_bytes: A = 2*1*... choose shapes so that a 256-byte slab holds 2 blocks of A, 1 of Bsh
A = KVShape(L=2, H=1, D=2, s=2, B=8)     # chunk 64 B, block 128 B  -> k = 2 in a 256 B slab
Bsh = KVShape(L=3, H=1, D=2, s=2, B=8)   # chunk 64 B, block 192 B  -> k = 1
SLAB = 256


def snapshot(p: SlabPool):
    return ([None if s is None else s for s in p.shape], [frozenset(o) for o in p.owned], dict(p.quarantine))


def check_invariants(p: SlabPool, live):
    # I1: no block owned twice (across live allocations)
    all_h = [h for hs in live.values() for h in hs]
    assert len(all_h) == len(set(all_h))
    owned = {(s, j) for s in range(p.n_slabs) for j in p.owned[s]}
    assert owned == set(all_h)
    for s in range(p.n_slabs):
        q = {j for (qs, j) in p.quarantine if qs == s}
        if p.shape[s] is None:
            # I4: unassigned slabs are empty
            assert not p.owned[s] and not q
        else:
            k = p.k(p.shape[s])
            # I2: owned and quarantined are disjoint subsets of the slab's blocks
            assert p.owned[s] <= set(range(k)) and q <= set(range(k)) and not (p.owned[s] & q)
            # "reclaims slabs that contain no occupied blocks" (reading 10: nor quarantined)
            assert p.owned[s] or q


def admissible_choices(p: SlabPool, shape, n, done_reclaimable):
    """All n-subsets the paper's rule allows: free non-quarantined blocks of existing same-shape
    slabs first; new slabs only when those are exhausted, as few as needed."""
    quarantined = {b for b, xs in p.quarantine.items() if not (xs <= done_reclaimable)}
    existing = [(s, j) for s in range(p.n_slabs) if p.shape[s] == shape
                for j in range(p.k(shape)) if j not in p.owned[s] and (s, j) not in quarantined]
    unassigned = [s for s in range(p.n_slabs) if p.shape[s] is None]
    k = p.k(shape)
    if n <= len(existing):
        return [tuple(sorted(c)) for c in itertools.combinations(existing, n)], existing, unassigned
    need = n - len(existing)
    n_new = -(-need // k)
    out = []
    for slabs in itertools.combinations(unassigned, n_new):
        pool = [(s, j) for s in slabs for j in range(k)]
        for c in itertools.combinations(pool, need):
            if len({s for s, _ in c}) == n_new:
                out.append(tuple(sorted(existing + list(c))))
    return out, existing, unassigned


def do_alloc(p, shape, n, live, tag):
    before = snapshot(p)
    done = set(p.done)
    # slabs that only hold completed-quarantine blocks become unassigned by the on-demand reclaim;
    # model that by computing admissible choices after a reclaim on a copy
    import copy
    pc = copy.deepcopy(p)
    pc.reclaim()
    choices, existing, unassigned = admissible_choices(pc, shape, n, done)
    try:
        got = p.alloc(shape, n)
    except AllocError as e:
        assert e.code == OOM
        # completeness: fails only when capacity is short (after the on-demand reclaim)
        cap = len(existing) + len(unassigned) * pc.k(shape)
        assert cap < n
        # I6: all-or-nothing — ownership and slab assignment unchanged
        after = snapshot(p)
        assert after[1] == before[1]
        return None
    # I7: distinct handles
    assert len(got) == len(set(got)) == n
    # I5: never a quarantined (move-list) block whose transfer is unfinished, never an owned one
    for s, j in got:
        assert j not in before[1][s]
        xs = before[2].get((s, j))
        assert xs is None or xs <= done
    # paper rule + reading 6: the choice is admissible and the lowest-first one among them
    assert tuple(sorted(got)) in choices
    assert tuple(sorted(got)) == min(choices)
    # reading 6 also fixes the order: blocks of already-assigned slabs first, then blocks of newly
    # acquired slabs, each part ascending (slab, index)
    old = [h for h in got if pc.shape[h[0]] == shape]
    new = [h for h in got if pc.shape[h[0]] is None]
    assert list(got) == sorted(old) + sorted(new)
    live[tag] = list(got)
    return got


OPS = [("alloc", A, 1), ("alloc", A, 2), ("alloc", A, 3), ("alloc", Bsh, 1), ("alloc", Bsh, 2),
       ("free", 0), ("free", -1), ("xfer", 0), ("complete",), ("reclaim",)]


def run_seq(seq, n_slabs=3):
    p = SlabPool(n_slabs * SLAB, SLAB)
    live, order, tag, xfers = {}, [], 0, []
    for op in seq:
        if op[0] == "alloc":
            if do_alloc(p, op[1], op[2], live, tag) is not None:
                order.append(tag)
            tag += 1
        elif op[0] == "free":
            if not order:
                continue
            t = order.pop(op[1])
            hs = live.pop(t)
            busy = {h for x, bs in p.touch.items() if x not in p.done for h in bs}
            p.free(hs)
            for h in hs:
                # I3: the block went back to its own slab: not owned; quarantined iff busy
                assert h[1] not in p.owned[h[0]]
                assert (h in p.quarantine) == (h in busy)
        elif op[0] == "xfer":
            if not order:
                continue
            xfers.append(p.begin(live[order[op[1]]]))
        elif op[0] == "complete":
            if xfers:
                p.complete(xfers.pop(0))
        elif op[0] == "reclaim":
            q_before = dict(p.quarantine)
            p.reclaim()
            # step ⑧: exactly the move-list blocks whose transfers completed are released
            for b, xs in q_before.items():
                assert (b in p.quarantine) == (not xs <= p.done)
        check_invariants(p, live)
    return p


def test_exhaustive_sequences_len4():
    n = 0
    for seq in itertools.product(OPS, repeat=4):
        run_seq(seq)
        n += 1
    assert n == len(OPS) ** 4


@pytest.mark.parametrize("seed", range(60))
def test_random_long_sequences(seed):
    r = random.Random(seed)
    run_seq([r.choice(OPS) for _ in range(60)], n_slabs=4)


def test_move_list_blocks_skipped_until_reclaimed():
    """blocks of an ongoing transfer, once freed, sit in the move list and
    are neglected by allocation until the daemon reclaims them after completion (Ry example,
    PAPER.md:1497-1502)."""
    p = SlabPool(2 * SLAB, SLAB)
    ry = p.alloc(A, 2)                 # Ry's CPU blocks
    x = p.begin(ry)                    # C->D transfer of Ry in flight
    p.free(ry)                         # Ry swapped to another instance: blocks freed ...
    assert set(ry) <= set(p.quarantine)
    r1 = p.alloc(A, 2)                 # ... but R1's allocation avoids them
    assert not set(r1) & set(ry)
    p.complete(x)
    assert p.reclaim() == 2
    p.free(r1)
    assert p.alloc(A, 2) == sorted(ry)


def test_slab_reclaim_and_reassignment():
    p = SlabPool(2 * SLAB, SLAB)
    a = p.alloc(A, 2)
    assert p.shape[0] == A
    p.free(a)
    assert p.shape[0] is None          # empty slab reclaimed
    b = p.alloc(Bsh, 2)                # now free for another shape
    assert [s for s, _ in b] == [0, 1]


def test_errors_and_all_or_nothing():
    p = SlabPool(2 * SLAB, SLAB)
    a = p.alloc(A, 3)
    with pytest.raises(AllocError) as e:
        p.alloc(Bsh, 1)                # only one unassigned slab left? no: slab1 holds A
    assert e.value.code == OOM
    with pytest.raises(AllocError) as e:
        p.free([a[0], a[0]])           # duplicate
    assert e.value.code == STATE
    assert p.owner_count() == 3
    big = KVShape(L=3, H=2, D=2, s=2, B=8)
    with pytest.raises(AllocError) as e:
        p.alloc(big, 1)                # block larger than a slab
    assert e.value.code == INVALID
    p.free(a)
    with pytest.raises(AllocError) as e:
        p.free(a[:1])                  # double free
    assert e.value.code in (STATE, INVALID)


def test_fragmentation_metric_hand_trace():
    """Fig. 16's metric, "unused memory to peak allocated memory", on a
    4-step trace whose values are worked out by hand from that definition (slab 256 B; A blocks
    128 B, two per slab; Bsh blocks 192 B, one per slab)."""
    p = SlabPool(4 * SLAB, SLAB)
    a = p.alloc(A, 1)        # assigned 256, used 128, peak 256 -> 128/256
    assert p.fragmentation() == pytest.approx(0.5)
    p.alloc(Bsh, 1)          # assigned 512, used 320, peak 512 -> 192/512
    assert p.fragmentation() == pytest.approx(0.375)
    p.free(a)                # A's slab reclaimed: assigned 256, used 192, peak stays 512 -> 64/512
    assert p.fragmentation() == pytest.approx(0.125)
    assert p.unused_over_assigned() == pytest.approx(0.25)       # the current-denominator figure
    p.alloc(A, 2)            # slab 0 back for A, full: assigned 512, used 448, peak 512 -> 64/512
    assert p.fragmentation() == pytest.approx(0.125)
    # per shape: A peaked at 256 B (one slab) and now fills it; Bsh peaked at 256 B, uses 192
    assert p.fragmentation(A) == pytest.approx(0.0)
    assert p.fragmentation(Bsh) == pytest.approx(64 / 256)


def test_fragmentation_empty_pool_and_slab_tail():
    p = SlabPool(4 * SLAB, SLAB)
    assert p.fragmentation() == 0.0
    C3 = KVShape(L=1, H=1, D=5, s=2, B=8)     # chunk = block = 2*1*5*2*8 = 160 B -> 1 per slab, 96 B tail
    c = p.alloc(C3, 1)
    assert p.fragmentation() == pytest.approx(96 / 256)
    b = p.alloc(Bsh, 2)      # assigned 768 (peak), used 160 + 384
    assert p.fragmentation() == pytest.approx((768 - 544) / 768)
    p.free(b)
    p.free(c)                # everything reclaimed: assigned 0, peak 768
    assert p.fragmentation() == 0.0
    p.alloc(A, 1)            # assigned 256, used 128; the peak is still 768 -> 128/768
    assert p.fragmentation() == pytest.approx(128 / 768)


def test_zero_block_request_is_a_no_op():
    """An empty request (an instance with nothing to move) allocates nothing, claims no slab and is
    not an error (include/aeg.h aeg_kv_alloc: "n == 0 is a no-op"); a negative count is invalid."""
    sh = KVShape(2, 4, 64, 2, 16)
    p = SlabPool(8 * sh.block_bytes() * 4, 8 * sh.block_bytes())
    assert p.alloc(sh, 0) == []
    per, free = p.stats()
    assert per == {} and free == p.n_slabs
    with pytest.raises(AllocError) as e:
        p.alloc(sh, -1)
    assert e.value.code == INVALID
