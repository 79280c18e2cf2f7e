"""Pins for O10 (oracle/rules.py): the Fig. 10 scenario replayed as
a log of Table 2 primitives passes; removing any one of the synchronisations the paper describes
makes the checker name the rule that breaks."""
import pytest

from oracle.rules import RuleViolation, check

R1_DEV_P = [("P", b, l) for b in range(2) for l in range(2)]     # R1's blocks on the prefill GPU
R1_CPU = [("C", b, l) for b in range(2) for l in range(2)]       # R1's blocks in the CPU cache
R1_DEV_D = [("D", b, l) for b in range(2) for l in range(2)]     # R1's blocks on the decode GPU
RY_CPU = [("C", b, l) for b in range(2, 4) for l in range(2)]


def fig10_log(skip=None):
    log = [
        ("op", "P.default", "prefill{R1}", [], R1_DEV_P),
        ("record", "P.default", "ev_prefill"),
        ("wait", "P.kvout", "ev_prefill"),
        # ① record + ② memcpy P->C on the KV-Out stream
        ("op", "P.kvout", "P->C R1", R1_DEV_P, R1_CPU),
        ("record", "P.kvout", "ev_out_R1"),
        # ③ decode instance waits on R1's swap-out event before swap-in
        ("wait", "D.kvin", "ev_out_R1"),
        # ④ record + ⑤ memcpy C->D
        ("op", "D.kvin", "C->D R1", R1_CPU, R1_DEV_D),
        ("record", "D.kvin", "ev_in_R1"),
        # ⑥ query + ⑦ forward: the default stream waits on R1's swap-in event
        ("wait", "D.default", "ev_in_R1"),
        ("use", "D.default", R1_DEV_D),
    ]
    if skip == "③":
        log = [e for e in log if e != ("wait", "D.kvin", "ev_out_R1")]
    if skip == "⑥":
        log = [e for e in log if e != ("wait", "D.default", "ev_in_R1")]
    if skip == "wait-before-record":
        i = log.index(("wait", "D.kvin", "ev_out_R1"))
        j = log.index(("record", "P.kvout", "ev_out_R1"))
        log[i], log[j] = log[j], log[i]
        # move the wait ahead of the op it must capture
        log.remove(("wait", "D.kvin", "ev_out_R1"))
        log.insert(3, ("wait", "D.kvin", "ev_out_R1"))
    return log


def test_fig10_correct_log_passes():
    assert check(fig10_log())


def test_missing_wait_breaks_rule2():
    with pytest.raises(RuleViolation, match="❷"):
        check(fig10_log("③"))


def test_missing_query_breaks_rule1():
    with pytest.raises(RuleViolation, match="❶"):
        check(fig10_log("⑥"))


def test_wait_before_record_captures_nothing():
    with pytest.raises(RuleViolation):
        check(fig10_log("wait-before-record"))


def ry_log(move_list: bool):
    """Ry's CPU blocks are being read by a C->D transfer to another decode instance when Ry is
    freed; R1's swap-out must not write into them before that transfer ends (rule ❸)."""
    target = R1_CPU if move_list else RY_CPU[:4]
    return [
        ("op", "D2.kvin", "C->D Ry", RY_CPU, [("D2", b, l) for b in range(2) for l in range(2)]),
        ("record", "D2.kvin", "ev_in_Ry"),
        ("op", "P.kvout", "P->C R1", R1_DEV_P, target),
    ]


def test_move_list_prevents_rule3_violation():
    assert check(ry_log(move_list=True))
    with pytest.raises(RuleViolation, match="❸"):
        check(ry_log(move_list=False))


def test_daemon_sync_orders_reuse():
    """After the daemon observes ev_in_Ry complete (step ⑧), reusing Ry's blocks is ordered."""
    log = ry_log(move_list=False)
    log.insert(2, ("sync", "ev_in_Ry"))
    assert check(log)


def test_per_layer_granularity():
    """Swap-in of layer l waits only on swap-out ev[l] (reading 12) — still rule-correct."""
    log = []
    for l in range(2):
        log += [("op", "out", f"out l{l}", [("D", 0, l)], [("C", 0, l)]), ("record", "out", f"o{l}")]
    for l in range(2):
        log += [("wait", "in", f"o{l}"), ("op", "in", f"in l{l}", [("C", 0, l)], [("D", 1, l)]),
                ("record", "in", f"i{l}")]
    for l in range(2):
        log += [("wait", "dec", f"i{l}"), ("use", "dec", [("D", 1, l)])]
    assert check(log)
    # consumer of layer 1 waiting only on layer 0's event is early
    bad = [e for e in log if e != ("wait", "dec", "i1")]
    with pytest.raises(RuleViolation, match="❶"):
        check(bad)


def test_record_captures_only_its_own_stream():
    """Table 2: cudaEventRecord captures "the current work in stream" — not other streams' work."""
    ok = [("op", "A", "wA", [], ["x"]), ("op", "B", "wB", [], ["y"]), ("record", "A", "e"),
          ("wait", "C", "e"), ("use", "C", ["x"])]
    assert check(ok)
    bad = [("op", "A", "wA", [], ["x"]), ("op", "B", "wB", [], ["y"]), ("record", "B", "e"),
           ("wait", "C", "e"), ("use", "C", ["x"])]
    with pytest.raises(RuleViolation, match="❶"):
        check(bad)


def test_ordering_is_transitive_through_another_stream():
    """Table 2: a wait orders all future work of a stream after the captured work, so an order
    established through an intermediate stream (P -> S -> D, no direct P -> D wait) holds: D may read
    what P wrote.  Without the middle link the same read breaks rule ❷."""
    cells = [("C", 0, 0)]
    log = [
        ("op", "P.kvout", "P->C", [], cells),
        ("record", "P.kvout", "e1"),
        ("wait", "S.aux", "e1"),
        ("op", "S.aux", "unrelated", [], [("X", 0, 0)]),
        ("record", "S.aux", "e2"),
        ("wait", "D.kvin", "e2"),
        ("op", "D.kvin", "C->D", cells, [("D", 0, 0)]),
    ]
    assert check(log)
    with pytest.raises(RuleViolation, match="❷"):
        check([e for e in log if e != ("wait", "S.aux", "e1")])
