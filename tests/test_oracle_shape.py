"""Pins for O1 (oracle/shape.py) against PAPER.md Table 1 and brute force."""
import os

import numpy as np
import pytest

from oracle.shape import KVShape

GOLD = os.path.join(os.path.dirname(__file__), "golden", "table1_kv_sizes.txt")


def table1():
    rows = []
    for line in open(GOLD):
        if line.startswith("#") or not line.strip():
            continue
        name, L, two, H, D, kb = line.split()
        rows.append((name, int(L), int(two), int(H), int(D), int(kb)))
    return rows


@pytest.mark.parametrize("row", table1(), ids=lambda r: r[0])
def test_table1_token_bytes(row):
    name, L, two, H, D, kb = row
    assert two == 2
    sh = KVShape(L, H, D, 2, 16)
    assert sh.token_bytes() == kb * 1024          # PAPER.md:1120-1128, KB = KiB (reading 20)
    # a block is B tokens, and equals L chunks (reading 2): two independent products agree
    assert sh.block_bytes() == sh.B * sh.token_bytes()
    assert sh.chunk_bytes() * sh.L == sh.block_bytes()


def test_blocks_and_live_tokens_bruteforce():
    sh = KVShape(2, 4, 64, 2, 16)
    for T in range(0, 300):
        nb = sh.blocks_for(T)
        # smallest nb with nb*B >= T
        assert nb * sh.B >= T and (nb == 0 or (nb - 1) * sh.B < T)
        live = [sh.live_tokens(T, j) for j in range(nb + 2)]
        assert sum(live) == T
        assert all(0 <= x <= sh.B for x in live)
        assert all(x == 0 for x in live[nb:])
        assert all(x == sh.B for x in live[: max(0, nb - 1)])


def test_elem_offset_is_nhd_layout():
    sh = KVShape(1, 3, 5, 2, 4)
    # independent formulation: the chunk as a C-ordered array [2][B][H][D][s]
    ref = np.arange(sh.chunk_bytes()).reshape(2, sh.B, sh.H, sh.D, sh.s)
    seen = set()
    for c in range(2):
        for t in range(sh.B):
            for h in range(sh.H):
                for d in range(sh.D):
                    o = sh.elem_offset(c, t, h, d)
                    assert o == ref[c, t, h, d, 0]
                    seen.add(o)
    assert len(seen) == 2 * sh.B * sh.H * sh.D


def test_fig9_and_eq4_context_values():
    """Fig. 9 / §4.2 sizes are consistent with the model recipes (sizes only)."""
    import aeg_inputs as gi
    vals = {}
    for line in open(os.path.join(os.path.dirname(__file__), "golden", "eq4_switch.txt")):
        if line.startswith("#") or not line.strip():
            continue
        k, v = line.split()[:2]
        vals[k] = float(v)
    # 13B at 16-bit is "at least 26 GB"
    assert gi.model_bytes("llama-2-13b") >= vals["lower_bound_13b_bytes_gb"] * 1e9
    assert vals["lower_bound_13b_bytes_gb"] / vals["lower_bound_13b_bw_gbs"] == vals["lower_bound_13b_s"]
    # Fig. 9: "Model Weights (14 GB)" for the 7B example; Llama-7B recipe is 13.48 GB
    assert 13e9 < gi.model_bytes("llama-7b") < 14.5e9
