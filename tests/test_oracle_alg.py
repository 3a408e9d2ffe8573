"""Pins for the step oracles in oracle/alg.py (Alg. 1, Alg. 2, Alg. 3, pool estimate,
canonical segments) against the paper's printed worked example, Table 3, brute force
and definitions.  CPU only."""
import json
import os
import random

import numpy as np
import pytest

from oracle import alg

GOLD = os.path.join(os.path.dirname(__file__), "golden")


# ------------------------------------------------------------------ Alg. 1 --

def _brute_row_of(row_ptr, nz):
    for r in range(len(row_ptr) - 1):
        if row_ptr[r] <= nz < row_ptr[r + 1]:
            return r
    raise AssertionError


@pytest.mark.parametrize("seed", range(20))
def test_alg1_definition(seed):
    rng = random.Random(seed)
    rows = rng.randint(1, 60)
    lens = [0 if rng.random() < 0.3 else rng.randint(1, 40) for _ in range(rows)]
    rp = [0]
    for L in lens:
        rp.append(rp[-1] + L)
    npb = rng.choice([1, 2, 3, 8, 16, 512])
    got = alg.alg1_block_row_starts(rp, npb)
    nblocks = -(-rp[-1] // npb)
    assert len(got) == nblocks
    for b in range(nblocks):
        assert got[b] == _brute_row_of(rp, b * npb)


def test_alg1_empty_rows_and_base():
    # leading/trailing empty rows: reading R4 (skip a == b)
    rp = [0, 0, 0, 3, 3, 7, 7]
    assert alg.alg1_block_row_starts(rp, 2) == [2, 2, 4, 4]
    # segment base: blocks counted from nonzero 5 (absolute row_ptr values)
    rp2 = [5, 5, 9, 12]
    assert alg.alg1_block_row_starts(rp2, 3, nnz_base=5) == [1, 1, 2]
    assert alg.alg1_block_row_starts([0, 0, 0], 4) == []


# ------------------------------------------------------------------ Alg. 2 --

def test_alg2_fig3_worked_example():
    g = json.load(open(os.path.join(GOLD, "fig3_work_distribution.json")))
    wd = alg.WorkDistribution(len(g["lengths"]))
    wd.placework(g["lengths"])
    assert wd.size() == sum(g["lengths"])
    for draw, pairs, rem in zip(g["draws"], g["pairs"], g["remaining_after"]):
        A, Bv = wd.receivework(draw)
        assert [[a, b] for a, b in zip(A, Bv)] == pairs
        assert wd.remaining() == rem
    # the paper-printed row after the first draw
    wd2 = alg.WorkDistribution(6)
    wd2.placework(g["lengths"])
    wd2.receivework(10)
    assert wd2.remaining() == g["remaining_printed_by_paper"]["after_draw_1"]


@pytest.mark.parametrize("seed", range(25))
def test_alg2_enumerates_every_product_once(seed):
    """Brute force: draining the distribution with arbitrary draws yields every
    (entry, offset) exactly once; each draw takes a contiguous top range of each
    entry's remaining offsets (rows are drained from their end, L210)."""
    rng = random.Random(seed)
    npb = rng.choice([1, 4, 7, 16, 64])
    lens = [rng.choice([0, 0, 1, 2, 5, 17, 40]) for _ in range(npb)]
    wd = alg.WorkDistribution(npb)
    wd.placework(lens)
    seen = set()
    rem = list(lens)
    while wd.size() > 0:
        consume = min(wd.size(), rng.randint(1, 30))
        A, Bv = wd.receivework(consume)
        assert len(A) == consume
        assert A == sorted(A)                       # products ordered by entry
        for e in set(A):
            offs = [b for a, b in zip(A, Bv) if a == e]
            assert offs == list(range(rem[e] - 1, rem[e] - 1 - len(offs), -1))
            rem[e] -= len(offs)
        for a, b in zip(A, Bv):
            assert (a, b) not in seen and 0 <= b < lens[a]
            seen.add((a, b))
        assert wd.remaining() == rem
    assert len(seen) == sum(lens)


def test_alg2_restart_replay():
    """Restart: "we execute line 36 with the stored count" (L254) reproduces the
    state reached by drawing that many products."""
    lens = [3, 0, 9, 4, 4, 1, 12]
    a = alg.WorkDistribution(7)
    a.placework(lens)
    a.receivework(6)
    a.receivework(5)
    b = alg.WorkDistribution(7)
    b.placework(lens)
    b.consume_only(11)
    assert a.WDState == b.WDState


# ------------------------------------------------------------------ Alg. 3 --

def _random_sorted_stream(rng, n, int_values):
    rows = sorted(rng.randint(0, 6) for _ in range(n))
    items = []
    for r in rows:
        items.append((r, rng.randint(0, 5)))
    items.sort()
    keys = [(r, c) for r, c in items]
    rws = [r for r, _ in items]
    vals = [float(rng.randint(-5, 5)) if int_values else rng.uniform(-1, 1) for _ in items]
    return rws, keys, vals


@pytest.mark.parametrize("seed", range(40))
def test_alg3_against_bruteforce(seed):
    rng = random.Random(seed)
    n = rng.randint(1, 60)
    rows, keys, vals = _random_sorted_stream(rng, n, int_values=False)
    out = alg.compaction_scan(rows, keys, vals)
    run_idx = -1
    row_runs = {}
    for i in range(n):
        run_end = i == n - 1 or keys[i + 1] != keys[i]
        row_end = i == n - 1 or rows[i + 1] != rows[i]
        re_, cc, rowe, rc = alg.decode_state(out[i][3])
        assert re_ == int(run_end) and rowe == int(row_end)
        if run_end:
            run_idx += 1
            row_runs[rows[i]] = row_runs.get(rows[i], 0) + 1
            start = i
            while start > 0 and keys[start - 1] == keys[i]:
                start -= 1
            s = 0.0
            for v in vals[start:i + 1]:
                s += v
            assert out[i][2] == s                    # sequential segmented sum, exact
            assert cc == run_idx + 1                 # position in chunk (1-based)
            assert rc == row_runs[rows[i]]           # position in row (1-based)


@pytest.mark.parametrize("seed", range(40))
def test_alg3_tree_equals_sequential(seed):
    """Associativity: a Hillis-Steele tree gives the same states, and the same values
    on integer data (reading R6)."""
    rng = random.Random(100 + seed)
    rows, keys, vals = _random_sorted_stream(rng, rng.randint(1, 80), int_values=True)
    seq = alg.compaction_scan(rows, keys, vals)
    tree = alg.compaction_scan_tree(rows, keys, vals)
    assert [s[3] for s in seq] == [t[3] for t in tree]
    assert [s[2] for s in seq] == [t[2] for t in tree]


def test_alg3_literal_transcript_masks_are_wrong():
    """Documents reading R6: with the masks as printed in the transcript the row
    counter is not reset at a new row."""
    def literal(a, b):
        arow, akey, aval, astate = a
        brow, bkey, bval, bstate = b
        state = (astate & 0xFFFE) if arow == brow else (astate & 0xFFFEFFFE)
        return (brow, bkey, aval + bval if akey == bkey else bval, (state + bstate) & 0xFFFFFFFF)
    rows, keys, vals = [0, 0, 1, 1], [(0, 0), (0, 1), (1, 0), (1, 1)], [1.0, 1.0, 1.0, 1.0]
    st = alg.compaction_initial_states(rows, keys)
    acc, lit = None, []
    for i in range(4):
        e = (rows[i], keys[i], vals[i], st[i])
        acc = e if acc is None else literal(acc, e)
        lit.append(acc)
    ok = alg.compaction_scan(rows, keys, vals)
    assert [alg.decode_state(s[3])[3] for s in ok] == [1, 2, 1, 2]
    assert [alg.decode_state(s[3])[3] for s in lit] != [1, 2, 1, 2]


# ---------------------------------------------------------- pool estimate --

def test_pool_estimate_table3():
    g = json.load(open(os.path.join(GOLD, "table3_pool.json")))
    for m in g["matrices"]:
        nA, mA, nnz = m["rows"], m["cols"], m["nnz"]
        if m["transpose"]:
            nB, mB = mA, nA              # B = Aᵀ
        else:
            nB, mB = nA, mA
        mb = alg.pool_estimate_bytes(nA, nnz, nB, mB, nnz, g["value_bytes"]) / 1e6
        assert abs(mb - m["table3_pool_mb"]) <= g["tolerance_rel"] * m["table3_pool_mb"], m["name"]


def test_pool_estimate_closed_form_limits():
    # p_b -> 0 limit: S -> n_A · a · b (no collisions)
    S = alg.pool_estimate_elements(1000, 5000, 10**12, 10**12, 3 * 10**12)
    assert abs(S - 1000 * 5 * 3) / (1000 * 5 * 3) < 1e-6
    # dense B rows (p_b = 1): S = n_A · b = n_A · m_B (every column hit)
    assert alg.pool_estimate_elements(10, 20, 40, 40, 1600) == pytest.approx(400)


# ----------------------------------------------------- canonical segments --

@pytest.mark.parametrize("seed", range(10))
def test_canonical_segments_definition(seed):
    rng = np.random.default_rng(seed)
    lens = rng.integers(0, 30, rng.integers(1, 200))
    rp = np.concatenate([[0], np.cumsum(lens)])
    S = 8
    seg = alg.canonical_segments(rp, S)
    nnz = int(rp[-1])
    assert seg[0] == 0 and seg[-1] == len(lens) and len(seg) == S + 1
    for s in range(1, S):
        target = -(-(s * nnz) // S)
        r = seg[s]
        assert r == len(lens) or rp[r] >= target
        assert r == 0 or rp[r - 1] < target
    assert all(seg[i] <= seg[i + 1] for i in range(S))
