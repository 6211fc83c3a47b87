"""Pins for oracle/p2p.py: Alg.1, swap, local merge, Alg.2 (no GPU).

  * the paper's worked examples: Fig.8 and Fig.9,
    tests/golden/fig8.json, fig9.json;
  * Alg.1 against the closed form p = #{i : B[i] < A[s-1-i]} (DESIGN reading Q5,
    an independent derivation), the pivot invariant of P:1635-1640 and
    minimality ("leftmost pivot"), p = 0 when no swap is needed
    (P:1676-1681);
  * Alg.2: g-1 stages, recursive order == staged order, final
    result == library sort (brute force on random duplicate-heavy inputs);
  * swap volume claims: sorted 0, reverse (g-1)*n/2,
    uniform ~ (n/2)(g-1) counted over both directions.
"""
import json
import os

import numpy as np
import pytest

from oracle import p2p

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _load(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


def _arr(rows):
    return [np.array(r, dtype=np.uint32) for r in rows]


def test_fig8():
    fx = _load("fig8.json")
    A, B = _arr(fx["before"])
    p = p2p.select_pivot(A, B)
    assert p == fx["pivot_p"]
    chunks = _arr(fx["before"])
    # swap only (no merge) to check the printed middle row
    c = fx["c"]
    x = p
    sw = [np.concatenate([chunks[0][: c - x], chunks[1][:x]]), np.concatenate([chunks[0][c - x:], chunks[1][x:]])]
    assert [list(s) for s in sw] == fx["after_swap"]
    xs = p2p.swap_and_merge(chunks, 0, 2, p)
    assert xs == [2]
    assert [list(ch) for ch in chunks] == fx["after_merge"]


def test_fig9():
    fx = _load("fig9.json")
    ch = _arr(fx["after_stage1"])
    A, B = p2p.Concat(ch[:2]), p2p.Concat(ch[2:])
    p = p2p.select_pivot(A, B)
    assert p == fx["stage2_pivot_p"]
    # printed swap row: apply the Q6 mapping without merging
    c = fx["c"]
    sw = [x.copy() for x in ch]
    for d in range(2):
        L, R = 1 - d, 2 + d
        x = min(max(p - d * c, 0), c)
        sw[L], sw[R] = np.concatenate([ch[L][: c - x], ch[R][:x]]), np.concatenate([ch[L][c - x:], ch[R][x:]])
    assert [list(s) for s in sw] == fx["stage2_after_swap"]
    xs = p2p.swap_and_merge(ch, 0, 4, p)
    assert xs == [4, 2]
    assert [list(s) for s in ch] == fx["stage2_after_merge"]
    ps = []
    for lo in (0, 2):
        q = p2p.select_pivot(ch[lo], ch[lo + 1])
        ps.append(q)
        p2p.swap_and_merge(ch, lo, lo + 2, q)
    assert ps == fx["stage3_pivots_derived"]
    assert [list(s) for s in ch] == fx["final"]


def _closed_form(A, B):
    s = len(A)
    return sum(1 for i in range(s) if B[i] < A[s - 1 - i])


def _valid(A, B, p):
    """Invariant P:1635-1640 after swapping the last p of A with the first p of B:
    max(new A) <= min(new B)."""
    s = len(A)
    newA = list(A[: s - p]) + list(B[:p])
    newB = list(A[s - p:]) + list(B[p:])
    if not newA or not newB:
        return True
    return max(newA) <= min(newB)


def test_alg1_closed_form_invariant_minimality():
    rng = np.random.default_rng(11)
    for trial in range(20000):
        s = int(rng.integers(1, 9))
        hi = int(rng.integers(1, 6))
        A = np.sort(rng.integers(0, hi, s)).astype(np.uint32)
        B = np.sort(rng.integers(0, hi, s)).astype(np.uint32)
        p = p2p.select_pivot(A, B)
        assert p == _closed_form(A, B)
        assert _valid(A, B, p)
        if p > 0:
            assert not _valid(A, B, p - 1)
        # p is the leftmost valid pivot: no smaller q is valid
        for q in range(p):
            assert not _valid(A, B, q)


def test_alg1_extremes():
    A = np.arange(0, 100, dtype=np.uint32)
    B = np.arange(100, 200, dtype=np.uint32)
    assert p2p.select_pivot(A, B) == 0          # already ordered: no swap
    assert p2p.select_pivot(B, A) == 100        # fully reversed: swap everything
    assert p2p.select_pivot(A, A.copy()) == 50  # #{i : i < 99 - i}
    E = np.full(100, 5, dtype=np.uint32)
    assert p2p.select_pivot(E, E.copy()) == 0   # all ties stay (strict <)


def test_stage_schedule():
    assert p2p.stage_labels(2) == [2]
    assert p2p.stage_labels(4) == [2, 4, 2]
    assert p2p.stage_labels(8) == [2, 4, 2, 8, 2, 4, 2]
    for g in (2, 4, 8, 16):
        st = p2p.stage_schedule(g)
        assert len(st) == g - 1
        for stage in st:
            covered = sorted(i for lo, hi in stage for i in range(lo, hi))
            assert covered == list(range(g))


@pytest.mark.parametrize("g", [2, 4, 8, 16])
def test_alg2_recursive_equals_staged_and_sorts(g):
    rng = np.random.default_rng(g)
    for trial in range(150 if g < 16 else 40):
        c = int(rng.integers(1, 7))
        hi = int(rng.integers(1, 2 * g * c + 2))
        data = rng.integers(0, hi, g * c).astype(np.uint32)
        ch1 = [np.sort(data[i * c:(i + 1) * c]) for i in range(g)]
        ch2 = [x.copy() for x in ch1]
        log = []
        p2p.merge_chunks(ch1, 0, g, log)
        stages = p2p.run_stages(ch2)
        assert np.array_equal(np.concatenate(ch1), np.sort(data))
        assert np.array_equal(np.concatenate(ch2), np.sort(data))
        # the same group operations happen in both orders (multiset of (lo,hi,p,xs))
        rec = sorted((op.lo, op.hi, op.p, tuple(op.xs)) for op in log)
        stg = sorted((op.lo, op.hi, op.p, tuple(op.xs)) for st in stages for op in st)
        assert rec == stg


def test_p2p_sort_padding():
    rng = np.random.default_rng(5)
    for n in (0, 1, 3, 7, 8, 9, 31, 33, 100):
        for g in (1, 2, 4, 8):
            codes = rng.integers(0, 1 << 32, n, dtype=np.uint64).astype(np.uint32)
            codes[: n // 3] = 0xFFFFFFFF      # keys equal to the pad value
            out, _ = p2p.p2p_sort_codes(codes, g)
            assert np.array_equal(out, np.sort(codes))


@pytest.mark.parametrize("g", [2, 4, 8])
def test_swap_volume_claims(g):
    n = g * 4096
    c = n // g
    srt = np.arange(n, dtype=np.uint32)
    _, st = p2p.p2p_sort_codes(srt, g, with_log=True)
    assert p2p.swap_volume(st, g)[0] == 0                       # sorted: no swaps
    _, st = p2p.p2p_sort_codes(srt[::-1].copy(), g, with_log=True)
    tot, _ = p2p.swap_volume(st, g)
    assert tot == (g - 1) * n // 2                              # reverse: worst case
    for s in st:
        for op in s:
            assert all(x == c for x in op.xs)
    rng = np.random.default_rng(9)
    u = rng.integers(0, 1 << 32, n, dtype=np.uint64).astype(np.uint32)
    _, st = p2p.p2p_sort_codes(u, g, with_log=True)
    tot, _ = p2p.swap_volume(st, g)
    both = 2 * tot
    expect = (n / 2) * (g - 1)                                  # P:2164-2170, both directions (reading Q12)
    assert abs(both - expect) / expect < {2: 0.1, 4: 0.1, 8: 0.25}[g] * 2


def test_multiway_splitter_brute_force():
    """NEXT-1 splitters (reading Q15): the first s_r keys of every chunk are
    exactly the k smallest keys of the union; ties go to lower chunks first;
    monotone in k."""
    rng = np.random.default_rng(21)
    for trial in range(400):
        g = int(rng.choice([2, 3, 4, 8]))
        c = int(rng.integers(1, 9))
        hi = int(rng.integers(1, 3 * g * c))
        chunks = [np.sort(rng.integers(0, hi, c)).astype(np.uint32) for _ in range(g)]
        union = np.sort(np.concatenate(chunks))
        prev = [0] * g
        for k in range(g * c + 1):
            s = p2p.multiway_splitter(chunks, k)
            assert sum(s) == k
            taken = np.concatenate([ch[:sr] for ch, sr in zip(chunks, s)])
            assert np.array_equal(np.sort(taken), union[:k])
            assert all(a <= b for a, b in zip(prev, s))
            prev = s
            if 0 < k < g * c:
                v = union[k - 1]
                # a chunk with an untaken key equal to v: no later chunk took a v
                for r in range(g):
                    if s[r] < c and chunks[r][s[r]] == v:
                        assert all(chunks[q][s[q] - 1] != v for q in range(r + 1, g) if s[q] > 0)
        out, _ = p2p.alltoall_sort_chunks(chunks)
        assert np.array_equal(np.concatenate(out), union)
        assert all(len(o) == c for o in out)
