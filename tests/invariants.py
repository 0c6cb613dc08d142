"""Soundness invariants every MEM output must satisfy (SURVEY.md §8(c) C4 row
"Soundness invariants"), straight from the definition PAPER.md:53-56:
exact match, left- and right-maximal (or touching an end), len >= L, sorted by
(r, q), no duplicate (r, q), and no two triples on one diagonal overlapping or
abutting (a mismatch or an end must separate maximal runs). Vectorised, O(sum len).
"""
import numpy as np


def _upper(x):
    a = np.frombuffer(bytes(x), dtype=np.uint8) if not isinstance(x, np.ndarray) else x.astype(np.uint8)
    return np.where((a >= 97) & (a <= 122), a - 32, a).astype(np.uint8)


def check(R, Q, L, T, batch=1 << 24):
    """Raise AssertionError on the first violated invariant. T: (N,3) [r, q, len]."""
    R, Q = _upper(R), _upper(Q)
    T = np.asarray(T, dtype=np.int64).reshape(-1, 3)
    if len(T) == 0:
        return
    r, q, lam = T[:, 0], T[:, 1], T[:, 2]
    assert (lam >= L).all(), "len < L"
    assert (r + lam <= len(R)).all() and (q + lam <= len(Q)).all(), "out of range"
    key = r * (1 << 32) + q
    assert (np.diff(key) > 0).all(), "not strictly sorted by (r, q) (unsorted or duplicate)"
    # left maximal
    inner = (r > 0) & (q > 0)
    assert (R[r[inner] - 1] != Q[q[inner] - 1]).all(), "not left-maximal"
    # right maximal
    e_r, e_q = r + lam, q + lam
    inner = (e_r < len(R)) & (e_q < len(Q))
    assert (R[e_r[inner]] != Q[e_q[inner]]).all(), "not right-maximal"
    # exact match, batched over total length
    cs = np.cumsum(lam)
    start = 0
    while start < len(T):
        base = cs[start - 1] if start else 0
        stop = int(np.searchsorted(cs, base + batch, side="right"))
        stop = max(stop, start + 1)
        l = lam[start:stop]
        off = np.arange(int(l.sum()), dtype=np.int64) - np.repeat(np.cumsum(l) - l, l)
        ri = np.repeat(r[start:stop], l) + off
        qi = np.repeat(q[start:stop], l) + off
        assert (R[ri] == Q[qi]).all(), "not an exact match"
        start = stop
    # same diagonal: sorted by (d, r), consecutive runs must be separated by >= 1
    d = r - q
    o = np.lexsort((r, d))
    dd, rr, ll = d[o], r[o], lam[o]
    same = dd[1:] == dd[:-1]
    assert (rr[1:][same] > rr[:-1][same] + ll[:-1][same]).all(), "overlapping/abutting on a diagonal"
