"""Pins for the CPU oracle (oracle/): each test checks it against something other
than itself -- hand-worked fixtures, the definition by brute force (two
independent implementations), a closed form, symmetry, ground truth planted by
the generator, and a probabilistic expectation. CPU only."""
import itertools

import numpy as np
import pytest

import oracle
from oracle import pyoracle
from paper_conf_ipps_abu_dolehkac14_b200 import synth
from tests.conftest import read_golden
from tests import invariants

GOLDEN_MEMS = ["w1.txt", "w2.txt", "w3.txt", "w4.txt"]


def as_set(T):
    return {tuple(int(x) for x in t) for t in T}


@pytest.mark.parametrize("name", GOLDEN_MEMS)
def test_golden_examples(name):
    g = read_golden(name)
    R, Q, L, want = g["R"], g["Q"], g["L"], set(g["mem"])
    assert set(pyoracle.brute(R, Q, L)) == want
    assert as_set(oracle.brute(R, Q, L)) == want
    for ls in range(1, L + 1):                       # any admissible seed length
        for step in range(1, L - ls + 2):            # any step allowed by Eq. (1)
            assert as_set(oracle.mems(R, Q, L, ls, step)) == want, (ls, step)
            assert set(pyoracle.sampled(R, Q, L, ls, step)) == want, (ls, step)
    # lowercase input is folded (reading R4)
    assert as_set(oracle.mems(R.lower(), Q, L, 1)) == want


def test_golden_index_w2():
    g = read_golden("w2_index.txt")
    ptrs, locs = oracle.index(g["R"], g["ls"], g["step"])
    assert ptrs.tolist() == g["ptrs"]
    assert locs.tolist() == g["locs"]


def test_canonical_trace_w2():
    """The per-hit decision the GPU takes (left run capped at step, drop when it
    reaches step) reproduces the definition's MEM set on W2."""
    g = read_golden("canonical_trace_w2.txt")
    R, Q, L, ls, step = g["R"], g["Q"], g["L"], g["ls"], g["step"]
    emitted = set()
    for h in g["hit"]:
        p, q, e_want = int(h[0]), int(h[1]), int(h[2])
        assert R[p:p + ls] == Q[q:q + ls]
        e = 0
        while e < step and e < p and e < q and R[p - e - 1] == Q[q - e - 1]:
            e += 1
        assert e == e_want
        if e == step:
            assert h[4] == "drop"
            continue
        f = ls
        while p + f < len(R) and q + f < len(Q) and R[p + f] == Q[q + f]:
            f += 1
        assert f == int(h[3])
        if e + f >= L:
            assert h[4] == "emit" and (p - e, q - e, e + f) == tuple(int(x) for x in h[5:8])
            emitted.add((p - e, q - e, e + f))
        else:
            assert h[4] == "short"
    assert emitted == set(read_golden("w2.txt")["mem"])


@pytest.mark.parametrize("n,m", [(n, m) for n in (1, 2, 5, 13, 24) for m in (1, 3, 8, 24)])
def test_homopolymer_closed_form(n, m):
    R, Q = "A" * n, "A" * m
    for L in (1, 2, 3, 6):
        want = set(pyoracle.homopolymer(n, m, L))
        assert as_set(oracle.brute(R, Q, L)) == want
        assert set(pyoracle.brute(R, Q, L)) == want
        for ls in range(1, L + 1):
            assert as_set(oracle.mems(R, Q, L, ls)) == want


ALPHABETS = [b"A", b"AC", b"ACG", b"ACGT"]


def test_random_tiny_vs_both_brute_forces():
    rng = np.random.default_rng(12345)
    for trial in range(400):
        alpha = ALPHABETS[trial % 4]
        nR, nQ = int(rng.integers(0, 90)), int(rng.integers(0, 90))
        R, Q = synth.random_pair(rng, nR, nQ, alpha)
        L = int(rng.integers(1, 13))
        ls = int(rng.integers(1, min(L, 15) + 1))
        step = int(rng.integers(1, L - ls + 2))
        want = as_set(oracle.brute(R, Q, L))
        assert set(pyoracle.brute(R.tobytes(), Q.tobytes(), L)) == want
        got = oracle.mems(R, Q, L, ls, step)
        assert as_set(got) == want, (trial, alpha, nR, nQ, L, ls, step)
        invariants.check(R, Q, L, got)


def test_swap_symmetry():
    rng = np.random.default_rng(7)
    for trial in range(60):
        R, Q = synth.random_pair(rng, int(rng.integers(1, 300)), int(rng.integers(1, 300)), ALPHABETS[trial % 4])
        L = int(rng.integers(2, 12))
        ls = min(L, 4)
        a = as_set(oracle.mems(R, Q, L, ls))
        b = {(q, r, l) for r, q, l in as_set(oracle.mems(Q, R, L, ls))}
        assert a == b


def test_eq1_coverage():
    """Eq. (1): with step <= L - ls + 1 every MEM of length >= L contains a
    sampled seed start p (p % step == 0, r <= p <= r + len - ls)."""
    rng = np.random.default_rng(3)
    for trial in range(200):
        R, Q = synth.random_pair(rng, 120, 120, ALPHABETS[trial % 4])
        L = int(rng.integers(2, 14))
        ls = int(rng.integers(1, L + 1))
        step = L - ls + 1
        for r, q, lam in oracle.brute(R, Q, L).tolist():
            first = -(-r // step) * step
            assert first <= r + lam - ls


def test_random_mem_expectation():
    """Unrelated iid uniform sequences: E[#MEMs] ~= |R||Q| * 3/4 * 4^-L (a run of
    >= L equal cells preceded by a mismatch). Accept within 4 sigma (Poisson)."""
    rng = np.random.default_rng(2024)
    n, L = 1500, 5
    R, Q = synth.random_pair(rng, n, n)
    got = len(oracle.mems(R, Q, L, 3))
    exp = n * n * 0.75 * 4.0 ** -L
    assert abs(got - exp) < 4 * exp ** 0.5, (got, exp)
    assert got == len(oracle.brute(R, Q, L))


def test_qrange_partition():
    rng = np.random.default_rng(11)
    for trial in range(40):
        R, Q = synth.random_pair(rng, 400, 400, ALPHABETS[1 + trial % 3])
        L, ls = 8, 4
        whole = oracle.mems(R, Q, L, ls)
        cuts = sorted(set([0, 400] + rng.integers(0, 400, 3).tolist()))
        parts = np.concatenate([oracle.mems(R, Q, L, ls, 0, a, b) for a, b in zip(cuts[:-1], cuts[1:])])
        parts = parts[np.lexsort((parts[:, 1], parts[:, 0]))]
        assert np.array_equal(parts, whole)


def test_alphabet_and_args():
    with pytest.raises(oracle.OracleError):
        oracle.mems("ACGN", "ACG", 2, 1)
    with pytest.raises(oracle.OracleError):
        oracle.mems("ACG", "ACG", 2, 3)          # ls > L
    with pytest.raises(oracle.OracleError):
        oracle.mems("ACG", "ACG", 4, 2, step=4)  # step > L - ls + 1 violates Eq. (1)
    assert len(oracle.mems("", "ACGT", 2, 1)) == 0
    assert len(oracle.mems("AC", "A", 2, 2)) == 0


def _code(s):
    v = 0
    for ch in s:
        v = v * 4 + b"ACGT".index(ch)
    return v


@pytest.mark.parametrize("ls,step,n", [(3, 2, 500), (5, 1, 777), (6, 7, 3000), (10, 11, 20000)])
def test_index_invariants(ls, step, n):
    """ptrs/locs per PAPER.md:84: monotone prefix sums, last == |locs|, bucket s
    holds exactly the sampled positions whose seed is s, ascending (step 4)."""
    R = synth.make_pair("c1", scale=n / 100_000).R[:n].tobytes()
    ptrs, locs = oracle.index(R, ls, step)
    n_locs = (len(R) - ls) // step + 1
    assert len(locs) == n_locs and ptrs[-1] == n_locs and ptrs[0] == 0
    assert (np.diff(ptrs.astype(np.int64)) >= 0).all()
    assert sorted(locs.tolist()) == list(range(0, len(R) - ls + 1, step))
    nz = np.flatnonzero(np.diff(ptrs.astype(np.int64)))
    for s in nz:
        seg = locs[ptrs[s]:ptrs[s + 1]]
        assert (np.diff(seg.astype(np.int64)) > 0).all()
        for p in seg[:3]:
            assert _code(R[p:p + ls]) == s


@pytest.mark.slow
def test_c1_full_vs_brute_force_and_planted():
    """Config C1 in full: oracle == brute force over 10^10 cells; every planted
    copy is reported; all invariants hold; output independent of ls / step."""
    P = synth.make_pair("c1")
    want = oracle.brute(P.R, P.Q, P.L)
    got = oracle.mems(P.R, P.Q, P.L, P.ls)
    assert np.array_equal(got, want)
    assert len(got) > 500
    invariants.check(P.R, P.Q, P.L, got)
    s = as_set(got)
    for t in P.planted:
        assert tuple(t) in s
    assert np.array_equal(oracle.mems(P.R, P.Q, P.L, 8), got)
    assert np.array_equal(oracle.mems(P.R, P.Q, P.L, 12, step=5), got)


def test_golden_mums_w2():
    g = read_golden("w2_mums.txt")
    want = set(g["mem"])
    assert set(pyoracle.mums(g["R"], g["Q"], g["L"])) == want
    for ls in (1, 2, 3):
        assert as_set(oracle.mums(g["R"], g["Q"], g["L"], ls)) == want
    assert len(oracle.mums("ACGTACGT", "ACGT", 2, 2)) == 0  # W1: "ACGT" twice in R


def test_mums_random_vs_python_twin():
    rng = np.random.default_rng(77)
    for trial in range(60):
        R, Q = synth.random_pair(rng, int(rng.integers(5, 120)), int(rng.integers(5, 120)), ALPHABETS[trial % 4])
        L = int(rng.integers(2, 10))
        want = set(pyoracle.mums(R.tobytes(), Q.tobytes(), L))
        assert as_set(oracle.mums(R, Q, L, min(L, 3))) == want


def test_golden_rare_w3():
    """Rare MEMs (R23) of the hand-worked W3 fixture at k = 1 and k = 2, both oracles."""
    g = read_golden("w3_rare.txt")
    for k in (1, 2):
        want = set(g[f"k{k}"])
        assert set(pyoracle.rare(g["R"], g["Q"], g["L"], k)) == want
        for ls in (1, 2, 4):
            assert as_set(oracle.rare(g["R"], g["Q"], g["L"], ls, k)) == want
    assert as_set(oracle.rare(g["R"], g["Q"], g["L"], 4, 1)) == as_set(oracle.mums(g["R"], g["Q"], g["L"], 4))


@pytest.mark.parametrize("n,m,L,k", [(30, 20, 5, 1), (30, 20, 5, 3), (25, 25, 4, 7), (12, 40, 2, 15)])
def test_rare_homopolymer_closed_form(n, m, L, k):
    """A^n vs A^m: the MEM of length len has A^len, which occurs n - len + 1 times in R and
    m - len + 1 times in Q; it is rare iff both counts are <= k."""
    want = {t for t in pyoracle.homopolymer(n, m, L) if n - t[2] + 1 <= k and m - t[2] + 1 <= k}
    assert set(pyoracle.rare("A" * n, "A" * m, L, k)) == want
    assert as_set(oracle.rare("A" * n, "A" * m, L, min(L, 3), k)) == want


def test_rare_random_vs_python_twin():
    rng = np.random.default_rng(78)
    for trial in range(60):
        R, Q = synth.random_pair(rng, int(rng.integers(5, 120)), int(rng.integers(5, 120)), ALPHABETS[trial % 4])
        L = int(rng.integers(2, 10))
        k = int(rng.integers(1, 6))
        want = set(pyoracle.rare(R.tobytes(), Q.tobytes(), L, k))
        assert as_set(oracle.rare(R, Q, L, min(L, 3), k)) == want
