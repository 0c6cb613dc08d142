"""Pure-Python twins of the oracle for tiny inputs -- TEST INFRASTRUCTURE ONLY.

brute(R, Q, L): the MEM definition checked cell by cell:
    (r, q, lam) with R[r+i] == Q[q+i] for i < lam, lam >= L,
    (r == 0 or q == 0 or R[r-1] != Q[q-1])        -- left-maximal (end = mismatch, reading R3)
    (r+lam == |R| or q+lam == |Q| or R[r+lam] != Q[q+lam])  -- right-maximal
  enumerated over every start cell (r, q): O(|R||Q| * lam). Independent of the
  C++ brute force (which walks diagonals).

sampled(R, Q, L, ls, step): the paper's method in its own words
  (index every step-th ls-mer of R, look up every query position, extend both
  ways, keep >= L, deduplicate) with a dict -- the Python twin of oracle_mems.

homopolymer(n, m, L): closed form for R = A^n, Q = A^m:
  every MEM touches a sequence start on one side and an end on the other:
  {(0, q, min(n, m-q)) : q < m} U {(r, 0, min(n-r, m)) : 1 <= r < n}, lam >= L.
"""
from __future__ import annotations


def _s(x):
    if isinstance(x, (bytes, bytearray)):
        x = x.decode("ascii")
    elif not isinstance(x, str):
        x = bytes(x).decode("ascii")
    return x.upper()


def brute(R, Q, L):
    R, Q = _s(R), _s(Q)
    out = []
    for r in range(len(R)):
        for q in range(len(Q)):
            if r > 0 and q > 0 and R[r - 1] == Q[q - 1]:
                continue  # not left-maximal
            lam = 0
            while r + lam < len(R) and q + lam < len(Q) and R[r + lam] == Q[q + lam]:
                lam += 1
            # (r+lam, q+lam) is now an end or a mismatch: right-maximal by construction
            if lam >= L:
                out.append((r, q, lam))
    return sorted(out)


def sampled(R, Q, L, ls, step=None):
    R, Q = _s(R), _s(Q)
    if step is None:
        step = L - ls + 1
    H = {}
    for p in range(0, len(R) - ls + 1, step):
        H.setdefault(R[p:p + ls], []).append(p)
    found = set()
    for q in range(0, len(Q) - ls + 1):
        for p in H.get(Q[q:q + ls], ()):
            a = 0
            while a < p and a < q and R[p - a - 1] == Q[q - a - 1]:
                a += 1
            b = ls
            while p + b < len(R) and q + b < len(Q) and R[p + b] == Q[q + b]:
                b += 1
            if a + b >= L:
                found.add((p - a, q - a, a + b))
    return sorted(found)


def homopolymer(n, m, L):
    out = {(0, q, min(n, m - q)) for q in range(m)}
    out |= {(r, 0, min(n - r, m)) for r in range(1, n)}
    return sorted(t for t in out if t[2] >= L and t[2] > 0)


def mums(R, Q, L):
    """MEMs (by the definition) whose string occurs exactly once in R and in Q."""
    R, Q = _s(R), _s(Q)

    def count(T, S):
        return sum(1 for i in range(len(T) - len(S) + 1) if T[i:i + len(S)] == S)

    return [t for t in brute(R, Q, L) if count(R, R[t[0]:t[0] + t[2]]) == 1 and count(Q, R[t[0]:t[0] + t[2]]) == 1]


def rare(R, Q, L, k):
    """MEMs (by the definition) whose string occurs at most k times in R and in Q."""
    R, Q = _s(R), _s(Q)

    def count(T, S):
        return sum(1 for i in range(len(T) - len(S) + 1) if T[i:i + len(S)] == S)

    return [t for t in brute(R, Q, L) if count(R, R[t[0]:t[0] + t[2]]) <= k and count(Q, R[t[0]:t[0] + t[2]]) <= k]


def fasta(text):
    """Records [(name, sequence)] of a multi-FASTA text (name = first word of the header)."""
    text = text.decode() if isinstance(text, (bytes, bytearray)) else text
    out = []
    for block in text.split(">")[1:]:
        head, _, body = block.partition("\n")
        out.append((head.split()[0] if head.split() else "", "".join(body.split())))
    return out


def multi_brute(R_text, Q_text, L):
    """MEMs of multi-FASTA inputs by the definition (R24): for every pair of
    records, every diagonal walked base by base; a position matches when both bases are
    in ACGT (either case) and equal; maximal runs of length >= L. Sorted
    (r_record, r_pos, q_record, q_pos, len), 0-based positions inside the records."""
    out = []
    R, Q = fasta(R_text), fasta(Q_text)
    for ri, (_, r) in enumerate(R):
        r = r.upper()
        for qi, (_, q) in enumerate(Q):
            q = q.upper()
            for d in range(-len(q) + 1, len(r)):
                i, j, run = max(d, 0), max(-d, 0), 0
                while i < len(r) and j < len(q):
                    if r[i] == q[j] and r[i] in "ACGT":
                        run += 1
                    else:
                        if run >= L:
                            out.append((ri, i - run, qi, j - run, run))
                        run = 0
                    i += 1
                    j += 1
                if run >= L:
                    out.append((ri, i - run, qi, j - run, run))
    return sorted(out)
