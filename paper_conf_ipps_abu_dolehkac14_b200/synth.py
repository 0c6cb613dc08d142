"""Seeded synthetic genome pairs shaped like the paper's workloads.

This module is the ONLY code shared by the CUDA path's tests/bench and the
CPU oracle's tests: it produces input bytes (ASCII A/C/G/T) and the ground
truth of what it planted, and holds none of the MEM method's arithmetic
(no seeds, no sampling, no extension, no encoding used by either side).

Workload recipe: SURVEY.md §8(d) D1-D5, restated in DESIGN.md §"Input recipe".
The paper's own data (Table II, real chromosomes) is not
available offline; these are synthetic stand-ins with the same sizes and the
structure the paper says matters: homologous query (Fig. 4, :210), repeats
that skew seed-bucket sizes (Fig. 6, :268-270) and low-complexity stress for
load balancing (Fig. 7, :276).

Everything is deterministic in (config name, seed, scale).
"""
from __future__ import annotations

import dataclasses
import hashlib

import numpy as np

_ASCII = np.frombuffer(b"ACGT", dtype=np.uint8)
_CHUNK = 1 << 24


@dataclasses.dataclass
class Pair:
    name: str
    R: np.ndarray          # uint8 ASCII
    Q: np.ndarray          # uint8 ASCII
    L: int                 # minimum MEM length (paper's L)
    ls: int                # seed length (paper's l_s)
    planted: list          # [(r, q, length)] exact copies with forced mismatching flanks
    recipe: dict

    def sha256(self):
        return (hashlib.sha256(self.R.tobytes()).hexdigest(),
                hashlib.sha256(self.Q.tobytes()).hexdigest())


# ---------------------------------------------------------------- primitives
# Internal symbol ids 0..3 are just indices into b"ACGT" for this generator.

def random_symbols(rng, n, gc=0.5):
    """iid bases with GC fraction gc, generated in chunks (bounded memory)."""
    out = np.empty(n, dtype=np.uint8)
    # thresholds on a uint16 draw: A,T get (1-gc)/2 each, C,G gc/2 each
    t_a = int(round(65536 * (1 - gc) / 2))
    t_c = t_a + int(round(65536 * gc / 2))
    t_g = t_c + int(round(65536 * gc / 2))
    for s in range(0, n, _CHUNK):
        e = min(n, s + _CHUNK)
        u = rng.integers(0, 65536, e - s, dtype=np.uint32)
        c = np.full(e - s, 3, dtype=np.uint8)          # T
        c[u < t_g] = 2                                  # G
        c[u < t_c] = 1                                  # C
        c[u < t_a] = 0                                  # A
        out[s:e] = c
    return out


def _event_positions(rng, n, rate):
    if n <= 0 or rate <= 0:
        return np.zeros(0, dtype=np.int64)
    k = rng.binomial(n, rate)
    return np.unique(rng.integers(0, n, k, dtype=np.int64))


def substitute(rng, seq, rate):
    """Point substitutions (SNPs) at `rate`, each to a uniformly chosen other base."""
    pos = _event_positions(rng, len(seq), rate)
    seq[pos] = (seq[pos] + rng.integers(1, 4, len(pos), dtype=np.uint8)) & 3
    return seq


def mutate(rng, seq, p_snp, p_indel, mean_indel=3.0):
    """SNPs at p_snp, indels at p_indel (half insertions, half deletions,
    length ~ Geometric(mean mean_indel)). Returns a new array."""
    out = substitute(rng, seq.copy(), p_snp)
    n = len(out)
    ev = _event_positions(rng, n, p_indel)
    if len(ev) == 0:
        return out
    lens = rng.geometric(1.0 / mean_indel, len(ev)).astype(np.int64)
    ins = rng.random(len(ev)) < 0.5
    # deletions: mark [start, start+len) removed
    d0, dl = ev[~ins], lens[~ins]
    delta = np.zeros(n + 1, dtype=np.int32)
    np.add.at(delta, d0, 1)
    np.add.at(delta, np.minimum(d0 + dl, n), -1)
    keep = np.cumsum(delta[:n]) == 0
    # insertions: random bases placed before position ev
    ipos = np.repeat(ev[ins], lens[ins])
    ivals = rng.integers(0, 4, len(ipos), dtype=np.uint8)
    out = np.insert(out, ipos, ivals)
    keep = np.insert(keep, ipos, True)
    return out[keep]


def overwrite_copies(rng, dst, unit, count, divergence):
    """Write `count` diverged copies of `unit` at random offsets of dst (in place)."""
    n, m = len(dst), len(unit)
    if m == 0 or n < m:
        return
    offs = rng.integers(0, n - m + 1, count, dtype=np.int64)
    for o in offs:
        dst[o:o + m] = substitute(rng, unit.copy(), divergence)


def segmental_dups(rng, seq, count, lo, hi, dlo, dhi):
    """Copy `count` segments of length U[lo,hi] within seq at divergence U[dlo,dhi]."""
    n = len(seq)
    for _ in range(count):
        m = int(rng.integers(lo, hi + 1))
        if m >= n:
            continue
        a = int(rng.integers(0, n - m))
        b = int(rng.integers(0, n - m))
        seq[b:b + m] = substitute(rng, seq[a:a + m].copy(), float(rng.uniform(dlo, dhi)))


def _to_sym(b):
    lut = np.full(256, 255, dtype=np.uint8)
    for i, ch in enumerate(b"ACGT"):
        lut[ch] = i
    return lut[np.frombuffer(b, dtype=np.uint8)]


def place(rng, seq, unit, count):
    """Overwrite `count` copies of `unit` (exact) at random offsets of seq."""
    n, m = len(seq), len(unit)
    if n < m:
        return []
    offs = rng.integers(0, n - m + 1, count, dtype=np.int64)
    for o in offs:
        seq[o:o + m] = unit
    return offs.tolist()


def plant_exact(rng, R, Q, count, lo, hi):
    """Copy R[a:a+l] into Q[b:b+l] at non-overlapping Q sites, forcing
    Q[b-1] != R[a-1] and Q[b+l] != R[a+l] where those exist.
    Returns the planted (a, b, l) list (ground truth: each is a MEM of R,Q
    provided no later edit touches Q[b-1 .. b+l])."""
    nR, nQ = len(R), len(Q)
    out = []
    if nQ < 2 * hi + 2 or nR < hi + 2:
        return out
    slot = nQ // count
    for i in range(count):
        l = int(rng.integers(lo, hi + 1))
        if slot < l + 2:
            break
        a = int(rng.integers(0, nR - l + 1))
        b = i * slot + 1 + int(rng.integers(0, slot - l - 1))
        Q[b:b + l] = R[a:a + l]
        if b > 0 and a > 0 and Q[b - 1] == R[a - 1]:
            Q[b - 1] = (R[a - 1] + 1) & 3
        if b + l < nQ and a + l < nR and Q[b + l] == R[a + l]:
            Q[b + l] = (R[a + l] + 1) & 3
        out.append((a, b, l))
    return out


def to_ascii(sym):
    return _ASCII[sym]


# ---------------------------------------------------------------- configs
# (L, ls) per BASELINE.json configs; ls=13 for C4/C5 per SURVEY.md §8 (paper's
# setting for all large pairs, Table III/IV captions PAPER.md:230, :245).
CONFIG_PARAMS = {
    "c1": (20, 10), "c2": (20, 12), "c3": (50, 13), "c4": (100, 13),
    "c5_l20": (20, 13), "c5_l50": (50, 13), "c5_l100": (100, 13), "c5_l300": (300, 13),
}
CONFIG_SEED = {"c1": 1, "c2": 2, "c3": 3, "c4": 4}


def _sc(x, scale, minimum=1):
    return max(minimum, int(round(x * scale)))


def make_c1(scale=1.0, seed=1):
    rng = np.random.default_rng(seed)
    n = _sc(100_000, scale, 400)
    R = random_symbols(rng, n, 0.5)
    Q = mutate(rng, R, 0.01, 0.0)
    motifs = [("AC", 25), ("AAT", 30), ("AG", 25), ("CAG", 20), ("TTA", 22),
              ("GT", 28), ("ACGT", 15), ("A", 60), ("TC", 26), ("GGC", 18)]
    for mo, c in motifs[:_sc(10, scale)]:
        u = _to_sym(bytes(mo, "ascii") * c)
        place(rng, R, u, 1)
        place(rng, Q, u, 1)
    planted = plant_exact(rng, R, Q, _sc(20, scale), 20, 200)
    return R, Q, planted, dict(n=n, snp=0.01, indel=0.0, planted=len(planted), tandem=len(motifs))


def make_c2(scale=1.0, seed=2):
    rng = np.random.default_rng(seed)
    n = _sc(5_000_000, scale, 1000)
    R = random_symbols(rng, n, 0.5)
    Q = mutate(rng, R, 0.045, 0.005)
    return R, Q, [], dict(n=n, snp=0.045, indel=0.005)


def make_c3(scale=1.0, seed=3):
    rng = np.random.default_rng(seed)
    n = _sc(50_000_000, scale, 20_000)
    R = random_symbols(rng, n, 0.41)
    fam_a = random_symbols(rng, 300, 0.41)
    fam_b = random_symbols(rng, 6000, 0.41)
    overwrite_copies(rng, R, fam_a, _sc(5000, scale), 0.12)
    overwrite_copies(rng, R, fam_b, _sc(300, scale), 0.08)
    segmental_dups(rng, R, _sc(200, scale), 10_000 if n > 1_000_000 else 500, 100_000 if n > 1_000_000 else 2_000, 0.01, 0.04)
    Q = mutate(rng, R, 0.01, 0.001)
    segmental_dups(rng, Q, _sc(50, scale), 10_000 if n > 1_000_000 else 500, 100_000 if n > 1_000_000 else 2_000, 0.01, 0.04)
    return R, Q, [], dict(n=n, gc=0.41, fam=[(300, 5000, 0.12), (6000, 300, 0.08)], sd=200, snp=0.01,
                          indel=0.001, q_sd=50)


def make_c4(scale=1.0, seed=4):
    rng = np.random.default_rng(seed)
    n = _sc(250_000_000, scale, 40_000)
    R = random_symbols(rng, n, 0.41)
    fam_a = random_symbols(rng, 300, 0.41)      # Alu-like
    fam_b = random_symbols(rng, 6000, 0.41)     # L1-like
    overwrite_copies(rng, R, fam_a, _sc(20_000, scale), 0.20)
    overwrite_copies(rng, R, fam_b, _sc(1000, scale), 0.15)
    big = n > 5_000_000
    segmental_dups(rng, R, _sc(500, scale), 10_000 if big else 500, 200_000 if big else 4_000, 0.01, 0.03)
    # Q: syntenic blocks of 1-10 Mbp (scaled) taken from R in order, ~60% of R
    target = int(0.6 * n)
    blo, bhi = (1_000_000, 10_000_000) if big else (max(200, n // 200), max(400, n // 25))
    pieces, pos, got = [], 0, 0
    while got < target and pos < n:
        m = int(rng.integers(blo, bhi + 1))
        gap = int(rng.integers(0, max(1, int(m * 0.66))))
        a = pos + gap
        if a >= n:
            break
        m = min(m, n - a, target - got)
        pieces.append(mutate(rng, R[a:a + m], 0.012, 0.002))
        got += m
        pos = a + m
    Q = np.concatenate(pieces) if pieces else R[:1].copy()
    # low-complexity stress, inserted into R after Q is derived
    na = _sc(1000, scale)
    for _ in range(na):
        place(rng, R, np.zeros(int(rng.integers(50, 151)), dtype=np.uint8), 1)       # poly-A
        place(rng, R, _to_sym(b"AC" * int(rng.integers(25, 76))), 1)                 # (AC)n
    for _ in range(_sc(10, scale)):
        place(rng, Q, np.zeros(int(rng.integers(50, 151)), dtype=np.uint8), 1)
        place(rng, Q, _to_sym(b"AC" * int(rng.integers(25, 76))), 1)
    return R, Q, [], dict(n_R=n, n_Q=len(Q), gc=0.41, famA=(300, 20000, 0.20), famB=(6000, 1000, 0.15),
                          sd=500, synteny=0.6, snp=0.012, indel=0.002, lowcx_R=2 * na)


_MAKERS = {"c1": make_c1, "c2": make_c2, "c3": make_c3, "c4": make_c4}


def make_pair(name, scale=1.0, seed=None):
    """Return the Pair for config `name` ('c1'..'c4', 'c5_l20/50/100/300').
    `scale` shrinks every count/length of the recipe (tests use small scales)."""
    L, ls = CONFIG_PARAMS[name]
    base = "c4" if name.startswith("c5") else name
    s = CONFIG_SEED[base] if seed is None else seed
    R, Q, planted, recipe = _MAKERS[base](scale=scale, seed=s)
    recipe = dict(recipe, config=name, seed=s, scale=scale)
    return Pair(name, to_ascii(R), to_ascii(Q), L, ls, planted, recipe)


def random_pair(rng, nR, nQ, alphabet=b"ACGT"):
    """Tiny random pairs for property tests over a restricted alphabet."""
    a = np.frombuffer(alphabet, dtype=np.uint8)
    return a[rng.integers(0, len(a), nR)], a[rng.integers(0, len(a), nQ)]
