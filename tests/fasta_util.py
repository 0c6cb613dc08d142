"""Helpers for the multi-FASTA tests: the golden fixture reader, the documented
concatenation layout (R24: records in order, one separator base between
consecutive records) and random multi-FASTA texts."""
import os

import numpy as np

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def read_mummer_golden(name="mummer_multi.txt"):
    sec, out = None, {"R": [], "Q": [], "expect": []}
    L = None
    for line in open(os.path.join(GOLDEN, name)).read().splitlines():
        if line.startswith("#") and sec is None:
            continue
        if line.startswith("L ") and sec is None:
            L = int(line.split()[1])
        elif line in (">R", ">Q", ">expect"):
            sec = line[1:]
        elif sec:
            out[sec].append(line)
    return "\n".join(out["R"]) + "\n", "\n".join(out["Q"]) + "\n", L, "\n".join(out["expect"]) + "\n"


def record_starts(records):
    """Start of every record in the concatenation (one separator base between records)."""
    starts, pos = [], 0
    for _, seq in records:
        starts.append(pos)
        pos += len(seq) + 1
    return starts


def to_concat(rows, R_records, Q_records):
    """(r_rec, r_pos, q_rec, q_pos, len) -> sorted (r, q, len) in concatenated coordinates."""
    rs, qs = record_starts(R_records), record_starts(Q_records)
    t = sorted((rs[a] + b, qs[c] + d, n) for a, b, c, d, n in rows)
    return np.array(t, dtype=np.uint32).reshape(-1, 3)


def random_fasta(rng, n_rec, max_len, n_rate=0.02, alphabet="ACGT", prefix="s"):
    recs = []
    for i in range(n_rec):
        n = int(rng.integers(0, max_len + 1))
        s = np.array(list(alphabet))[rng.integers(0, len(alphabet), n)]
        s[rng.random(n) < n_rate] = "N"
        recs.append((f"{prefix}{i}", "".join(s)))
    return "".join(f">{name} rec\n{seq}\n" for name, seq in recs)
