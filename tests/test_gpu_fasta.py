"""NEXT-F4 on the GPU: multi-FASTA inputs through the CUDA path (the concatenations
packed, indexed and searched, then gpumem_split_masked cuts the MEMs at record
boundaries and non-ACGT letters), both strands, against the per-segment oracle
(oracle.mems_multi, pinned to the definition in tests/test_fasta.py), and the
MUMmer-style text of the hand-worked fixture byte for byte."""
import numpy as np
import pytest

import oracle
from oracle import pyoracle
from paper_conf_ipps_abu_dolehkac14_b200 import synth
from tests.fasta_util import random_fasta, read_mummer_golden, record_starts, to_concat

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

from paper_conf_ipps_abu_dolehkac14_b200 import gpumem as gm  # noqa: E402


def _rc(s):
    return s[::-1].translate(str.maketrans("ACGTNacgtn", "TGCANtgcan"))


def gpu_multi(R_text, Q_text, L, ls, reverse=False):
    fr, fq = gm.fasta_parse(R_text), gm.fasta_parse(Q_text)
    Rs, Qs = gm.pack(fr.seq()), gm.pack(fq.seq())
    if reverse:
        Qs = gm.revcomp(Qs)
    m = gm.find_mems(gm.index_build(Rs, ls, L), Qs)
    return gm.split_masked(m, fr, fq, L, q_reverse=reverse).numpy(), fr, fq


def expected(R_text, Q_text, L, ls, reverse=False):
    Rrec, Qrec = pyoracle.fasta(R_text), pyoracle.fasta(Q_text)
    if not reverse:
        return to_concat(oracle.mems_multi(R_text, Q_text, L, ls), Rrec, Qrec)
    rows = oracle.mems_multi(R_text, "".join(f">{n}\n{_rc(s)}\n" for n, s in Qrec), L, ls)
    rs, qs = record_starts(Rrec), record_starts(Qrec)
    nQ = sum(len(s) for _, s in Qrec) + len(Qrec) - 1
    # position in the reverse complement of the whole concatenated query
    t = sorted((rs[a] + b, nQ - (qs[c] + len(Qrec[c][1])) + d, n) for a, b, c, d, n in rows)
    return np.array(t, dtype=np.uint32).reshape(-1, 3)


def test_golden_multi_fasta_and_mummer_text(tmp_path):
    R, Q, L, expect = read_mummer_golden()
    for ls in (1, 2, 3):
        fwd, fr, fq = gpu_multi(R, Q, L, ls)
        assert np.array_equal(fwd, expected(R, Q, L, ls)), ls
        rev, _, _ = gpu_multi(R, Q, L, ls, reverse=True)
        assert np.array_equal(rev, expected(R, Q, L, ls, reverse=True)), ls
    path = tmp_path / "gpu.mums"
    gm.write_mummer(path, fwd, fr, fq, rev=rev)
    assert path.read_text() == expect


@pytest.mark.parametrize("alphabet", ["AC", "ACGT"])
def test_random_multi_fasta_both_strands(alphabet):
    rng = np.random.default_rng(7 + len(alphabet))
    for trial in range(40):
        Rt = random_fasta(rng, int(rng.integers(1, 5)), 120, 0.03, alphabet, "r")
        Qt = random_fasta(rng, int(rng.integers(1, 5)), 120, 0.03, alphabet, "q")
        L = int(rng.integers(2, 12))
        ls = int(rng.integers(1, min(L, 15) + 1))
        for rev in (False, True):
            got, _, _ = gpu_multi(Rt, Qt, L, ls, reverse=rev)
            assert np.array_equal(got, expected(Rt, Qt, L, ls, reverse=rev)), (trial, rev)


def test_genome_scale_records_with_n_runs():
    """A C2-like pair cut into records, with N runs (assembly gaps) and IUPAC letters."""
    P = synth.make_pair("c2", scale=0.05)
    rng = np.random.default_rng(3)

    def to_fasta(seq, n_rec, prefix):
        s = bytearray(seq.tobytes())
        for _ in range(6):  # gaps
            a, g = int(rng.integers(0, len(s) - 200)), int(rng.integers(1, 150))
            s[a:a + g] = b"N" * g
        for _ in range(20):
            s[int(rng.integers(0, len(s)))] = ord("RYKMSWN"[int(rng.integers(0, 7))])
        cuts = sorted(rng.choice(np.arange(1, len(s)), n_rec - 1, replace=False).tolist())
        parts = [bytes(s[a:b]) for a, b in zip([0] + cuts, cuts + [len(s)])]
        return "".join(f">{prefix}{i}\n{p.decode()}\n" for i, p in enumerate(parts))

    Rt, Qt = to_fasta(P.R, 4, "chr"), to_fasta(P.Q, 3, "read")
    got, _, _ = gpu_multi(Rt, Qt, P.L, P.ls)
    want = expected(Rt, Qt, P.L, P.ls)
    assert len(want) > 1000 and np.array_equal(got, want)
