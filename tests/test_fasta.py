"""NEXT-F4 on CPU: the multi-FASTA oracle pinned (definition vs method), the library's
host-side FASTA parser (record table, masks, layout) and its MUMmer-style writer against
the hand-worked fixture tests/golden/mummer_multi.txt."""
import numpy as np
import pytest

import oracle
from oracle import pyoracle
from tests.fasta_util import random_fasta, read_mummer_golden, record_starts, to_concat

gm = pytest.importorskip("paper_conf_ipps_abu_dolehkac14_b200.gpumem")


def test_multi_oracles_agree_on_golden_and_random():
    R, Q, L, _ = read_mummer_golden()
    assert pyoracle.multi_brute(R, Q, L) == oracle.mems_multi(R, Q, L, 2)
    assert len(pyoracle.multi_brute(R, Q, L)) == 9
    rng = np.random.default_rng(31)
    for trial in range(40):
        Rt = random_fasta(rng, int(rng.integers(1, 4)), 60, 0.05, ["AC", "ACGT"][trial % 2], "r")
        Qt = random_fasta(rng, int(rng.integers(1, 4)), 60, 0.05, ["AC", "ACGT"][trial % 2], "q")
        L = int(rng.integers(2, 8))
        assert pyoracle.multi_brute(Rt, Qt, L) == oracle.mems_multi(Rt, Qt, L, min(L, 3)), trial


def test_fasta_parse_layout_and_masks():
    f = gm.fasta_parse(">a x y\nACgt\nNNA\n>b\n\n>c\nRYAC\n")
    recs = f.records()
    assert [r[0] for r in recs] == ["a", "b", "c"]
    assert [(r[1], r[2]) for r in recs] == [(0, 7), (8, 0), (9, 4)]  # one separator between records
    assert f.seq().tobytes() == b"ACGTAAAAAAAAC"
    assert f.info()[3] == 2  # masked intervals: NN [4, 6); sep, sep, RY merged [7, 11)
    for bad in (b"ACGT\n", b">a\nAC\x01G\n"):
        with pytest.raises(gm.GpumemError):
            gm.fasta_parse(bad)


def test_mummer_writer_on_oracle_triples(tmp_path):
    """The writer (host C++) fed the oracle's triples, mapped to concatenated coordinates
    by the documented layout, prints the hand-worked fixture byte for byte."""
    R, Q, L, expect = read_mummer_golden()
    fr, fq = gm.fasta_parse(R), gm.fasta_parse(Q)
    Rrec, Qrec = pyoracle.fasta(R), pyoracle.fasta(Q)
    assert [r[1] for r in fr.records()] == record_starts(Rrec)
    fwd = to_concat(oracle.mems_multi(R, Q, L, 2), Rrec, Qrec)

    def rc(s):
        return s[::-1].translate(str.maketrans("ACGTN", "TGCAN"))

    # reverse strand: the MEMs against the reverse complement of the concatenated query
    Qrc_text = "".join(f">{n}\n{rc(s)}\n" for n, s in Qrec)
    rev_rows = oracle.mems_multi(R, Qrc_text, L, 2)
    qs, nQ = record_starts(Qrec), sum(len(s) for _, s in Qrec) + len(Qrec) - 1
    rev = sorted((record_starts(Rrec)[a] + b, nQ - (qs[c] + len(Qrec[c][1])) + d, n) for a, b, c, d, n in rev_rows)
    path = tmp_path / "out.mums"
    gm.write_mummer(path, fwd, fr, fq, rev=np.array(rev, np.uint32).reshape(-1, 3))
    assert path.read_text() == expect
