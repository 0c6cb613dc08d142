"""Small workloads for compute-sanitizer (memcheck, racecheck, synccheck, initcheck):
every kernel of the library on C1 and the adversarial tiny cases, through direct
calls and through the CUDA-graph pipeline, each result checked against the oracle.

    compute-sanitizer --tool memcheck --error-exitcode 9 python tools/sanitize_cases.py [quick]
"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
from oracle import pyoracle  # noqa: E402
from paper_conf_ipps_abu_dolehkac14_b200 import gpumem, synth  # noqa: E402

quick = "quick" in sys.argv[1:]
torch.cuda.set_device(0)


def direct(R, Q, L, ls, **opts):
    for k, v in opts.items():
        gpumem.set_option(k, v)
    try:
        return gpumem.mems(R, Q, L, ls)
    finally:
        for k in opts:
            gpumem.set_option(k, {"index_alg1": 0, "sort_impl": 0, "find_spill": 64, "static_lb": 0,
                                  "use_bitmap": 1, "rank_sectors": -1, "out_capacity": 0, "index_tiled": -1}[k])


def piped(R, Q, L, ls):
    R, Q = (x.encode() if isinstance(x, str) else x for x in (R, Q))
    Rt = torch.from_numpy(np.frombuffer(bytes(R), np.uint8).copy()).cuda()
    Qt = torch.from_numpy(np.frombuffer(bytes(Q), np.uint8).copy()).cuda()
    pl = gpumem.Pipeline(Rt.numel(), Qt.numel(), ls, L)
    pl.run(Rt, Qt)
    pl.result()
    out = pl.numpy()
    pl.free()
    return out


n_checks = 0


def check(got, want, what):
    global n_checks
    want = np.asarray(want, dtype=np.uint32).reshape(-1, 3)
    assert np.array_equal(got, want), what
    n_checks += 1


# C1 (scaled for racecheck's cost), every index/find/sort path
P = synth.make_pair("c1", scale=0.2 if quick else 1.0)
want = oracle.mems(P.R, P.Q, P.L, P.ls)
R, Q = P.R.tobytes(), P.Q.tobytes()
check(direct(R, Q, P.L, P.ls), want, "c1 direct")
check(piped(R, Q, P.L, P.ls), want, "c1 pipeline")
for opts in ({"index_alg1": 1}, {"sort_impl": 1}, {"sort_impl": 2}, {"find_spill": 1}, {"static_lb": 1},
             {"use_bitmap": 0}, {"rank_sectors": 1}, {"out_capacity": 5}, {"index_tiled": 0},
             {"index_tiled": 1, "rank_sectors": 1}):
    check(direct(R, Q, P.L, P.ls, **opts), want, f"c1 {opts}")

# adversarial tiny cases: homopolymers (heavy queue, coop extensions), (AC)^n, long
# left checks (step 288), ls = 1 and ls = L, self-match, empty inputs
for n, m, L, ls in ((300, 2000, 20, 10), (5000, 5000, 4500, 13), (2, 3000, 1, 1), (700, 700, 300, 13)):
    check(direct("A" * n, "A" * m, L, ls), pyoracle.homopolymer(n, m, L), f"homopolymer {n} {m} {L}")
check(piped("A" * 3000, "A" * 3000, 20, 10), pyoracle.homopolymer(3000, 3000, 20), "homopolymer pipeline")
# tiled index: a hot bin past the CTA's shared memory (global-memory steps 3-4), long
# buckets placed in input order, rank sectors; the radix path on the same input
check(direct("A" * 45000, "A" * 500, 20, 13, index_tiled=1), pyoracle.homopolymer(45000, 500, 20),
      "tiled global-memory bin")
hot = b"A" * 3000 + b"AC" * 1000 + b"ACGT" * 400 + b"T" * 300
hot_want = oracle.mems(hot, hot[100:], 20, 13)
for tiled, sect in ((1, 0), (1, 1), (0, 0)):
    check(direct(hot, hot[100:], 20, 13, index_tiled=tiled, rank_sectors=sect), hot_want,
          f"hot seeds tiled={tiled} sect={sect}")
rng = np.random.default_rng(5)
for trial in range(20 if quick else 60):
    R1, Q1 = synth.random_pair(rng, int(rng.integers(0, 300)), int(rng.integers(0, 300)), [b"AC", b"ACGT"][trial % 2])
    L1 = int(rng.integers(1, 40))
    ls1 = int(rng.integers(1, min(L1, 15) + 1))
    check(direct(R1, Q1, L1, ls1), oracle.brute(R1, Q1, L1), f"random {trial}")
tandem = b"AC" * 400 + b"GATTACA" * 50 + b"A" * 300
check(direct(tandem, tandem[5:], 300, 13), oracle.brute(tandem, tandem[5:], 300), "step 288")
check(direct(tandem, tandem, 13, 13), oracle.brute(tandem, tandem, 13), "ls = L")
check(direct(b"", b"ACGT", 4, 2), [], "empty R")

# K9 merge of query shards, MUM filter, reverse complement
Rs, Qs = gpumem.pack(R), gpumem.pack(Q)
idx = gpumem.index_build(Rs, P.ls, P.L)
cuts = [len(Q) * g // 3 for g in range(4)]
parts = [gpumem.find_mems(idx, Qs, (a, b)) for a, b in zip(cuts[:-1], cuts[1:])]
m = gpumem.merge_sorted([p.view_u32().view(torch.int32) for p in parts])
check(m.numpy(), want, "merge")
mu = gpumem.mums(m)
check(mu.numpy(), oracle.mums(P.R, P.Q, P.L, P.ls), "mums")
rc = gpumem.revcomp(Qs)
assert len(rc) == len(Q)
torch.cuda.synchronize()
print(f"sanitize cases ok: {n_checks} checks")
