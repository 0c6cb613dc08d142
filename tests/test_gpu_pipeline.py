"""GPU parity of the CUDA-graph pipeline (gpumem_pipeline_*, the launch configuration
bench.py times): the same kernels as pack + index_build + find_mems, captured once
and replayed, with the output sort sized by the device-resident MEM count. Checked
bit-exact against the CPU oracle (and brute force on tiny inputs), across relaunches,
recaptures, q ranges, the overflow fallback and alphabet errors."""
import numpy as np
import pytest

import oracle
from paper_conf_ipps_abu_dolehkac14_b200 import synth
from tests import invariants

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # collected on CPU boxes, skipped there
    pytest.skip("needs a CUDA device", allow_module_level=True)

from paper_conf_ipps_abu_dolehkac14_b200 import gpumem  # noqa: E402


@pytest.fixture(autouse=True)
def _default_options():
    yield
    gpumem.set_option("out_capacity", 0)
    gpumem.set_option("sort_impl", 0)
    gpumem.set_option("index_alg1", 0)
    gpumem.set_option("index_tiled", -1)
    gpumem.set_option("pipe_events", 0)


def _dev(x):
    b = x.tobytes() if isinstance(x, np.ndarray) else (x.encode() if isinstance(x, str) else bytes(x))
    if not b:
        return torch.empty(0, dtype=torch.uint8, device="cuda")
    return torch.from_numpy(np.frombuffer(b, dtype=np.uint8).copy()).cuda()


def pipe_mems(R, Q, L, ls, q_range=None, runs=1):
    Rt, Qt = _dev(R), _dev(Q)
    pl = gpumem.Pipeline(Rt.numel(), Qt.numel(), ls, L, q_range)
    outs = []
    for _ in range(runs):
        pl.run(Rt, Qt)
        pl.result()
        outs.append(pl.numpy())
    for o in outs[1:]:
        assert np.array_equal(o, outs[0])  # graph relaunch: identical
    st = pl.stats()
    pl.free()
    return outs[0], st


@pytest.mark.parametrize("cfg,scale", [("c1", 1.0), ("c2", 0.3), ("c3", 0.05), ("c4", 0.02), ("c5_l20", 0.02),
                                       ("c5_l300", 0.02)])
def test_pipeline_config_parity(cfg, scale):
    P = synth.make_pair(cfg, scale=scale)
    want = oracle.mems(P.R, P.Q, P.L, P.ls)
    got, st = pipe_mems(P.R, P.Q, P.L, P.ls, runs=3)
    assert np.array_equal(got, want)
    assert st["mems"] == len(want) and st["attempts"] == 1
    invariants.check(P.R, P.Q, P.L, got)


@pytest.mark.parametrize("impl", [0, 1, 2])
@pytest.mark.parametrize("n,m,L", [(300, 20000, 20), (20000, 300, 20), (2, 50000, 1)])
def test_pipeline_sort_skewed(impl, n, m, L):
    """Device-count output sorts (auto, LSD, MSD) on skewed keys: one r with 20 000 MEMs
    (a prefix run far past shared memory -> the global fallback), or many small runs."""
    from oracle import pyoracle
    gpumem.set_option("sort_impl", impl)
    want = np.array(pyoracle.homopolymer(n, m, L), dtype=np.uint32).reshape(-1, 3)
    got, _ = pipe_mems("A" * n, "A" * m, L, 1 if L < 13 else 13)
    assert np.array_equal(got, want)


@pytest.mark.parametrize("impl", [0, 2])
@pytest.mark.parametrize("copies", [2, 33, 70, 1100])
def test_pipeline_sort_equal_r_runs(impl, copies):
    """The MSD segment sort orders r's digits only and then ranks each key inside its run
    of equal r; runs past 1024 keys take the full-digit fallback. Q holds `copies` copies
    of several R segments, so each of their r has that many MEMs."""
    rng = np.random.default_rng(copies)
    R = rng.choice(np.frombuffer(b"ACGT", dtype=np.uint8), 20000)
    parts = []
    for c in range(copies):
        for a in (1000, 5000, 12000):
            parts.append(R[a:a + 300])
            parts.append(rng.choice(np.frombuffer(b"ACGT", dtype=np.uint8), 40 + c % 7))
    Q = np.concatenate(parts)
    want = oracle.mems(R.tobytes(), Q.tobytes(), 100, 13)
    assert len(want) >= 3 * copies
    gpumem.set_option("sort_impl", impl)
    try:
        got, _ = pipe_mems(R.tobytes().decode(), Q.tobytes().decode(), 100, 13)
        assert np.array_equal(got, want)
    finally:
        gpumem.set_option("sort_impl", 0)


@pytest.mark.parametrize("alg1,tiled", [(0, 1), (0, 0), (1, 0)])
def test_pipeline_index_paths(alg1, tiled):
    """Every index build (tiled Alg. 1 / stable radix sort / Alg. 1 as written) under the
    captured graph."""
    gpumem.set_option("index_alg1", alg1)
    gpumem.set_option("index_tiled", tiled)
    for cfg, scale in (("c5_l20", 0.02), ("c1", 1.0)):
        P = synth.make_pair(cfg, scale=scale)
        got, _ = pipe_mems(P.R, P.Q, P.L, P.ls, runs=2)
        assert np.array_equal(got, oracle.mems(P.R, P.Q, P.L, P.ls)), (cfg, alg1, tiled)


def test_pipeline_random_tiny_vs_brute_force():
    rng = np.random.default_rng(7)
    alph = [b"A", b"AC", b"ACGT"]
    for trial in range(40):
        R, Q = synth.random_pair(rng, int(rng.integers(1, 300)), int(rng.integers(1, 300)), alph[trial % 3])
        L = int(rng.integers(1, 30))
        ls = int(rng.integers(1, min(L, 15) + 1))
        got, _ = pipe_mems(R, Q, L, ls)
        assert np.array_equal(got, oracle.brute(R, Q, L)), trial


def test_pipeline_qrange_and_recapture():
    P = synth.make_pair("c2", scale=0.05)
    n = len(P.Q)
    for a, b in ((0, n // 3), (n // 3, n), (n // 2, n // 2)):
        got, _ = pipe_mems(P.R, P.Q, P.L, P.ls, q_range=(a, b))
        assert np.array_equal(got, oracle.mems(P.R, P.Q, P.L, P.ls, 0, a, b)), (a, b)
    # new input buffers (other contents, same sizes) -> recapture on the same pipeline
    gpumem.set_option("pipe_events", 1)  # stage events in the graph (profile below)
    Rt, Qt = _dev(P.R), _dev(P.Q)
    pl = gpumem.Pipeline(len(P.R), n, P.ls, P.L)
    pl.run(Rt, Qt)
    first = (pl.result(), pl.numpy())
    Q2 = P.Q.copy()
    Q2[: n // 2] = P.R[: n // 2]
    Qt2 = _dev(Q2)
    pl.run(Rt, Qt2)
    pl.result()
    assert np.array_equal(pl.numpy(), oracle.mems(P.R, Q2, P.L, P.ls))
    pl.run(Rt, Qt)
    assert pl.result() == first[0] and np.array_equal(pl.numpy(), first[1])
    prof = pl.profile()
    assert {"pack", "find", "sort"} <= set(prof) and all(v[0] > 0 for k, v in prof.items() if k in ("find", "sort"))
    pl.free()


def test_pipeline_overflow_fallback():
    P = synth.make_pair("c1")
    want = oracle.mems(P.R, P.Q, P.L, P.ls)
    gpumem.set_option("out_capacity", 100)  # fewer than the MEMs: the graph's output overflows
    got, st = pipe_mems(P.R, P.Q, P.L, P.ls, runs=2)
    assert np.array_equal(got, want)
    assert st["attempts"] >= 2


def test_pipeline_edges_and_alphabet():
    R = synth.make_pair("c1", scale=0.2).R.tobytes()
    got, _ = pipe_mems(R, R, 20, 10)
    assert (0, 0, len(R)) in {tuple(t) for t in got.tolist()}
    assert np.array_equal(got, oracle.mems(R, R, 20, 10))
    assert len(pipe_mems(R, b"ACGT" * 4, 20, 10)[0]) == 0
    assert len(pipe_mems(R, b"", 20, 10)[0]) == 0
    bad = bytearray(R[:5000])
    bad[1234] = ord("N")
    Rt, Qt = _dev(bytes(bad)), _dev(R[:3000])
    pl = gpumem.Pipeline(Rt.numel(), Qt.numel(), 10, 20)
    pl.run(Rt, Qt)
    with pytest.raises(gpumem.GpumemError) as ei:
        pl.result()
    assert ei.value.name == "ERR_ALPHABET" and "1234" in str(ei.value)
    pl.free()


def test_pipeline_host_inputs():
    """run_host: H2D copies overlapped with the R half of the graph; same MEM set, and
    switching between host and device inputs recaptures correctly."""
    P = synth.make_pair("c2", scale=0.2)
    want = oracle.mems(P.R, P.Q, P.L, P.ls)
    Rh = torch.from_numpy(P.R).pin_memory()
    Qh = torch.from_numpy(P.Q).pin_memory()
    pl = gpumem.Pipeline(len(P.R), len(P.Q), P.ls, P.L)
    for src in ("host", "host", "dev", "host", "numpy"):
        if src == "host":
            pl.run_host(Rh, Qh)
        elif src == "numpy":
            pl.run_host(P.R, P.Q)
        else:
            pl.run(_dev(P.R), _dev(P.Q))
        assert pl.result() == len(want), src
        assert np.array_equal(pl.numpy(), want), src
    pl.free()


@pytest.mark.parametrize("spill", [64, 1])
@pytest.mark.parametrize("chunks", [1, 2, 5, 16])
@pytest.mark.parametrize("cfg,scale", [("c4", 0.03), ("c5_l20", 0.03), ("c3", 0.1)])
def test_pipeline_streamed_query(cfg, scale, chunks, spill):
    """Host-input runs with Q streamed in pieces (option q_chunks): MEMs cut at the data
    present are finished after the last piece; the set equals the oracle's and the
    whole-Q (q_chunks = 1) result, relaunch after relaunch. find_spill = 1 sends every
    hit through the heavy queue, whose pieces must keep their piece's ownership range
    (seed positions within step of a piece end are scanned by both pieces)."""
    gpumem.set_option("q_chunks", chunks)
    gpumem.set_option("find_spill", spill)
    try:
        P = synth.make_pair(cfg, scale=scale)
        want = oracle.mems(P.R, P.Q, P.L, P.ls)
        pl = gpumem.Pipeline(len(P.R), len(P.Q), P.ls, P.L)
        Rh, Qh = torch.from_numpy(P.R).pin_memory(), torch.from_numpy(P.Q).pin_memory()
        for _ in range(3):
            pl.run_host(Rh, Qh)
            assert pl.result() == len(want)
            assert np.array_equal(pl.numpy(), want)
            assert pl.stats()["attempts"] == 1
        pl.free()
    finally:
        gpumem.set_option("q_chunks", 8)
        gpumem.set_option("find_spill", 64)


def test_pipeline_streamed_query_long_matches():
    """Matches far longer than a piece run through every piece boundary: the self-match
    of a 5 Mbp sequence (one MEM of 5 Mbp) and poly-A arrays across piece boundaries."""
    gpumem.set_option("q_chunks", 5)
    try:
        rng = np.random.default_rng(11)
        S = np.frombuffer(b"ACGT", np.uint8)[rng.integers(0, 4, 5_000_000)].copy()
        for a in (1_000_000 - 3000, 2_000_000 - 17, 3_999_990):  # poly-A runs over piece boundaries
            S[a:a + 6000] = ord("A")
        want = oracle.mems(S, S, 50, 13)
        assert (0, 0, len(S)) in {tuple(t) for t in want.tolist()}
        pl = gpumem.Pipeline(len(S), len(S), 13, 50)
        pl.run_host(torch.from_numpy(S).pin_memory(), torch.from_numpy(S).pin_memory())
        pl.result()
        assert np.array_equal(pl.numpy(), want)
        pl.free()
    finally:
        gpumem.set_option("q_chunks", 8)


@pytest.mark.parametrize("events,want", [(0, set()), (2, {"find"}), (1, {"pack", "index.tiled", "find", "sort"})])
def test_pipeline_event_modes(events, want):
    """pipe_events: no stage events (default), find's only (the timed bench graph), every
    stage; the MEM set never depends on it."""
    P = synth.make_pair("c1")
    gpumem.set_option("pipe_events", events)
    Rt, Qt = _dev(P.R), _dev(P.Q)
    pl = gpumem.Pipeline(len(P.R), len(P.Q), P.ls, P.L)
    pl.run(Rt, Qt)
    pl.result()
    prof = pl.profile()
    assert want <= set(prof) and (events != 0 or not prof) and (events != 2 or set(prof) == {"find"})
    assert np.array_equal(pl.numpy(), oracle.mems(P.R, P.Q, P.L, P.ls))
    pl.free()


def test_gather_ceiling_diag():
    """The instrumentation kernel bench.py uses for k_find's ceiling runs and scales."""
    a = gpumem.gather_ceiling(10_000_000, 16 << 20)
    b = gpumem.gather_ceiling(40_000_000, 16 << 20)
    assert 0 < a < b < 50 * a
    with pytest.raises(gpumem.GpumemError):
        gpumem.gather_ceiling(0, 16 << 20)
