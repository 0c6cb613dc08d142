"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element
by element, on seeded inputs. Bit-exact: MEMs are integer triples (r, q, len)
and the set is unique (reading R20), sorted by (r, q)."""
import numpy as np
import pytest

import oracle
from oracle import pyoracle
from paper_conf_ipps_abu_dolehkac14_b200 import synth
from tests import invariants
from tests.conftest import read_golden

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # collected on CPU boxes, skipped there
    pytest.skip("needs a CUDA device", allow_module_level=True)

from paper_conf_ipps_abu_dolehkac14_b200 import gpumem  # noqa: E402


@pytest.fixture(autouse=True)
def _default_options():
    yield
    for k, v in (("find_grid", 0), ("find_spill", 64), ("out_capacity", 0), ("use_bitmap", 1), ("static_lb", 0),
                 ("sort_impl", 0), ("radix_bits", 0),
                 ("rank_sectors", -1), ("rec8", -1), ("pdl", 1), ("index_alg1", 0), ("index_tiled", -1)):
        gpumem.set_option(k, v)


def gpu_mems(R, Q, L, ls, step=None, q_range=None, device_input=False):
    if device_input:
        Rt = torch.from_numpy(np.frombuffer(bytes(R), dtype=np.uint8).copy()).cuda()
        Qt = torch.from_numpy(np.frombuffer(bytes(Q), dtype=np.uint8).copy()).cuda()
        Rs, Qs = gpumem.pack(Rt), gpumem.pack(Qt)
    else:
        Rs, Qs = gpumem.pack(R), gpumem.pack(Q)
    idx = gpumem.index_build(Rs, ls, L, step)
    m = gpumem.find_mems(idx, Qs, q_range)
    out = m.numpy()
    torch.cuda.synchronize()
    return out


def _b(x):
    return x.tobytes() if isinstance(x, np.ndarray) else (x.encode() if isinstance(x, str) else bytes(x))


# ------------------------------------------------------------------ K1 pack
def _decode(words, n):
    w = words.astype(np.uint64)
    i = np.arange(n, dtype=np.uint64)
    c = (w[i // 32] >> (np.uint64(62) - np.uint64(2) * (i % np.uint64(32)))) & np.uint64(3)
    return np.frombuffer(b"ACGT", dtype=np.uint8)[c.astype(np.int64)]


def test_pack_known_word():
    s = gpumem.pack(b"ACGT" * 8)
    w = s.words().cpu().numpy()
    assert int(w[0]) == 0x1B1B1B1B1B1B1B1B
    assert len(w) == 5 and not w[1:].any()  # four zero padding words


@pytest.mark.parametrize("n", [0, 1, 31, 32, 33, 1000, 4097, 100_003])
@pytest.mark.parametrize("offset", [0, 1, 7, 16])
def test_pack_roundtrip_device_and_host(n, offset):
    rng = np.random.default_rng(n + offset)
    raw = np.frombuffer(b"ACGTacgt", dtype=np.uint8)[rng.integers(0, 8, n + offset)]
    dev = torch.from_numpy(raw.copy()).cuda()[offset:]
    for s in (gpumem.pack(dev), gpumem.pack(raw[offset:].tobytes())):
        s.check()
        nn, _, nw = s.info()
        assert nn == n and nw == (n + 31) // 32 + 4
        w = s.words().cpu().numpy()
        assert not w[(n + 31) // 32:].any()  # four zero padding words
        up = raw[offset:] & 0xDF
        assert np.array_equal(_decode(w, n), up)
        if n % 32:
            last = int(w[n // 32])
            assert last & ((1 << (64 - 2 * (n % 32))) - 1) == 0  # padding bases are 00


@pytest.mark.parametrize("bad", [b"N", b"n", b"-", b"\x00", b"U", b"\xc1", b"B"])
@pytest.mark.parametrize("pos", [0, 5, 31, 32, 999])
def test_pack_alphabet_error(bad, pos):
    s = bytearray(b"ACGT" * 300)
    s[pos:pos + 1] = bad
    q = gpumem.pack(bytes(s))
    with pytest.raises(gpumem.GpumemError) as ei:
        q.check()
    assert ei.value.name == "ERR_ALPHABET"
    assert f"position {pos}" in str(ei.value)
    # find_mems reports it too
    R = gpumem.pack(b"ACGT" * 10)
    idx = gpumem.index_build(R, 4, 8)
    with pytest.raises(gpumem.GpumemError) as ei:
        gpumem.find_mems(idx, q)
    assert ei.value.name == "ERR_ALPHABET"


# ------------------------------------------------------------------ K2-K5 index
def _index_gpu(R, ls, step):
    s = gpumem.pack(R)
    idx = gpumem.index_build(s, ls, ls + step - 1, step)
    p, l = idx.view()
    out = p.cpu().numpy().copy(), l.cpu().numpy().copy()
    torch.cuda.synchronize()
    return out


def test_index_golden_w2():
    g = read_golden("w2_index.txt")
    p, l = _index_gpu(g["R"], g["ls"], g["step"])
    assert p.tolist() == g["ptrs"] and l.tolist() == g["locs"]


@pytest.mark.parametrize("cfg,ls,step,scale", [("c1", 10, 11, 1.0), ("c1", 1, 1, 0.01), ("c1", 3, 5, 0.2),
                                                ("c2", 12, 9, 1.0), ("c3", 13, 38, 0.1), ("c4", 13, 8, 0.02),
                                                ("c4", 15, 1, 0.01), ("c1", 7, 64, 0.5)])
def test_index_parity_word_for_word(cfg, ls, step, scale):
    """ptrs (expanded from the lookup directory + compact table, both directory kinds)
    and locs word for word against Alg. 1."""
    P = synth.make_pair(cfg, scale=scale)
    op, ol = oracle.index(P.R.tobytes(), ls, step)
    for tiled in (1, 0):  # Alg. 1 tiled over the seed space (tindex.cu) / the radix path
        gpumem.set_option("index_tiled", tiled)
        for sect in (-1, 0, 1):
            gpumem.set_option("rank_sectors", sect)
            p, l = _index_gpu(P.R.tobytes(), ls, step)
            assert np.array_equal(p, op), (tiled, sect)
            assert np.array_equal(l, ol), (tiled, sect)


def test_index_hot_seed_chunks():
    """Directory build on runs far longer than a block (poly-A / (AC)^n seeds: one code
    with tens of thousands of sampled locations), every block/run boundary case."""
    R = b"A" * 70000 + b"AC" * 20000 + b"ACGT" * 3000 + b"T" * 1500
    for ls, step in ((13, 1), (12, 3), (5, 2)):
        op, ol = oracle.index(R, ls, step)
        for sect in (0, 1):
            # Alg. 1 as written (buckets of 70 000: global sorting network), the tiled Alg. 1
            # (a bin of 70 000: beyond a CTA's shared memory, steps 3-4 in global memory),
            # the radix path
            for alg1, tiled in ((1, 0), (0, 1), (0, 0)):
                gpumem.set_option("rank_sectors", sect)
                gpumem.set_option("index_alg1", alg1)
                gpumem.set_option("index_tiled", tiled)
                p, l = _index_gpu(R, ls, step)
                assert np.array_equal(p, op) and np.array_equal(l, ol), (ls, step, sect, alg1, tiled)


@pytest.mark.parametrize("opts", [{"radix_bits": 8, "index_tiled": 0}, {"radix_bits": 10, "index_tiled": 0},
                                  {"index_alg1": 1}, {"index_alg1": 1, "rank_sectors": 1}, {"index_alg1": 0},
                                  {"rank_sectors": 1, "rec8": 1}, {"rank_sectors": 1, "rec8": 1, "index_tiled": 0}])
def test_index_sort_paths(opts):
    """Every index path (stable LSD radix sort at each digit width, Alg. 1 as written)
    gives the oracle's Alg. 1 ptrs/locs word for word."""
    P = synth.make_pair("c3", scale=0.05)
    op, ol = oracle.index(P.R.tobytes(), 13, 38)
    for k, v in opts.items():
        gpumem.set_option(k, v)
    p, l = _index_gpu(P.R.tobytes(), 13, 38)
    assert np.array_equal(p, op) and np.array_equal(l, ol)


@pytest.mark.parametrize("L,ls", [(20, 13), (28, 13), (12, 5)])
def test_heavy_bucket_minority_skip(L, ls):
    """Heavy buckets reordered minority-left-flank first (k_hv_part) and spilled as that
    prefix for query positions with the majority flank (step <= record flank width):
    poly-A / (AC)^n / (ACGT)^n hot seeds, run starts, p < step, both the heavy-queue
    threshold and find_spill 1 (every bucket spilled), 8- and 16-byte records."""
    rng = np.random.default_rng(11)
    rnd = lambda n: bytes(rng.choice(list(b"ACGT"), n).tolist())
    R = b"A" * 1500 + rnd(300) + b"AC" * 700 + rnd(200) + b"A" * 900 + b"ACGT" * 400 + rnd(500) + b"A" * 40
    Q = rnd(100) + b"A" * 1200 + rnd(50) + b"AC" * 600 + b"A" * 30 + rnd(300) + b"ACGT" * 300 + b"A" * 700
    want = oracle.mems(R, Q, L, ls)
    for spill in (64, 1):
        gpumem.set_option("index_tiled", 0)  # the radix path lists heavy buckets
        gpumem.set_option("find_spill", spill)
        got = gpu_mems(R, Q, L, ls)
        assert np.array_equal(got, want), (L, ls, spill)
    gpumem.set_option("find_spill", 64)


def test_index_short_reference():
    p, l = _index_gpu(b"ACG", 4, 1)
    assert len(l) == 0 and not p.any()


# ------------------------------------------------------------------ find: small exact cases
@pytest.mark.parametrize("name", ["w1.txt", "w2.txt", "w3.txt", "w4.txt"])
def test_golden_examples(name):
    g = read_golden(name)
    want = sorted(g["mem"])
    for ls in range(1, min(g["L"], 15) + 1):
        for step in range(1, g["L"] - ls + 2):
            got = gpu_mems(g["R"], g["Q"], g["L"], ls, step)
            assert [tuple(t) for t in got.tolist()] == want, (ls, step)


def test_random_tiny_vs_brute_force():
    rng = np.random.default_rng(99)
    alph = [b"A", b"AC", b"ACG", b"ACGT"]
    for trial in range(300):
        R, Q = synth.random_pair(rng, int(rng.integers(0, 200)), int(rng.integers(0, 200)), alph[trial % 4])
        L = int(rng.integers(1, 40))
        ls = int(rng.integers(1, min(L, 15) + 1))
        step = int(rng.integers(1, L - ls + 2))
        want = oracle.brute(R, Q, L)
        got = gpu_mems(R.tobytes(), Q.tobytes(), L, ls, step)
        assert np.array_equal(got, want), (trial, len(R), len(Q), L, ls, step)


@pytest.mark.parametrize("n,m", [(1, 1), (5, 3), (40, 70), (300, 257), (1000, 64)])
def test_homopolymer_closed_form(n, m):
    for L, ls in ((2, 1), (20, 10), (33, 13), (100, 15)):
        if ls > L:
            continue
        want = np.array(pyoracle.homopolymer(n, m, L), dtype=np.uint32).reshape(-1, 3)
        got = gpu_mems("A" * n, "A" * m, L, ls)
        assert np.array_equal(got, want), (n, m, L, ls)


@pytest.mark.parametrize("impl", [0, 1, 2])
@pytest.mark.parametrize("n,m,L", [(300, 20000, 20), (20000, 300, 20), (9000, 9000, 8000), (2, 50000, 1)])
def test_sort_skewed_buckets(impl, n, m, L):
    """Output sort on skewed key sets: most MEMs share r = 0 (one MSD bucket far past
    shared memory -> the global LSD fallback) or q = 0 (many small buckets), checked
    against the homopolymer closed form, under every output sort path (auto, LSD, MSD)."""
    gpumem.set_option("sort_impl", impl)
    want = np.array(pyoracle.homopolymer(n, m, L), dtype=np.uint32).reshape(-1, 3)
    got = gpu_mems("A" * n, "A" * m, L, 1 if L < 13 else 13)
    assert np.array_equal(got, want), (impl, n, m, L)


@pytest.mark.parametrize("L,ls", [(20, 10), (50, 13), (100, 13), (300, 13), (7, 1), (13, 13), (40, 15)])
def test_adversarial_repeats(L, ls):
    """Tandem repeats, (AC)^n, multi-word left checks (step > 32, > 64, 288),
    ls = 1, ls = L (step 1), MEMs touching all four sequence ends."""
    rng = np.random.default_rng(L * 31 + ls)
    parts_r = [b"AC" * 200, bytes(synth.to_ascii(rng.integers(0, 4, 500).astype(np.uint8))), b"AAT" * 100,
               b"G" * 150]
    R = b"".join(parts_r)
    Q = R[:400] + b"T" + b"AC" * 150 + bytes(synth.to_ascii(rng.integers(0, 4, 300).astype(np.uint8))) + R[-500:]
    want = oracle.mems(R, Q, L, ls)
    got = gpu_mems(R, Q, L, ls)
    assert np.array_equal(got, want)
    invariants.check(R, Q, L, got)
    for sect in (0, 1):  # both lookup directories (rank sectors: saturated repeat counts)
        for rec8 in (0, 1):  # both record widths
            gpumem.set_option("rank_sectors", sect)
            gpumem.set_option("rec8", rec8)
            assert np.array_equal(gpu_mems(R, Q, L, ls), want), (sect, rec8)
    gpumem.set_option("rank_sectors", -1)
    gpumem.set_option("rec8", -1)
    if len(want):
        assert np.array_equal(gpu_mems(R, Q, L, ls, device_input=True), want)


def test_self_match_and_edges():
    P = synth.make_pair("c1", scale=0.3)
    R = P.R.tobytes()
    got = gpu_mems(R, R, 20, 10)
    assert (0, 0, len(R)) in {tuple(t) for t in got.tolist()}
    assert np.array_equal(got, oracle.mems(R, R, 20, 10))
    assert len(gpu_mems(R, b"ACG", 20, 10)) == 0          # |Q| < ls
    assert len(gpu_mems(R, b"ACGT" * 4, 20, 10)) == 0     # |Q| < L
    assert len(gpu_mems(b"", R, 20, 10)) == 0
    assert len(gpu_mems(R, b"", 20, 10)) == 0


def test_overflow_retry_grid_spill_and_bitmap_invariance():
    P = synth.make_pair("c1")
    want = oracle.mems(P.R, P.Q, P.L, P.ls)
    base = gpu_mems(P.R, P.Q, P.L, P.ls)
    assert np.array_equal(base, want)
    for opt, vals in (("out_capacity", [1, 100]), ("find_grid", [1, 3, 148]), ("find_spill", [1, 2, 10**9]),
                      ("use_bitmap", [0]), ("static_lb", [1]), ("sort_impl", [1, 2]),
                      ("rank_sectors", [0, 1]), ("rec8", [0, 1]),
                      ("radix_bits", [8, 9, 10]), ("pdl", [0]), ("index_alg1", [1, -1]), ("index_tiled", [0, 1])):
        for v in vals:
            gpumem.set_option(opt, v)
            assert np.array_equal(gpu_mems(P.R, P.Q, P.L, P.ls), want), (opt, v)
        gpumem.set_option(opt, {"out_capacity": 0, "find_grid": 0, "find_spill": 64, "use_bitmap": 1,
                                "static_lb": 0, "sort_impl": 0, "rank_sectors": -1,
                                "rec8": -1,
                                "radix_bits": 0, "pdl": 1, "index_alg1": 0, "index_tiled": -1}[opt])


def test_l2_persisting_window_invariance():
    """The persisting-L2 access-policy window (options l2_persist / l2_window) changes
    only cache placement: every window choice, partial hit ratios and the reset are exact."""
    P = synth.make_pair("c1")
    want = oracle.mems(P.R, P.Q, P.L, P.ls)
    try:
        for persist, window in ((32, 1), (1, 1), (8, 2), (64, 3), (0, 1)):
            gpumem.set_option("l2_persist", persist)
            gpumem.set_option("l2_window", window)
            for sect in (0, 1):
                gpumem.set_option("rank_sectors", sect)
                assert np.array_equal(gpu_mems(P.R, P.Q, P.L, P.ls), want), (persist, window, sect)
    finally:
        gpumem.set_option("l2_window", 0)
        gpumem.set_option("l2_persist", 0)


def test_seed_length_and_step_invariance():
    P = synth.make_pair("c1", scale=0.5)
    want = oracle.mems(P.R, P.Q, 20, 10)
    for ls, step in ((10, None), (8, None), (12, 5), (1, 3), (15, 6), (13, 1)):
        assert np.array_equal(gpu_mems(P.R, P.Q, 20, ls, step), want), (ls, step)


def test_qrange_shards_union_to_whole():
    P = synth.make_pair("c2", scale=0.05)
    whole = gpu_mems(P.R, P.Q, P.L, P.ls)
    assert np.array_equal(whole, oracle.mems(P.R, P.Q, P.L, P.ls))
    n = len(P.Q)
    for G in (2, 3, 8):
        cuts = [n * g // G for g in range(G + 1)]
        parts = [gpu_mems(P.R, P.Q, P.L, P.ls, q_range=(a, b)) for a, b in zip(cuts[:-1], cuts[1:])]
        for (a, b), part in zip(zip(cuts[:-1], cuts[1:]), parts):
            assert np.array_equal(part, oracle.mems(P.R, P.Q, P.L, P.ls, 0, a, b))
        cat = np.concatenate(parts)
        cat = cat[np.lexsort((cat[:, 1], cat[:, 0]))]
        assert np.array_equal(cat, whole)


def _random_runs(rng, n, G, r_max, q_max, skew):
    """n unique (r, q) keys with a length each, dealt to G runs at random, each run
    sorted by (r, q) (lexsort), plus the whole set sorted -- the merge's expected output."""
    if skew == "one_r":  # every key on one r: one bucket far past shared memory
        r = np.zeros(n, np.uint64)
        q = rng.choice(q_max, size=n, replace=False).astype(np.uint64)
    elif skew == "hot":  # half the keys on a handful of r values
        r = np.where(rng.random(n) < 0.5, rng.integers(0, 4, n), rng.integers(0, r_max, n)).astype(np.uint64)
        q = rng.integers(0, q_max, n).astype(np.uint64)
    else:
        r = rng.integers(0, r_max, n).astype(np.uint64)
        q = rng.integers(0, q_max, n).astype(np.uint64)
    keys = np.unique((r << np.uint64(32)) | q)
    t = np.stack([(keys >> np.uint64(32)).astype(np.uint32), (keys & np.uint64(0xffffffff)).astype(np.uint32),
                  rng.integers(20, 1000, len(keys)).astype(np.uint32)], axis=1)
    owner = rng.integers(0, G, len(t))
    return [t[owner == g] for g in range(G)], t


@pytest.mark.parametrize("G", [1, 2, 3, 8, 64])
@pytest.mark.parametrize("n,skew", [(0, "uniform"), (1, "uniform"), (5000, "uniform"), (2_000_000, "uniform"),
                                    (300_000, "hot"), (20_000, "one_r")])
def test_merge_kernel(G, n, skew):
    """K9 merge (merge.cu): G sorted disjoint runs -> one (r, q)-sorted run, against a
    plain lexicographic sort of the union; empty runs, tiny runs, 2M triples, a hot-r
    skew and one bucket far past shared memory (all keys on r = 0)."""
    rng = np.random.default_rng(1000 * G + n)
    runs, want = _random_runs(rng, n, G, 250_000_000, 150_000_000, skew)
    dev = [torch.from_numpy(r.copy()).cuda().view(torch.int32) for r in runs]
    m = gpumem.merge_sorted(dev)
    got = m.numpy()
    m.free()
    assert got.shape == want.shape and np.array_equal(got, want)


def test_merge_of_query_shards():
    """The merge's real input: per-shard find_mems results (disjoint by the ownership
    rule, sorted) merged == the whole set == the oracle."""
    P = synth.make_pair("c3", scale=0.05)
    want = oracle.mems(P.R, P.Q, P.L, P.ls)
    for G in (2, 5, 8):
        cuts = [len(P.Q) * g // G for g in range(G + 1)]
        R, Q = gpumem.pack(P.R), gpumem.pack(P.Q)
        idx = gpumem.index_build(R, P.ls, P.L)
        parts = [gpumem.find_mems(idx, Q, (a, b)) for a, b in zip(cuts[:-1], cuts[1:])]
        m = gpumem.merge_sorted([p.view_u32().view(torch.int32) for p in parts])
        assert np.array_equal(m.numpy(), want), G
        for h in [m, *parts, idx, Q, R]:
            h.free()


def test_swap_symmetry():
    P = synth.make_pair("c1", scale=0.2)
    a = gpu_mems(P.R, P.Q, 20, 10)
    b = gpu_mems(P.Q, P.R, 20, 10)[:, [1, 0, 2]]
    b = b[np.lexsort((b[:, 1], b[:, 0]))]
    assert np.array_equal(a, b)


def test_kernels_are_ours():
    """The CUDA work of the path, as the CUDA profiler (CUPTI) sees it: every kernel that
    runs during pack + index + find + sort is one of libgpumem.so's own (namespace gm, no
    CUB/Thrust/torch kernels), the expected stages all run, and the library's launch
    counter agrees with the profiler's kernel count."""
    P = synth.make_pair("c2", scale=0.05)
    R, Q = P.R.tobytes(), P.Q.tobytes()
    gpu_mems(R, Q, P.L, P.ls)  # warm (workspaces, attributes)
    torch.cuda.synchronize()
    from torch.profiler import ProfilerActivity, profile
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        before = gpumem.launch_count()
        got = gpu_mems(R, Q, P.L, P.ls)
        torch.cuda.synchronize()
        launched = gpumem.launch_count() - before
    assert np.array_equal(got, oracle.mems(P.R, P.Q, P.L, P.ls))
    kernels = [e.name for e in prof.events() if e.device_type.name == "CUDA" and "Memcpy" not in e.name
               and "Memset" not in e.name]
    assert kernels, "no kernel seen by the profiler"
    foreign = [k for k in kernels if "gm::" not in k]
    assert not foreign, foreign
    for stage in ("k_pack", "k_seed_codes", "k_scatter", ("k_dir_fill", "k_tx_warp"), "k_seed_recs", "k_find",
                  "k_heavy", "k_bs_local"):
        alts = stage if isinstance(stage, tuple) else (stage,)  # radix / tiled index build
        assert any(a in k for k in kernels for a in alts), (stage, sorted(set(kernels)))
    assert launched == len(kernels), (launched, len(kernels))


# ------------------------------------------------------------------ configs (scaled and full)
@pytest.mark.parametrize("cfg,scale", [("c1", 1.0), ("c2", 1.0), ("c3", 0.2), ("c4", 0.04), ("c5_l20", 0.04),
                                       ("c5_l50", 0.04), ("c5_l300", 0.04)])
def test_config_parity(cfg, scale):
    P = synth.make_pair(cfg, scale=scale)
    want = oracle.mems(P.R, P.Q, P.L, P.ls)
    got = gpu_mems(P.R, P.Q, P.L, P.ls)
    assert len(got) == len(want)
    assert np.array_equal(got, want)
    invariants.check(P.R, P.Q, P.L, got)
    s = {tuple(t) for t in got.tolist()}
    assert all(tuple(t) in s for t in P.planted)


@pytest.fixture(scope="module")
def c4_full():
    return synth.make_pair("c4")


@pytest.mark.slow
@pytest.mark.parametrize("L", [100, 50])
def test_full_size_index_builders_identical(c4_full, L):
    """Both index builders at the full C4 / C5 L = 50 size (2.8 M / 6.6 M sampled
    locations, 4^13 seeds): the tiled Alg. 1 (forced; by default it serves only indexes
    up to 2^20 locations) and the radix path give the same locs and the same dense ptrs
    (expanded from each one's gapped table) word for word, and the same MEMs."""
    P = c4_full
    Rt, Qt = torch.from_numpy(P.R).cuda(), torch.from_numpy(P.Q).cuda()
    views, mems = {}, {}
    for tiled in (0, 1):
        gpumem.set_option("index_tiled", tiled)
        Rs = gpumem.pack(Rt)
        idx = gpumem.index_build(Rs, 13, L)
        p, l = idx.view()
        views[tiled] = (p.cpu().numpy().copy(), l.cpu().numpy().copy())
        mems[tiled] = gpumem.find_mems(idx, gpumem.pack(Qt)).numpy()
        del p, l, idx, Rs
        torch.cuda.synchronize()
    assert np.array_equal(views[0][0], views[1][0]) and np.array_equal(views[0][1], views[1][1])
    assert np.array_equal(mems[0], mems[1]) and len(mems[0]) > 0


@pytest.mark.slow
@pytest.mark.parametrize("L", [100, 300, 50, 20])
def test_full_size_c4_c5(c4_full, L):
    """BASELINE sizes (250 Mbp x 150 Mbp), bit-exact against the full oracle run."""
    P = c4_full
    want = oracle.mems(P.R, P.Q, L, 13)
    got = gpu_mems(P.R, P.Q, L, 13)
    assert np.array_equal(got, want)
    # the launch configuration bench.py times: the CUDA-graph pipeline, relaunched
    Rt, Qt = torch.from_numpy(P.R).cuda(), torch.from_numpy(P.Q).cuda()
    pl = gpumem.Pipeline(len(P.R), len(P.Q), 13, L)
    for _ in range(2):
        pl.run(Rt, Qt)
        assert pl.result() == len(want)
        assert np.array_equal(pl.numpy(), want)
    pl.free()


@pytest.mark.slow
@pytest.mark.parametrize("L", [100, 20])
def test_full_size_shards_byte_identical(c4_full, L):
    """SURVEY.md §8(e) check at the full C4 / C5 L = 20 size: the query-sharded runs of
    G = 1, 2, 4, 8 ranks (one pipeline per rank's MEM-start range, as bench.py --gpus G
    runs them; here all on one device) merge (K9, merge.cu) to the byte-identical whole
    set of the single pipeline."""
    P = c4_full
    Rt, Qt = torch.from_numpy(P.R).cuda(), torch.from_numpy(P.Q).cuda()
    from paper_conf_ipps_abu_dolehkac14_b200.dist import shard_range
    pl = gpumem.Pipeline(len(P.R), len(P.Q), P.ls, L)
    pl.run(Rt, Qt)
    pl.result()
    whole = pl.numpy()
    pl.free()
    assert len(whole) == {100: 811662, 20: 13420345}[L]
    for G in (2, 4, 8):
        runs = []
        for g in range(G):
            pl = gpumem.Pipeline(len(P.R), len(P.Q), P.ls, L, shard_range(len(P.Q), g, G))
            pl.run(Rt, Qt)
            pl.result()
            runs.append(pl.view_u32().clone())
            pl.free()
        merged = gpumem.merge_sorted([r.view(torch.int32) for r in runs])
        got = merged.numpy()
        merged.free()
        assert got.tobytes() == whole.tobytes(), G


@pytest.mark.slow
@pytest.mark.parametrize("L,band", [(100, 64_000_000), (20, 16_000_000)])
def test_full_size_band_sweep(c4_full, L, band):
    """F2 at the full C4 / C5 L = 20 size: the row sweep over a host-resident R with a
    16-64 Mbp window equals the whole-R pipeline result (itself bit-exact against the
    oracle in test_full_size_c4_c5)."""
    P = c4_full
    Rt, Qt = torch.from_numpy(P.R).cuda(), torch.from_numpy(P.Q).cuda()
    pl = gpumem.Pipeline(len(P.R), len(P.Q), P.ls, L)
    pl.run(Rt, Qt)
    pl.result()
    whole = pl.numpy()
    pl.free()
    m, st = gpumem.find_mems_banded(P.R, gpumem.pack(Qt), P.ls, L, band)
    assert st["bands"] > 1 and st["window_bytes"] < len(P.R) // 3
    assert m.numpy().tobytes() == whole.tobytes()


@pytest.mark.slow
@pytest.mark.parametrize("L", [100, 20])
def test_full_size_streamed_query(c4_full, L):
    """The host-input pipeline with Q streamed in 8 pieces at the full C4 / C5 L = 20 size
    equals the device-input pipeline byte for byte."""
    P = c4_full
    Rt, Qt = torch.from_numpy(P.R).cuda(), torch.from_numpy(P.Q).cuda()
    pl = gpumem.Pipeline(len(P.R), len(P.Q), P.ls, L)
    pl.run(Rt, Qt)
    pl.result()
    whole = pl.numpy()
    pl.free()
    pl = gpumem.Pipeline(len(P.R), len(P.Q), P.ls, L)
    for _ in range(2):
        pl.run_host(torch.from_numpy(P.R).pin_memory(), torch.from_numpy(P.Q).pin_memory())
        pl.result()
        assert pl.numpy().tobytes() == whole.tobytes()
    pl.free()


# ------------------------------------------------------------------ NEXT rows
def _rc(b):
    return bytes(b)[::-1].translate(bytes.maketrans(b"ACGTacgt", b"TGCAtgca"))


@pytest.mark.parametrize("cfg,scale,bands", [("c1", 1.0, 3), ("c2", 0.1, 5), ("c4", 0.02, 7)])
def test_band_index_union_is_whole(cfg, scale, bands):
    """F2: partial index per band of R: bands partition the MEM set."""
    P = synth.make_pair(cfg, scale=scale)
    Rs, Qs = gpumem.pack(P.R), gpumem.pack(P.Q)
    whole = gpumem.find_mems(gpumem.index_build(Rs, P.ls, P.L), Qs).numpy()
    n = len(P.R)
    cuts = [n * b // bands for b in range(bands + 1)]
    parts = [gpumem.find_mems(gpumem.index_build(Rs, P.ls, P.L, r_range=(a, b)), Qs).numpy()
             for a, b in zip(cuts[:-1], cuts[1:])]
    cat = np.concatenate(parts)
    cat = cat[np.lexsort((cat[:, 1], cat[:, 0]))]
    assert np.array_equal(cat, whole)                       # disjoint, complete
    assert np.array_equal(whole, oracle.mems(P.R, P.Q, P.L, P.ls))


@pytest.mark.parametrize("cfg,scale,band", [("c1", 1.0, 7000), ("c1", 1.0, 0), ("c2", 0.1, 50_000),
                                            ("c4", 0.02, 1_000_000), ("c5_l20", 0.02, 333_333), ("c3", 0.03, 80_000)])
def test_band_sweep_equals_whole(cfg, scale, band):
    """F2 row sweep with a band-local R window: only one window of
    R on the device, MEMs cut at a window's end carried to the next band -- the same set
    as the whole-R path and the oracle."""
    P = synth.make_pair(cfg, scale=scale)
    want = oracle.mems(P.R, P.Q, P.L, P.ls)
    Q = gpumem.pack(P.Q)
    m, st = gpumem.find_mems_banded(P.R, Q, P.ls, P.L, band)
    assert np.array_equal(m.numpy(), want), st
    if band:
        assert st["bands"] == -(-len(P.R) // st["band_len"]) and st["window_bytes"] < len(P.R)


def test_band_sweep_long_matches_cross_many_windows():
    """Homopolymers and a self-match: MEMs far longer than a band run through many
    windows (carried and continued band after band), against the closed form."""
    for n, m_, L, ls, band in ((20_000, 9_000, 30, 10, 2_100), (5_000, 5_000, 20, 13, 800), (3_000, 40_000, 1, 1, 64)):
        want = np.array(pyoracle.homopolymer(n, m_, L), dtype=np.uint32).reshape(-1, 3)
        got, st = gpumem.find_mems_banded("A" * n, gpumem.pack("A" * m_), ls, L, band)
        assert np.array_equal(got.numpy(), want), (n, m_, L, band)
        assert st["carried"] > 0
    P = synth.make_pair("c1", scale=0.5)
    got, st = gpumem.find_mems_banded(P.R, gpumem.pack(P.R), P.ls, P.L, 3000)
    assert (0, 0, len(P.R)) in {tuple(t) for t in got.numpy().tolist()} and st["carried"] > 0
    assert np.array_equal(got.numpy(), oracle.mems(P.R, P.R, P.L, P.ls))


@pytest.mark.parametrize("n", [1, 31, 32, 33, 100, 4097])
def test_revcomp_words(n):
    rng = np.random.default_rng(n)
    s = synth.to_ascii(rng.integers(0, 4, n).astype(np.uint8)).tobytes()
    rc = gpumem.revcomp(gpumem.pack(s))
    direct = gpumem.pack(_rc(s))
    assert np.array_equal(rc.words().cpu().numpy(), direct.words().cpu().numpy())


@pytest.mark.parametrize("cfg,scale", [("c1", 1.0), ("c4", 0.02)])
def test_reverse_strand_mems(cfg, scale):
    """F4: MEMs between R and the reverse complement of Q."""
    P = synth.make_pair(cfg, scale=scale)
    Q_rc = _rc(P.Q.tobytes())
    idx = gpumem.index_build(gpumem.pack(P.R), P.ls, P.L)
    got = gpumem.find_mems(idx, gpumem.revcomp(gpumem.pack(P.Q))).numpy()
    assert np.array_equal(got, oracle.mems(P.R, Q_rc, P.L, P.ls))


@pytest.mark.parametrize("cfg,scale,L", [("c1", 1.0, 20), ("c1", 0.3, 12), ("c3", 0.01, 50), ("c4", 0.01, 40)])
def test_mums(cfg, scale, L):
    """F3: MUMs = MEMs unique in both sequences, vs the substring-count oracle."""
    P = synth.make_pair(cfg, scale=scale)
    ls = min(P.ls, L)
    m = gpumem.find_mems(gpumem.index_build(gpumem.pack(P.R), ls, L), gpumem.pack(P.Q))
    got = gpumem.mums(m).numpy()
    want = oracle.mums(P.R, P.Q, L, ls)
    assert np.array_equal(got, want)
    assert len(want) > 0


def test_mums_tiny_random():
    rng = np.random.default_rng(5)
    for trial in range(80):
        R, Q = synth.random_pair(rng, int(rng.integers(2, 150)), int(rng.integers(2, 150)),
                                 [b"AC", b"ACG", b"ACGT"][trial % 3])
        L = int(rng.integers(2, 12))
        ls = int(rng.integers(1, L + 1))
        m = gpumem.find_mems(gpumem.index_build(gpumem.pack(R.tobytes()), min(ls, 15), L), gpumem.pack(Q.tobytes()))
        assert np.array_equal(gpumem.mums(m).numpy(), oracle.mums(R, Q, L, min(ls, 15))), trial


@pytest.mark.parametrize("cfg,scale,L", [("c1", 1.0, 20), ("c3", 0.01, 30), ("c4", 0.005, 30)])
@pytest.mark.parametrize("k", [1, 2, 5, 15])
def test_rare(cfg, scale, L, k):
    """F3: rare MEMs (string occurs <= k times in R and in Q; R23) vs the
    substring-count oracle; k = 1 equals gpumem_mums."""
    P = synth.make_pair(cfg, scale=scale)
    ls = min(P.ls, L)
    m = gpumem.find_mems(gpumem.index_build(gpumem.pack(P.R), ls, L), gpumem.pack(P.Q))
    got = gpumem.rare(m, k).numpy()
    want = oracle.rare(P.R, P.Q, L, ls, k)
    assert np.array_equal(got, want)
    if k == 1:
        assert np.array_equal(got, gpumem.mums(m).numpy())


def test_rare_golden_homopolymer_and_tiny():
    g = read_golden("w3_rare.txt")
    for k in (1, 2):
        m = gpumem.find_mems(gpumem.index_build(gpumem.pack(g["R"]), 2, g["L"]), gpumem.pack(g["Q"]))
        assert [tuple(t) for t in gpumem.rare(m, k).numpy().tolist()] == sorted(g[f"k{k}"])
    for n, mm, L, k in ((300, 200, 20, 1), (300, 200, 20, 100 // 10), (500, 520, 480, 15), (64, 64, 8, 7)):
        m = gpumem.find_mems(gpumem.index_build(gpumem.pack("A" * n), min(L, 13), L), gpumem.pack("A" * mm))
        want = [t for t in pyoracle.homopolymer(n, mm, L) if n - t[2] + 1 <= k and mm - t[2] + 1 <= k]
        assert [tuple(t) for t in gpumem.rare(m, k).numpy().tolist()] == want, (n, mm, L, k)
    rng = np.random.default_rng(6)
    for trial in range(80):
        R, Q = synth.random_pair(rng, int(rng.integers(2, 150)), int(rng.integers(2, 150)),
                                 [b"AC", b"ACG", b"ACGT"][trial % 3])
        L = int(rng.integers(2, 12))
        ls = min(int(rng.integers(1, L + 1)), 15)
        k = int(rng.integers(1, 16))
        m = gpumem.find_mems(gpumem.index_build(gpumem.pack(R.tobytes()), ls, L), gpumem.pack(Q.tobytes()))
        assert np.array_equal(gpumem.rare(m, k).numpy(), oracle.rare(R, Q, L, ls, k)), trial
    with pytest.raises(gpumem.GpumemError):
        gpumem.rare(m, 0)
    with pytest.raises(gpumem.GpumemError):
        gpumem.rare(m, 16)


@pytest.mark.slow
def test_full_size_c3():
    P = synth.make_pair("c3")
    want = oracle.mems(P.R, P.Q, P.L, P.ls)
    got = gpu_mems(P.R, P.Q, P.L, P.ls)
    assert np.array_equal(got, want)
    invariants.check(P.R, P.Q, P.L, got)
