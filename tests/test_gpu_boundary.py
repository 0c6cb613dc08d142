"""GPU tests of the boundary's ownership and error contract:
the allocator hook carries every device allocation (direct calls and the pipeline's
arena, workspaces and input staging), an allocator that returns NULL gives
GPUMEM_ERR_NOMEM with *out == NULL and nothing leaked, the pipeline graph's
workspaces are its own (gpumem_trim and the overflow fallback cannot free memory the
graph writes), and the find retry loop recovers coop-queue overflows."""
import numpy as np
import pytest

import oracle
from oracle import pyoracle
from paper_conf_ipps_abu_dolehkac14_b200 import synth

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # collected on CPU boxes, skipped there
    pytest.skip("needs a CUDA device", allow_module_level=True)

from paper_conf_ipps_abu_dolehkac14_b200 import gpumem  # noqa: E402


class CountingAllocator:
    """torch's caching allocator behind the hook, with a live-pointer ledger and an
    optional budget: allocation number `fail_at` (0-based) and every later one fail."""

    def __init__(self, fail_at=None):
        self.live, self.n_alloc, self.n_free, self.fail_at = {}, 0, 0, fail_at

    def alloc(self, n, s):
        k = self.n_alloc
        self.n_alloc += 1
        if self.fail_at is not None and k >= self.fail_at:
            return 0
        p = torch.cuda.caching_allocator_alloc(n, stream=torch.cuda.ExternalStream(s) if s else None)
        self.live[p] = n
        return p

    def free(self, p, s):
        assert p in self.live, "free of a pointer the hook never returned"
        del self.live[p]
        self.n_free += 1
        torch.cuda.caching_allocator_delete(p)

    def __enter__(self):
        gpumem.trim()  # workspaces allocated before the hook go back to their own allocator
        gpumem.set_allocator(self.alloc, self.free)
        return self

    def __exit__(self, *a):
        torch.cuda.synchronize()
        gpumem.trim()
        gpumem.set_allocator()
        torch.cuda.synchronize()


@pytest.fixture(autouse=True)
def _defaults():
    yield
    gpumem.set_allocator()
    gpumem.set_option("out_capacity", 0)


def _dev(b):
    return torch.from_numpy(np.frombuffer(bytes(b), dtype=np.uint8).copy()).cuda()


def test_hook_carries_direct_calls_and_pipeline():
    P = synth.make_pair("c2", scale=0.2)
    want = oracle.mems(P.R, P.Q, P.L, P.ls)
    with CountingAllocator() as A:
        assert np.array_equal(gpumem.mems(P.R.tobytes(), P.Q.tobytes(), P.L, P.ls), want)
        n_direct = A.n_alloc
        assert n_direct > 0
        R, Q = _dev(P.R.tobytes()), _dev(P.Q.tobytes())
        pl = gpumem.Pipeline(len(P.R), len(P.Q), P.ls, P.L)
        for _ in range(2):
            pl.run(R, Q)
            pl.result()
            assert np.array_equal(pl.numpy(), want)
        # host-input runs stage R and Q in a buffer from the hook too
        Rh, Qh = torch.from_numpy(P.R).pin_memory(), torch.from_numpy(P.Q).pin_memory()
        pl.run_host(Rh, Qh)
        pl.result()
        assert np.array_equal(pl.numpy(), want)
        assert A.n_alloc > n_direct  # arena (+ measuring-run buffers) + staging
        pl.free()
    assert A.live == {}, f"{len(A.live)} allocations leaked"


@pytest.mark.parametrize("path", ["direct", "pipeline"])
def test_null_allocator_is_nomem_and_leaks_nothing(path):
    """An allocator that fails from the k-th request on, for every k up to the number of
    allocations the call makes: each call either succeeds (bit-exact) or returns
    GPUMEM_ERR_NOMEM with no handle, and after trim nothing the hook handed out is live."""
    P = synth.make_pair("c1", scale=0.3)
    want = oracle.mems(P.R, P.Q, P.L, P.ls)
    with CountingAllocator() as A:  # count the allocations of one successful call
        if path == "direct":
            gpumem.mems(P.R.tobytes(), P.Q.tobytes(), P.L, P.ls)
        else:
            R, Q = _dev(P.R.tobytes()), _dev(P.Q.tobytes())
            pl = gpumem.Pipeline(len(P.R), len(P.Q), P.ls, P.L)
            pl.run(R, Q)
            pl.result()
            pl.free()
    total = A.n_alloc
    assert total > 3 and A.live == {}
    failures = 0
    for k in range(total + 1):
        with CountingAllocator(fail_at=k) as A:
            try:
                if path == "direct":
                    got = gpumem.mems(P.R.tobytes(), P.Q.tobytes(), P.L, P.ls)
                else:
                    pl = gpumem.Pipeline(len(P.R), len(P.Q), P.ls, P.L)
                    try:
                        pl.run(R, Q)
                        pl.result()
                        got = pl.numpy()
                    finally:
                        pl.free()
                assert np.array_equal(got, want), k
            except gpumem.GpumemError as e:
                assert e.name == "ERR_NOMEM", (k, str(e))
                failures += 1
        assert A.live == {}, (k, f"{len(A.live)} allocations leaked after NOMEM")
    assert failures >= total - 1  # every truncated budget failed cleanly


def test_nomem_sets_out_null():
    import ctypes
    gpumem.set_allocator(lambda n, s: 0, lambda p, s: None)
    gpumem.trim()
    out = ctypes.c_void_p(12345)
    st = gpumem._lib.gpumem_pack(b"ACGT" * 100, 400, 0, None, ctypes.byref(out))
    assert st == 4 and out.value is None
    assert b"allocator hook returned NULL" in gpumem._lib.gpumem_last_error()
    gpumem.set_allocator()


def test_pipeline_workspaces_survive_trim_and_fallback():
    """the captured graph used the per-stream workspaces, which the
    overflow fallback grows (frees + reallocates) and gpumem_trim frees. Now they are
    slices of the pipeline's arena: forced overflow -> fallback, trim, other work that
    reuses freed memory, relaunch -- every result bit-exact."""
    P = synth.make_pair("c1")
    want = oracle.mems(P.R, P.Q, P.L, P.ls)
    R, Q = _dev(P.R.tobytes()), _dev(P.Q.tobytes())
    gpumem.set_option("out_capacity", 64)  # read at capture (the first run): every graph run overflows
    pl = gpumem.Pipeline(len(P.R), len(P.Q), P.ls, P.L)
    for i in range(4):
        pl.run(R, Q)
        gpumem.set_option("out_capacity", 0)
        pl.result()
        assert pl.stats()["attempts"] >= 2
        assert np.array_equal(pl.numpy(), want), i
        gpumem.trim()
        junk = gpumem.mems(P.Q.tobytes(), P.R.tobytes(), P.L, P.ls)  # reuses freed pool memory
        assert len(junk) == len(want)
    pl.free()
    pl2 = gpumem.Pipeline(len(P.R), len(P.Q), P.ls, P.L)  # no overflow: graph path, then trim
    for _ in range(3):
        pl2.run(R, Q)
        pl2.result()
        assert pl2.stats()["attempts"] == 1 and np.array_equal(pl2.numpy(), want)
        gpumem.trim()
        gpumem.mems(P.R.tobytes()[: 50000], P.Q.tobytes()[: 50000], P.L, P.ls)
    pl2.free()


@pytest.mark.parametrize("n,L,ls", [(100_000, 20, 10), (60_000, 50, 13)])
def test_coop_queue_overflow_recovers(n, L, ls):
    """A^n vs A^n gives ~2n MEMs, ~2(n - 4096) of them longer than one
    lane's extension cap -> far more coop-queue entries than its capacity (|Q|/64 + 4096).
    The retry must size the output for the dropped entries too; checked against the
    homopolymer closed form, through direct calls and the pipeline."""
    want = np.array(pyoracle.homopolymer(n, n, L), dtype=np.uint32).reshape(-1, 3)
    assert len(want) > 100_000
    got = gpumem.mems("A" * n, "A" * n, L, ls)
    assert np.array_equal(got, want)
    R = _dev(b"A" * n)
    pl = gpumem.Pipeline(n, n, ls, L)
    pl.run(R, R)
    pl.result()
    assert np.array_equal(pl.numpy(), want)
    assert pl.stats()["attempts"] >= 2  # the graph's coop queue overflowed: the fallback ran
    pl.free()
