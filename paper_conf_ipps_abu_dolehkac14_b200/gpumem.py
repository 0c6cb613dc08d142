"""Thin Python binding over libgpumem.so (C ABI: include/gpumem.h).

Argument marshalling only: every step of the MEM path runs in the library's
CUDA kernels. PyTorch is used for device buffers and the current CUDA stream.
Importing this module fails loudly if the CUDA library has not been built --
there is no CPU fallback.

    import paper_conf_ipps_abu_dolehkac14_b200.gpumem as gm
    R = gm.pack(r_bytes)                     # bytes/numpy (host) or uint8 CUDA tensor
    Q = gm.pack(q_bytes)
    idx = gm.index_build(R, seed_len=13, min_len=100)
    mems = gm.find_mems(idx, Q)              # sorted by (r, q)
    mems.numpy()                             # (N, 3) uint32 [r, q, len] on the host
    mems.tensor()                            # (N, 3) int64 CUDA tensor (copy)
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
# GPUMEM_LIB: an alternative build of the same library (tuning experiments, tools/variants.py)
LIB_PATH = os.environ.get("GPUMEM_LIB") or os.path.join(_PKG, "libgpumem.so")
if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: build it with `python -m paper_conf_ipps_abu_dolehkac14_b200._build` "
                      "(the MEM path is CUDA-only; there is no CPU fallback)")
_lib = ctypes.CDLL(LIB_PATH)

_c_u64, _c_u32, _vp = ctypes.c_uint64, ctypes.c_uint32, ctypes.c_void_p
_P = ctypes.POINTER

SYMBOLS = {
    # name: (restype, argtypes)
    "gpumem_pack": (ctypes.c_int, [ctypes.c_void_p, _c_u64, ctypes.c_int, _vp, _P(_vp)]),
    "gpumem_seq_check": (ctypes.c_int, [_vp, _vp]),
    "gpumem_revcomp": (ctypes.c_int, [_vp, _vp, _P(_vp)]),
    "gpumem_seq_info": (ctypes.c_int, [_vp, _P(_c_u64), _P(_vp), _P(_c_u64)]),
    "gpumem_index_build": (ctypes.c_int, [_vp, _c_u32, _c_u32, _vp, _P(_vp)]),
    "gpumem_index_build_step": (ctypes.c_int, [_vp, _c_u32, _c_u32, _c_u32, _vp, _P(_vp)]),
    "gpumem_index_build_range": (ctypes.c_int, [_vp, _c_u32, _c_u32, _c_u64, _c_u64, _vp, _P(_vp)]),
    "gpumem_index_view": (ctypes.c_int, [_vp, _P(_vp), _P(_vp), _P(_c_u64)]),
    "gpumem_find_mems": (ctypes.c_int, [_vp, _vp, _c_u64, _c_u64, _vp, _P(_vp)]),
    "gpumem_mems_view": (ctypes.c_int, [_vp, _P(_vp), _P(_c_u64)]),
    "gpumem_mems_to_host": (ctypes.c_int, [_vp, _vp, _c_u64]),
    "gpumem_mems_stats": (ctypes.c_int, [_vp, _vp]),
    "gpumem_mums": (ctypes.c_int, [_vp, _vp, _P(_vp)]),
    "gpumem_rare": (ctypes.c_int, [_vp, _c_u32, _vp, _P(_vp)]),
    "gpumem_merge_sorted": (ctypes.c_int, [_P(_vp), _P(_c_u64), ctypes.c_int, _vp, _P(_vp)]),
    "gpumem_pipeline_create": (ctypes.c_int, [_c_u64, _c_u64, _c_u32, _c_u32, _c_u64, _c_u64, _vp, _P(_vp)]),
    "gpumem_pipeline_run": (ctypes.c_int, [_vp, _vp, _vp]),
    "gpumem_pipeline_run_host": (ctypes.c_int, [_vp, _vp, _vp]),
    "gpumem_pipeline_result": (ctypes.c_int, [_vp, _P(_vp), _P(_c_u64)]),
    "gpumem_pipeline_stats": (ctypes.c_int, [_vp, _vp]),
    "gpumem_pipeline_profile": (ctypes.c_int, [_vp, _P(ctypes.c_char_p), _P(ctypes.c_double), _P(_c_u64),
                                               ctypes.c_int]),
    "gpumem_pipeline_set_exportable": (ctypes.c_int, [_vp, ctypes.c_int]),
    "gpumem_pipeline_export": (ctypes.c_int, [_vp, _vp, _P(_c_u64), _P(_c_u64)]),
    "gpumem_ipc_open": (ctypes.c_int, [_vp, _P(_vp)]),
    "gpumem_ipc_close": (ctypes.c_int, [_vp]),
    "gpumem_fasta_parse": (ctypes.c_int, [ctypes.c_char_p, _c_u64, _P(_vp)]),
    "gpumem_fasta_info": (ctypes.c_int, [_vp, _P(_c_u64), _P(_vp), _P(_c_u64), _P(_c_u64)]),
    "gpumem_fasta_record": (ctypes.c_int, [_vp, _c_u64, _P(ctypes.c_char_p), _P(_c_u64), _P(_c_u64)]),
    "gpumem_split_masked": (ctypes.c_int, [_vp, _vp, _vp, _c_u32, ctypes.c_int, _vp, _P(_vp)]),
    "gpumem_write_mummer": (ctypes.c_int, [_vp, _c_u64, _vp, _c_u64, _vp, _vp, ctypes.c_char_p]),
    "gpumem_find_mems_banded": (ctypes.c_int, [_vp, _c_u64, _vp, _c_u32, _c_u32, _c_u64, _vp, _P(_vp), _vp]),
    "gpumem_free": (None, [_vp]),
    "gpumem_trim": (ctypes.c_int, []),
    "gpumem_last_error": (ctypes.c_char_p, []),
    "gpumem_set_allocator": (ctypes.c_int, [_vp, _vp, _vp]),
    "gpumem_set_option": (ctypes.c_int, [ctypes.c_char_p, ctypes.c_int64]),
    "gpumem_profile_enable": (ctypes.c_int, [ctypes.c_int]),
    "gpumem_profile_read": (ctypes.c_int, [_P(ctypes.c_char_p), _P(ctypes.c_double), _P(_c_u64), ctypes.c_int]),
    "gpumem_launch_count": (_c_u64, []),
    "gpumem_gather_ceiling": (ctypes.c_int, [_c_u64, _c_u64, _vp, _P(ctypes.c_double)]),
    "gpumem_version": (ctypes.c_char_p, []),
}
for _name, (_res, _args) in SYMBOLS.items():
    _f = getattr(_lib, _name)
    _f.restype = _res
    _f.argtypes = _args

STATUS = {0: "OK", 1: "ERR_ARG", 2: "ERR_ALPHABET", 3: "ERR_RANGE", 4: "ERR_NOMEM", 5: "ERR_CUDA",
          6: "ERR_UNSUPPORTED"}


class FindStats(ctypes.Structure):
    _fields_ = [("positions", _c_u64), ("occupied", _c_u64), ("hits", _c_u64), ("spilled_chunks", _c_u64),
                ("mems", _c_u64), ("attempts", _c_u32), ("max_warp_hits", _c_u64), ("warps", _c_u64)]

    def as_dict(self):
        return {k: int(getattr(self, k)) for k, _ in self._fields_}


class GpumemError(RuntimeError):
    def __init__(self, status, message):
        super().__init__(f"{STATUS.get(status, status)}: {message}")
        self.status = status
        self.name = STATUS.get(status, str(status))


def _check(st):
    if st != 0:
        raise GpumemError(st, (_lib.gpumem_last_error() or b"").decode())


def _stream(stream=None):
    if stream is not None:
        return ctypes.c_void_p(int(stream))
    import torch
    return ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)


class _Handle:
    __slots__ = ("_h", "_keep", "__weakref__")

    def __init__(self, h, keep=None):
        self._h = h
        self._keep = keep

    @property
    def handle(self):
        if not self._h:
            raise GpumemError(1, "handle already freed")
        return self._h

    def free(self):
        if self._h:
            _lib.gpumem_free(self._h)
            self._h = None
        self._keep = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


class Seq(_Handle):
    """A 2-bit packed sequence on the current device."""

    def info(self):
        n, w, nw = _c_u64(), _vp(), _c_u64()
        _check(_lib.gpumem_seq_info(self.handle, ctypes.byref(n), ctypes.byref(w), ctypes.byref(nw)))
        return n.value, w.value, nw.value

    def __len__(self):
        return self.info()[0]

    def check(self, stream=None):
        _check(_lib.gpumem_seq_check(self.handle, _stream(stream)))

    def words(self):
        """Packed words as a uint64 CUDA tensor view (borrowed from the handle)."""
        n, ptr, nw = self.info()
        return _device_view(ptr, (nw,), "<u8", self)


class Index(_Handle):
    def view(self):
        """(ptrs, locs) as uint32 CUDA tensor views (borrowed)."""
        p, l, n = _vp(), _vp(), _c_u64()
        _check(_lib.gpumem_index_view(self.handle, ctypes.byref(p), ctypes.byref(l), ctypes.byref(n)))
        ls = self._keep[1]
        return (_device_view(p.value, ((1 << (2 * ls)) + 1,), "<u4", self),
                _device_view(l.value, (n.value,), "<u4", self))


class Mems(_Handle):
    def view(self):
        ptr, cnt = _vp(), _c_u64()
        _check(_lib.gpumem_mems_view(self.handle, ctypes.byref(ptr), ctypes.byref(cnt)))
        return ptr.value, cnt.value

    def __len__(self):
        return self.view()[1]

    def stats(self):
        s = FindStats()
        _check(_lib.gpumem_mems_stats(self.handle, ctypes.byref(s)))
        return s.as_dict()

    def numpy(self):
        """(N, 3) uint32 [r, q, len] copied to the host (synchronous)."""
        _, n = self.view()
        out = np.empty((n, 3), dtype=np.uint32)
        _check(_lib.gpumem_mems_to_host(self.handle, out.ctypes.data_as(_vp), n))
        return out

    def view_u32(self):
        """(N, 3) uint32 CUDA tensor view (borrowed from the handle)."""
        ptr, n = self.view()
        return _device_view(ptr, (n, 3), "<u4", self)

    def tensor(self):
        """(N, 3) int64 CUDA tensor (copy)."""
        return self.view_u32().to(dtype=__import__("torch").int64)


class _CudaArray:
    def __init__(self, ptr, shape, typestr, owner):
        self.__cuda_array_interface__ = {"shape": shape, "typestr": typestr, "data": (ptr or 0, False),
                                         "version": 3, "strides": None, "stream": None}
        self._owner = owner


def _device_view(ptr, shape, typestr, owner):
    import torch
    if int(np.prod(shape)) == 0:
        dt = {"<u4": torch.uint32, "<u8": torch.uint64}[typestr]
        return torch.empty(shape, dtype=dt, device="cuda")
    return torch.as_tensor(_CudaArray(ptr, shape, typestr, owner), device="cuda")


def pack(x, stream=None) -> Seq:
    """2-bit encode `x`: a uint8 CUDA tensor (read in place), or host bytes/str/numpy/CPU tensor."""
    h = _vp()
    keep = None
    try:
        import torch
        is_tensor = isinstance(x, torch.Tensor)
    except ImportError:  # pragma: no cover
        is_tensor = False
    if is_tensor and x.is_cuda:
        if x.dtype != __import__("torch").uint8:
            raise TypeError("device input must be a uint8 tensor")
        x = x.contiguous()
        keep = x
        _check(_lib.gpumem_pack(_vp(x.data_ptr()), x.numel(), 1, _stream(stream), ctypes.byref(h)))
    else:
        if is_tensor:
            arr = x.contiguous().numpy()
        elif isinstance(x, str):
            arr = np.frombuffer(x.encode("ascii"), dtype=np.uint8)
        elif isinstance(x, (bytes, bytearray, memoryview)):
            arr = np.frombuffer(bytes(x), dtype=np.uint8)
        else:
            arr = np.ascontiguousarray(x, dtype=np.uint8)
        keep = arr
        _check(_lib.gpumem_pack(arr.ctypes.data_as(_vp), arr.size, 0, _stream(stream), ctypes.byref(h)))
    return Seq(h.value, keep)


def revcomp(S: Seq, stream=None) -> Seq:
    """Packed reverse complement of S (for reverse-strand MEMs)."""
    h = _vp()
    _check(_lib.gpumem_revcomp(S.handle, _stream(stream), ctypes.byref(h)))
    return Seq(h.value, S)


def index_build(R: Seq, seed_len: int, min_len: int, step: int | None = None, stream=None,
                r_range=None) -> Index:
    """Index of R (Alg. 1). r_range=(r_begin, r_end) builds the partial index of one band."""
    h = _vp()
    if r_range is not None:
        if step is not None:
            raise ValueError("step and r_range are exclusive")
        _check(_lib.gpumem_index_build_range(R.handle, seed_len, min_len, int(r_range[0]), int(r_range[1]),
                                             _stream(stream), ctypes.byref(h)))
    elif step is None:
        _check(_lib.gpumem_index_build(R.handle, seed_len, min_len, _stream(stream), ctypes.byref(h)))
    else:
        _check(_lib.gpumem_index_build_step(R.handle, seed_len, min_len, step, _stream(stream), ctypes.byref(h)))
    return Index(h.value, (R, seed_len))


def find_mems(idx: Index, Q: Seq, q_range=None, stream=None) -> Mems:
    qb, qe = (0, (1 << 64) - 1) if q_range is None else (int(q_range[0]), int(q_range[1]))
    h = _vp()
    _check(_lib.gpumem_find_mems(idx.handle, Q.handle, qb, qe, _stream(stream), ctypes.byref(h)))
    return Mems(h.value, (idx, Q))


def mums(m: Mems, stream=None) -> Mems:
    """Maximal unique matches: the MEMs of `m` unique in both sequences (order kept)."""
    h = _vp()
    _check(_lib.gpumem_mums(m.handle, _stream(stream), ctypes.byref(h)))
    return Mems(h.value, m)


def ipc_open(handle: bytes) -> int:
    """Map another process's exported pipeline arena; returns its device base address."""
    h = (ctypes.c_ubyte * 64).from_buffer_copy(handle)
    base = _vp()
    _check(_lib.gpumem_ipc_open(ctypes.byref(h), ctypes.byref(base)))
    return base.value


def ipc_close(base: int):
    _check(_lib.gpumem_ipc_close(_vp(base)))


def merge_runs(ptrs, counts, stream=None) -> Mems:
    """K9 merge of raw device runs (pointers to counts[i] triples, e.g. IPC-mapped peer
    memory), each sorted by (r, q) and pairwise disjoint."""
    p = (_vp * max(1, len(ptrs)))(*[_vp(int(x)) for x in ptrs])
    c = (_c_u64 * max(1, len(ptrs)))(*[int(x) for x in counts])
    h = _vp()
    _check(_lib.gpumem_merge_sorted(p, c, len(ptrs), _stream(stream), ctypes.byref(h)))
    return Mems(h.value)


class Fasta(_Handle):
    """A parsed multi-FASTA (gpumem_fasta_parse): records concatenated with one masked
    separator base, non-ACGT letters masked."""

    def info(self):
        nrec, ptr, n, nm = _c_u64(), _vp(), _c_u64(), _c_u64()
        _check(_lib.gpumem_fasta_info(self.handle, ctypes.byref(nrec), ctypes.byref(ptr), ctypes.byref(n),
                                      ctypes.byref(nm)))
        return nrec.value, ptr.value, n.value, nm.value

    def seq(self) -> np.ndarray:
        """The concatenated ASCII sequence (a copy)."""
        _, ptr, n, _ = self.info()
        return np.ctypeslib.as_array((ctypes.c_uint8 * n).from_address(ptr)).copy() if n else \
            np.zeros(0, np.uint8)

    def records(self):
        """[(name, start, length)] in input order."""
        out = []
        for i in range(self.info()[0]):
            nm, st, ln = ctypes.c_char_p(), _c_u64(), _c_u64()
            _check(_lib.gpumem_fasta_record(self.handle, i, ctypes.byref(nm), ctypes.byref(st), ctypes.byref(ln)))
            out.append((nm.value.decode(), st.value, ln.value))
        return out


def fasta_parse(text) -> Fasta:
    b = text.encode() if isinstance(text, str) else bytes(text)
    h = _vp()
    _check(_lib.gpumem_fasta_parse(b, len(b), ctypes.byref(h)))
    return Fasta(h.value)


def split_masked(m: Mems, R: Fasta, Q: Fasta, min_len: int, q_reverse=False, stream=None) -> Mems:
    """The multi-record MEMs: m (MEMs of the concatenations) cut at masked positions."""
    h = _vp()
    _check(_lib.gpumem_split_masked(m.handle, R.handle, Q.handle, int(min_len), 1 if q_reverse else 0,
                                    _stream(stream), ctypes.byref(h)))
    return Mems(h.value, (m, R, Q))


def write_mummer(path, fwd, R: Fasta, Q: Fasta, rev=None):
    """MUMmer-style text (1-based, per query record) from host (N, 3) uint32 triples."""
    f = np.ascontiguousarray(fwd, dtype=np.uint32)
    r = None if rev is None else np.ascontiguousarray(rev, dtype=np.uint32)
    _check(_lib.gpumem_write_mummer(f.ctypes.data_as(_vp) if len(f) else None, len(f),
                                    (r.ctypes.data_as(_vp) if len(r) else _vp(1)) if r is not None else None,
                                    0 if r is None else len(r), R.handle, Q.handle, str(path).encode()))


class BandStats(ctypes.Structure):
    _fields_ = [("bands", _c_u64), ("band_len", _c_u64), ("window_bytes", _c_u64), ("carried", _c_u64),
                ("mems", _c_u64)]

    def as_dict(self):
        return {k: int(getattr(self, k)) for k, _ in self._fields_}


def find_mems_banded(R_host, Q: Seq, seed_len: int, min_len: int, band_len: int, stream=None):
    """Row sweep over bands of a host-resident R (only one window of R on the device);
    returns (Mems, stats dict). Same MEM set as find_mems on the whole of R."""
    a = np.ascontiguousarray(np.frombuffer(R_host.encode(), np.uint8) if isinstance(R_host, str)
                             else (np.frombuffer(bytes(R_host), np.uint8)
                                   if isinstance(R_host, (bytes, bytearray)) else R_host), dtype=np.uint8)
    h = _vp()
    st = BandStats()
    _check(_lib.gpumem_find_mems_banded(a.ctypes.data_as(_vp), a.size, Q.handle, int(seed_len), int(min_len),
                                        int(band_len), _stream(stream), ctypes.byref(h), ctypes.byref(st)))
    return Mems(h.value, Q), st.as_dict()


def rare(m: Mems, k: int, stream=None) -> Mems:
    """MEMs whose string occurs at most k times in R and in Q (k = 1: MUMs), (r, q) order."""
    h = _vp()
    _check(_lib.gpumem_rare(m.handle, int(k), _stream(stream), ctypes.byref(h)))
    return Mems(h.value, m)


def merge_sorted(runs, stream=None) -> Mems:
    """Merge device runs of triples, each sorted by (r, q). `runs`: list of (N_i, 3) uint32/int32 CUDA tensors."""
    ptrs = (_vp * max(1, len(runs)))(*[_vp(r.data_ptr()) for r in runs])
    cnts = (_c_u64 * max(1, len(runs)))(*[r.shape[0] for r in runs])
    h = _vp()
    _check(_lib.gpumem_merge_sorted(ptrs, cnts, len(runs), _stream(stream), ctypes.byref(h)))
    return Mems(h.value, list(runs))


class Pipeline(_Handle):
    """The whole path for fixed sizes as one CUDA graph (gpumem_pipeline_*).

        pl = gm.Pipeline(len(R), len(Q), seed_len=13, min_len=100)
        pl.run(R_dev, Q_dev)      # async: one graph launch (captured on the first call)
        n = pl.result()           # sync; MEM count (same set as find_mems)
        pl.view_u32()             # (n, 3) uint32 CUDA view, valid until the next run
    """

    def __init__(self, r_len, q_len, seed_len, min_len, q_range=None, stream=None):
        qb, qe = (0, (1 << 64) - 1) if q_range is None else (int(q_range[0]), int(q_range[1]))
        h = _vp()
        _check(_lib.gpumem_pipeline_create(int(r_len), int(q_len), seed_len, min_len, qb, qe, _stream(stream),
                                           ctypes.byref(h)))
        super().__init__(h.value)
        self._inputs = None
        self._ptr, self._n = None, 0

    def run(self, R_dev, Q_dev):
        """R_dev, Q_dev: uint8 CUDA tensors of the sizes given at creation (kept alive
        until the next run)."""
        import torch
        for x in (R_dev, Q_dev):
            if not (isinstance(x, torch.Tensor) and x.is_cuda and x.dtype == torch.uint8 and x.is_contiguous()):
                raise TypeError("pipeline inputs must be contiguous uint8 CUDA tensors")
        self._inputs = (R_dev, Q_dev)
        self._ptr = None
        _check(_lib.gpumem_pipeline_run(self.handle, _vp(R_dev.data_ptr()), _vp(Q_dev.data_ptr())))

    def run_host(self, R_host, Q_host):
        """R_host, Q_host: host uint8 buffers (numpy arrays or CPU tensors; pinned for full
        PCIe speed) of the sizes given at creation, kept alive until the next run. The
        copies overlap the R half of the path (pack + index)."""
        import torch
        keep = []
        for x in (R_host, Q_host):
            if isinstance(x, torch.Tensor):
                if x.is_cuda or x.dtype != torch.uint8 or not x.is_contiguous():
                    raise TypeError("host inputs must be contiguous uint8 CPU tensors or numpy arrays")
                keep.append((x, x.data_ptr()))
            else:
                a = np.ascontiguousarray(x, dtype=np.uint8)
                keep.append((a, a.ctypes.data))
        self._inputs = tuple(k[0] for k in keep)
        self._ptr = None
        _check(_lib.gpumem_pipeline_run_host(self.handle, _vp(keep[0][1]), _vp(keep[1][1])))

    def result(self):
        ptr, n = _vp(), _c_u64()
        _check(_lib.gpumem_pipeline_result(self.handle, ctypes.byref(ptr), ctypes.byref(n)))
        self._ptr, self._n = ptr.value, n.value
        return self._n

    def __len__(self):
        if self._ptr is None:
            self.result()
        return self._n

    def view_u32(self):
        """(N, 3) uint32 CUDA view of the last result (borrowed; valid until the next run)."""
        if self._ptr is None:
            self.result()
        return _device_view(self._ptr, (self._n, 3), "<u4", self)

    def numpy(self):
        return self.view_u32().cpu().numpy()

    def set_exportable(self, on=True):
        """IPC-capable arena (cudaMalloc), so other processes can map the result."""
        _check(_lib.gpumem_pipeline_set_exportable(self.handle, 1 if on else 0))

    def export(self, handle=True):
        """(64-byte IPC handle or None, byte offset of the result triples, capture generation)."""
        h = (ctypes.c_ubyte * 64)()
        off, gen = _c_u64(), _c_u64()
        _check(_lib.gpumem_pipeline_export(self.handle, ctypes.byref(h) if handle else None, ctypes.byref(off),
                                           ctypes.byref(gen)))
        return (bytes(h) if handle else None), off.value, gen.value

    def stats(self):
        s = FindStats()
        _check(_lib.gpumem_pipeline_stats(self.handle, ctypes.byref(s)))
        return s.as_dict()

    def profile(self, max_stages=32):
        """Per-stage device ms of the last completed run: {name: (ms, launches)}."""
        names = (ctypes.c_char_p * max_stages)()
        ms = (ctypes.c_double * max_stages)()
        nl = (_c_u64 * max_stages)()
        n = _lib.gpumem_pipeline_profile(self.handle, names, ms, nl, max_stages)
        return {names[i].decode(): (ms[i], nl[i]) for i in range(n)}


def set_option(name: str, value: int):
    _check(_lib.gpumem_set_option(name.encode(), int(value)))


def profile_enable(on=True):
    _check(_lib.gpumem_profile_enable(1 if on else 0))


def profile_read(max_stages=32):
    names = (ctypes.c_char_p * max_stages)()
    ms = (ctypes.c_double * max_stages)()
    nl = (_c_u64 * max_stages)()
    n = _lib.gpumem_profile_read(names, ms, nl, max_stages)
    return {names[i].decode(): (ms[i], nl[i]) for i in range(n)}


ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)
FREE_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p)
_allocator_refs = None  # the ctypes callbacks must outlive their registration


def set_allocator(alloc=None, free=None):
    """Route every device allocation of the library through alloc(bytes, stream) -> ptr
    (0 = out of memory) and free(ptr, stream) (gpumem_set_allocator); no arguments
    restores the default stream-ordered pool. Handles allocated under one allocator
    must be freed under the same one."""
    global _allocator_refs
    if (alloc is None) != (free is None):
        raise ValueError("set both alloc and free, or neither")
    if alloc is None:
        _check(_lib.gpumem_set_allocator(None, None, None))
        _allocator_refs = None
        return
    a = ALLOC_FN(lambda n, s, ctx: alloc(int(n), s or 0) or None)
    f = FREE_FN(lambda ptr, s, ctx: free(ptr or 0, s or 0))
    _check(_lib.gpumem_set_allocator(ctypes.cast(a, _vp), ctypes.cast(f, _vp), None))
    _allocator_refs = (a, f)


def use_torch_allocator():
    """Allocate through torch's caching allocator (stream-ordered, on the calling stream)."""
    import torch

    def alloc(n, s):
        try:
            return torch.cuda.caching_allocator_alloc(n, stream=torch.cuda.ExternalStream(s) if s else None)
        except RuntimeError:  # torch.OutOfMemoryError
            return 0

    set_allocator(alloc, lambda p, s: torch.cuda.caching_allocator_delete(p))


def trim():
    """Release the library's per-stream workspaces (synchronises those streams)."""
    _check(_lib.gpumem_trim())


def gather_ceiling(n_probes: int, table_bytes: int, stream=None) -> float:
    """ms for n_probes random 8-byte loads into a table_bytes device table (k_find's ceiling)."""
    ms = ctypes.c_double()
    _check(_lib.gpumem_gather_ceiling(int(n_probes), int(table_bytes), _stream(stream), ctypes.byref(ms)))
    return ms.value


def launch_count() -> int:
    return int(_lib.gpumem_launch_count())


def version() -> str:
    return _lib.gpumem_version().decode()


def mems(R_bytes, Q_bytes, min_len, seed_len, q_range=None, stream=None):
    """Convenience: pack + index + find; returns the host (N, 3) uint32 array."""
    R = pack(R_bytes, stream)
    Q = pack(Q_bytes, stream)
    idx = index_build(R, seed_len, min_len, stream=stream)
    m = find_mems(idx, Q, q_range, stream=stream)
    out = m.numpy()
    for h in (m, idx, Q, R):
        h.free()
    return out
