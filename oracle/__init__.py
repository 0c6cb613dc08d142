"""CPU oracle for GPUMEM's MEM extraction -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg and
--impl reference) may import this package. The product package
(paper_conf_ipps_abu_dolehkac14_b200) never imports it, and it imports
nothing from the product (the seeded input generator synth.py is the only
shared module and holds no method arithmetic).

  mems(R, Q, L, ls, ...)  -> (N,3) uint32 [r, q, len], sorted by (r, q)
                             C++ oracle O1 (mem_oracle.cpp: oracle_mems)
  brute(R, Q, L)          -> same, by the O(|R||Q|) definition (brute_mems)
  index(R, ls, step)      -> (ptrs, locs) by Algorithm 1 (oracle_index)
  mums(R, Q, L, ls)       -> MUMs: MEMs unique in both sequences (oracle_mums)
  pyoracle                -> pure-Python twins for tiny inputs

See mem_oracle.cpp's header for the PAPER.md passages each function follows
and what pins it. Every function here is pinned (no "parity unpinned").
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "mem_oracle.cpp")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None


def build(force=False):
    """Compile liboracle.so (g++ -O2 -fopenmp). Building the checker is not using it."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.run(["g++", "-O2", "-std=c++17", "-fopenmp", "-shared", "-fPIC", _SRC, "-o", tmp],
                       check=True)
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            build()
            lib = ctypes.CDLL(_LIB)
            P = ctypes.POINTER
            u32pp = P(P(ctypes.c_uint32))
            lib.oracle_mems.argtypes = [ctypes.c_char_p, ctypes.c_uint64, ctypes.c_char_p, ctypes.c_uint64,
                                        ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32,
                                        ctypes.c_uint64, ctypes.c_uint64, ctypes.c_int, u32pp]
            lib.oracle_mems.restype = ctypes.c_int64
            lib.brute_mems.argtypes = [ctypes.c_char_p, ctypes.c_uint64, ctypes.c_char_p, ctypes.c_uint64,
                                       ctypes.c_uint32, ctypes.c_int, u32pp]
            lib.brute_mems.restype = ctypes.c_int64
            lib.oracle_index.argtypes = [ctypes.c_char_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32,
                                         P(ctypes.c_uint32), P(ctypes.c_uint32)]
            lib.oracle_index.restype = ctypes.c_int64
            lib.oracle_mums.argtypes = [ctypes.c_char_p, ctypes.c_uint64, ctypes.c_char_p, ctypes.c_uint64,
                                        ctypes.c_uint32, ctypes.c_uint32, ctypes.c_int, u32pp]
            lib.oracle_mums.restype = ctypes.c_int64
            lib.oracle_rare.argtypes = [ctypes.c_char_p, ctypes.c_uint64, ctypes.c_char_p, ctypes.c_uint64,
                                        ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_int,
                                        ctypes.POINTER(ctypes.POINTER(ctypes.c_uint32))]
            lib.oracle_rare.restype = ctypes.c_int64
            lib.oracle_free.argtypes = [ctypes.c_void_p]
            lib.oracle_num_threads.argtypes = [ctypes.c_int]
            lib.oracle_num_threads.restype = ctypes.c_int
            _lib = lib
    return _lib


class OracleError(ValueError):
    pass


_ERR = {-1: "bad argument", -2: "alphabet", -3: "range"}


def _bytes(x):
    if isinstance(x, np.ndarray):
        return x.astype(np.uint8, copy=False).tobytes()
    if isinstance(x, str):
        return x.encode("ascii")
    return bytes(x)


def _take(n, ptr):
    lib = _load()
    if n < 0:
        raise OracleError(_ERR.get(n, str(n)))
    try:
        if n == 0:
            return np.zeros((0, 3), dtype=np.uint32)
        buf = np.ctypeslib.as_array(ptr, shape=(n * 3,)).copy()
        return buf.reshape(n, 3)
    finally:
        lib.oracle_free(ptr)


def num_threads(threads=0):
    return _load().oracle_num_threads(int(threads))


def mems(R, Q, L, ls, step=0, q_begin=0, q_end=None, threads=0):
    """Oracle O1: sorted (r, q, len) uint32 array of MEMs with start q in [q_begin, q_end)."""
    lib = _load()
    Rb, Qb = _bytes(R), _bytes(Q)
    q_end = len(Qb) if q_end is None else min(int(q_end), len(Qb))
    out = ctypes.POINTER(ctypes.c_uint32)()
    n = lib.oracle_mems(Rb, len(Rb), Qb, len(Qb), int(L), int(ls), int(step), int(q_begin), int(q_end),
                        int(threads), ctypes.byref(out))
    return _take(n, out)


def brute(R, Q, L, threads=0):
    """Oracle O2: the definition, O(|R||Q|)."""
    lib = _load()
    Rb, Qb = _bytes(R), _bytes(Q)
    out = ctypes.POINTER(ctypes.c_uint32)()
    n = lib.brute_mems(Rb, len(Rb), Qb, len(Qb), int(L), int(threads), ctypes.byref(out))
    return _take(n, out)


def mums(R, Q, L, ls, threads=0):
    """MUMs: MEMs whose string occurs exactly once in R and once in Q (oracle_mums)."""
    lib = _load()
    Rb, Qb = _bytes(R), _bytes(Q)
    out = ctypes.POINTER(ctypes.c_uint32)()
    n = lib.oracle_mums(Rb, len(Rb), Qb, len(Qb), int(L), int(ls), int(threads), ctypes.byref(out))
    return _take(n, out)


def rare(R, Q, L, ls, k, threads=0):
    """Rare MEMs: MEMs whose string occurs at most k times in R and in Q (oracle_rare)."""
    lib = _load()
    Rb, Qb = _bytes(R), _bytes(Q)
    out = ctypes.POINTER(ctypes.c_uint32)()
    n = lib.oracle_rare(Rb, len(Rb), Qb, len(Qb), int(L), int(ls), int(k), int(threads), ctypes.byref(out))
    return _take(n, out)


def mems_multi(R_text, Q_text, L, ls, threads=0):
    """MEMs of multi-FASTA inputs (R24): oracle_mems on every pair of ACGT
    segments (the maximal runs of A/C/G/T letters inside each record), shifted to record
    coordinates. Sorted (r_record, r_pos, q_record, q_pos, len), 0-based."""
    from . import pyoracle
    import re

    def segments(seq):
        return [(m.start(), m.group()) for m in re.finditer(r"[ACGTacgt]+", seq)]

    out = []
    R, Q = pyoracle.fasta(R_text), pyoracle.fasta(Q_text)
    for ri, (_, r) in enumerate(R):
        for a, rs in segments(r):
            for qi, (_, q) in enumerate(Q):
                for b, qs in segments(q):
                    if len(rs) < L or len(qs) < L:
                        continue
                    for t in mems(rs.encode(), qs.encode(), L, min(ls, L), threads=threads).tolist():
                        out.append((ri, a + t[0], qi, b + t[1], t[2]))
    return sorted(out)


def index(R, ls, step):
    """Algorithm 1 on the whole of R: (ptrs uint32[4^ls+1], locs uint32[n_locs])."""
    lib = _load()
    Rb = _bytes(R)
    n_locs = 0 if len(Rb) < ls else (len(Rb) - ls) // step + 1
    ptrs = np.zeros((1 << (2 * ls)) + 1, dtype=np.uint32)
    locs = np.zeros(max(1, n_locs), dtype=np.uint32)
    n = lib.oracle_index(Rb, len(Rb), int(ls), int(step),
                         ptrs.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)),
                         locs.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)))
    if n < 0:
        raise OracleError(_ERR.get(n, str(n)))
    return ptrs, locs[:n]
