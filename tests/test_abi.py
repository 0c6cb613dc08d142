"""CPU-side checks of the C-ABI boundary: the library builds for sm_100a, loads,
exports every symbol include/gpumem.h declares, carries sm_100a SASS, and fails
cleanly (status code + message, no abort) when asked to compute without a GPU."""
import ctypes
import os
import re
import subprocess

import pytest

from tests.conftest import ROOT

HEADER = os.path.join(ROOT, "include", "gpumem.h")


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(gpumem_[a-z_0-9]+)\s*\(", src)))


@pytest.fixture(scope="module")
def lib_path():
    from paper_conf_ipps_abu_dolehkac14_b200 import _build
    return _build.build()


def test_header_declares_the_north_star_calls():
    fns = declared_functions()
    for f in ("gpumem_pack", "gpumem_index_build", "gpumem_find_mems", "gpumem_free"):
        assert f in fns


def test_every_declared_symbol_is_exported(lib_path):
    lib = ctypes.CDLL(lib_path)
    missing = [f for f in declared_functions() if not hasattr(lib, f)]
    assert not missing, missing
    nm = subprocess.run(["nm", "-D", "--defined-only", lib_path], capture_output=True, text=True).stdout
    exported = set(re.findall(r" T (gpumem_\w+)", nm))
    assert set(declared_functions()) <= exported


def test_binding_covers_the_header(lib_path):
    from paper_conf_ipps_abu_dolehkac14_b200 import gpumem
    assert set(declared_functions()) == set(gpumem.SYMBOLS)


def test_library_holds_sm100a_code(lib_path):
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", lib_path], capture_output=True,
                         text=True).stdout
    assert "sm_100a" in out
    sass = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", lib_path], capture_output=True,
                          text=True).stdout
    for k in ("k_pack", "k_find", "k_heavy", "k_coop", "k_seed_codes", "k_ptrs_fill", "k_seed_recs",
              "k_chunk_hist", "k_chunk_scan", "k_scatter", "k_revcomp", "k_occurrences", "k_merge_tile", "k_split_emit", "k_band_continue", "k_open_fix", "k_fill", "k_collect"):
        assert k in sass, k


def test_no_oracle_in_product():
    """The product path never imports or links the oracle (test infrastructure)."""
    pkg = os.path.join(ROOT, "paper_conf_ipps_abu_dolehkac14_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert not re.search(r"^\s*(import oracle|from oracle)", txt, re.M), f
                assert "mem_oracle" not in txt and "liboracle" not in txt, f


def test_errors_without_gpu_are_clean(lib_path):
    from paper_conf_ipps_abu_dolehkac14_b200 import gpumem
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present; covered by the gpu tests")
    with pytest.raises(gpumem.GpumemError) as ei:
        gpumem.pack(b"ACGT", stream=0)
    assert ei.value.name == "ERR_UNSUPPORTED"
    assert "device" in str(ei.value)
    lib = gpumem._lib
    out = ctypes.c_void_p()
    assert lib.gpumem_pack(None, 5, 0, None, ctypes.byref(out)) == 1   # NULL bases -> ERR_ARG
    assert out.value is None
    assert lib.gpumem_index_build(None, 13, 100, None, ctypes.byref(out)) == 1
    assert lib.gpumem_find_mems(None, None, 0, 0, None, ctypes.byref(out)) == 1
    assert lib.gpumem_set_option(b"nope", 1) == 1
    assert lib.gpumem_set_option(b"find_spill", 64) == 0
    assert lib.gpumem_set_option(b"radix_bits", 7) == 1 and lib.gpumem_set_option(b"radix_bits", 11) == 1
    assert lib.gpumem_set_option(b"radix_bits", 0) == 0
    assert lib.gpumem_set_option(b"l2_window", 4) == 1 and lib.gpumem_set_option(b"l2_window", -1) == 1
    assert lib.gpumem_set_option(b"l2_window", 0) == 0
    lib.gpumem_free(None)
    assert gpumem.version()
