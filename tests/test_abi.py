"""The C-ABI library builds for sm_100a, loads, and exports every symbol include/mv.h declares.
No compute calls here (no GPU on this box)."""
import ctypes
import os
import subprocess

import pytest

from paper_conf_sigmod_wangygjxlwglxyy21_b200 import _lib as L
from paper_conf_sigmod_wangygjxlwglxyy21_b200.build import build


@pytest.fixture(scope="module")
def lib():
    build()
    return L.load()


def test_header_declares_the_boundary():
    syms = L.header_symbols()
    for s in ["mv_index_create", "mv_index_set_centroids", "mv_index_train_sq8", "mv_index_set_sq8", "mv_index_add",
              "mv_search", "mv_merge_topk", "mv_index_destroy", "mv_last_error", "mv_search_probes",
              "mv_index_ntotal", "mv_index_storage", "mv_index_set_option", "mv_search_with_probes"]:
        assert s in syms


def test_library_exports_every_header_symbol(lib):
    for s in L.header_symbols():
        assert hasattr(lib, s), s
        assert ctypes.cast(getattr(lib, s), ctypes.c_void_p).value
    out = subprocess.run(["nm", "-D", "--defined-only", L.LIB_PATH], capture_output=True, text=True).stdout
    exported = {ln.split()[-1] for ln in out.splitlines() if " T " in ln}
    assert set(L.header_symbols()) <= exported
    # nothing else leaks out of the C ABI
    assert all(s.startswith("mv_") for s in exported if not s.startswith("_"))


def test_library_is_sm100a(lib):
    r = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", L.LIB_PATH], capture_output=True, text=True)
    assert "sm_100a" in r.stdout


def test_version_and_error_strings(lib):
    assert b"sm_100a" in lib.mv_version()
    assert lib.mv_last_error() is not None


def test_argument_errors_before_any_device_work(lib):
    # argument validation returns synchronously without touching a device
    h = ctypes.c_void_p()
    assert lib.mv_index_create(0, 0, 0, 4, 0, None, ctypes.byref(h)) == -1
    assert b"d must be" in lib.mv_last_error()
    assert lib.mv_index_create(513, 0, 0, 4, 0, None, ctypes.byref(h)) == -1   # d <= 512 (mv.h)
    assert lib.mv_index_create(8, 7, 0, 4, 0, None, ctypes.byref(h)) == -1
    assert lib.mv_index_create(8, 0, 0, 0, 0, None, ctypes.byref(h)) == -1
    half = L.MvAllocator(L.ALLOC_FN(lambda n, s, c: None), L.FREE_FN(), None)  # alloc without free
    assert lib.mv_index_create(8, 0, 0, 4, 0, ctypes.byref(half), ctypes.byref(h)) == -1
    assert b"allocator" in lib.mv_last_error()
    assert lib.mv_index_set_option(None, b"need", 1) == -1
    assert lib.mv_merge_topk(0, None, None, 0, 1, 1, None, None, None) == -1
    assert lib.mv_search(None, None, 1, 10, 1, None, 0, None, None, None) == -1
    assert lib.mv_index_ntotal(None) == 0
    lib.mv_index_destroy(None)


def test_no_cpu_fallback_in_the_binding():
    """The product path never imports the oracle and fails loudly without libmv.so."""
    pkg = os.path.dirname(L.__file__)
    for fn in os.listdir(pkg):
        if fn.endswith(".py"):
            src = open(os.path.join(pkg, fn)).read()
            assert "import oracle" not in src and "from oracle" not in src, fn


def test_f1_f4_entry_points_validate_arguments(lib):
    import ctypes as C
    assert lib.mv_kmeans(None, 10, 4, 0, 2, 1, 0, None, 0, None) == -1
    assert lib.mv_attr_bitset(None, None, -1, 0, 1, None, 8, None) == -1
    dims = (C.c_int32 * 1)(4)
    assert lib.mv_fuse_rows(None, dims, None, 0, 1, None, None) == -1      # m = 0
    assert lib.mv_fuse_rows(None, dims, None, 17, 1, None, None) == -1     # m > 16
