"""CPU-side checks of the boundary: the C-ABI library loads, exports every symbol include/gum.h
declares, the host-side CSR builder (a1) is a stable counting sort, and a context cannot be made
without a GPU (no CPU fallback exists)."""
import ctypes
import os
import re

import numpy as np
import pytest

import paper_conf_icde_menggltyz23_b200 as gum

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_functions():
    text = open(os.path.join(ROOT, "include", "gum.h")).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(gum_[a-z_]+)\s*\(", text)))


def test_header_declares_the_abi():
    fns = header_functions()
    assert set(fns) == set(gum.ABI_SYMBOLS)


def test_library_exports_every_header_symbol():
    lib = gum.load_library()
    for name in header_functions():
        assert hasattr(lib, name), name
    assert gum.version() >= 100


def test_library_has_no_oracle_dependency():
    # the product library never links or embeds the oracle
    data = open(gum.LIB_PATH, "rb").read()
    assert b"oracle_bfs" not in data and b"liboracle" not in data


def test_build_csr_is_stable_counting_sort():
    rng = np.random.default_rng(0)
    V, E = 1000, 20000
    src = rng.integers(0, V, E).astype(np.uint32)
    dst = rng.integers(0, V, E).astype(np.uint32)
    w = rng.integers(1, 256, E).astype(np.uint32)
    rp, col, wo = gum.build_csr(V, src, dst, w)
    order = np.argsort(src, kind="stable")
    assert np.array_equal(col, dst[order]) and np.array_equal(wo, w[order])
    assert np.array_equal(rp, np.concatenate([[0], np.cumsum(np.bincount(src, minlength=V))]).astype(np.uint64))


def test_build_csr_edge_cases():
    rp, col, wo = gum.build_csr(5, np.array([], np.uint32), np.array([], np.uint32))
    assert rp.tolist() == [0] * 6 and col.shape[0] == 0 and wo is None
    with pytest.raises(gum.GumError):
        gum.build_csr(3, np.array([0, 5], np.uint32), np.array([1, 1], np.uint32))


def test_struct_layouts_match_header():
    # sizes fixed by include/gum.h (LP64)
    assert ctypes.sizeof(gum.gum_run_stats) == 4 + 4 + 9 * 8 + 4 * 4 + 8 + 8
    assert ctypes.sizeof(gum.gum_iter_trace) == 4 * 8 * 8 + 16 + 8


def test_no_gpu_means_error_not_fallback():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(gum.GumError):
        gum.Context(num_gpus=1)
