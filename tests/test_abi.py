"""CPU-side checks of the boundary: the C-ABI library loads, exports every symbol include/gum.h
declares, the host-side CSR builder (a1) is a stable counting sort, and a context cannot be made
without a GPU (no CPU fallback exists)."""
import ctypes
import os
import re
import subprocess

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


def test_struct_layouts_match_header(tmp_path):
    # every field offset and struct size of the ctypes mirrors equals the C compiler's view of include/gum.h
    structs = {"gum_config": gum.gum_config, "gum_run_stats": gum.gum_run_stats,
               "gum_iter_trace": gum.gum_iter_trace, "gum_kernel_times": gum.gum_kernel_times,
               "gum_mp_config": gum.gum_mp_config}
    lines = ['#include <stdio.h>', '#include <stddef.h>', '#include "gum.h"', "int main(void) {"]
    for name, cls in structs.items():
        lines.append(f'printf("{name} size %zu\\n", sizeof({name}));')
        for fname, _ in cls._fields_:
            lines.append(f'printf("{name} {fname} %zu\\n", offsetof({name}, {fname}));')
    lines.append("return 0; }")
    src = tmp_path / "layout.c"
    src.write_text("\n".join(lines))
    exe = tmp_path / "layout"
    inc = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "include")
    subprocess.run(["gcc", "-I", inc, str(src), "-o", str(exe)], check=True)
    out = subprocess.run([str(exe)], check=True, capture_output=True, text=True).stdout.split("\n")
    got = {tuple(l.split()[:2]): int(l.split()[2]) for l in out if l.strip()}
    for name, cls in structs.items():
        assert got[(name, "size")] == ctypes.sizeof(cls), name
        for fname, _ in cls._fields_:
            assert got[(name, fname)] == getattr(cls, fname).offset, (name, fname)


def test_no_gpu_means_error_not_fallback():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(gum.GumError):
        gum.Context(num_gpus=1)
