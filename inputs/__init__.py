"""Seeded synthetic graph inputs shared by the oracle and the CUDA path (edge lists only).

This module holds none of the method's arithmetic (no CSR, partition or traversal): it turns a
seed into raw edge arrays, exactly as ``inputs/gen.c`` documents. See DESIGN.md "Input recipe"
and SURVEY.md §8(d) for the configs C1..C5.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libgen.so")
_lib = None

U32 = np.uint32


def _load():
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(_LIB_PATH):
        raise RuntimeError(f"{_LIB_PATH} missing: run `make -C {os.path.dirname(_HERE)} inputs`")
    lib = ctypes.CDLL(_LIB_PATH)
    p32 = ctypes.POINTER(ctypes.c_uint32)
    lib.gen_hash.restype = ctypes.c_uint64
    lib.gen_hash.argtypes = [ctypes.c_uint64] * 3
    lib.gen_splitmix_seq.restype = ctypes.c_uint64
    lib.gen_splitmix_seq.argtypes = [ctypes.c_uint64, ctypes.c_uint64]
    lib.gen_scramble.restype = ctypes.c_uint64
    lib.gen_scramble.argtypes = [ctypes.c_uint64, ctypes.c_int, ctypes.c_uint64]
    lib.gen_rmat.restype = ctypes.c_int
    lib.gen_rmat.argtypes = [ctypes.c_int, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_double,
                             ctypes.c_double, ctypes.c_double, ctypes.c_int, ctypes.c_int, p32, p32, p32]
    lib.gen_grid_num_edges.restype = ctypes.c_uint64
    lib.gen_grid_num_edges.argtypes = [ctypes.c_uint64, ctypes.c_int]
    lib.gen_grid.restype = ctypes.c_int
    lib.gen_grid.argtypes = [ctypes.c_uint64, ctypes.c_int, ctypes.c_uint64, ctypes.c_int, p32, p32, p32]
    _lib = lib
    return lib


def _p32(a):
    if a is None:
        return None
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32))


@dataclass
class EdgeList:
    """Directed multigraph edge list: edge i is (src[i] -> dst[i]) with weight w[i] (or None)."""
    num_vertices: int
    src: np.ndarray
    dst: np.ndarray
    w: np.ndarray | None
    name: str = ""

    @property
    def num_edges(self) -> int:
        return int(self.src.shape[0])


def rmat(scale: int, edge_factor: int = 16, seed: int = 1, weighted: bool = True, scramble: bool = True,
         a: float = 0.57, b: float = 0.19, c: float = 0.19) -> EdgeList:
    lib = _load()
    V = 1 << scale
    E = V * edge_factor
    src = np.empty(E, dtype=U32)
    dst = np.empty(E, dtype=U32)
    w = np.empty(E, dtype=U32) if weighted else None
    lib.gen_rmat(scale, E, seed, a, b, c, int(scramble), int(weighted), _p32(src), _p32(dst),
                 _p32(w) if weighted else None)
    return EdgeList(V, src, dst, w, f"rmat{scale}ef{edge_factor}s{seed}")


def grid(n: int, seed: int = 3, unit_weights: bool = False, torus: bool = False) -> EdgeList:
    lib = _load()
    E = int(lib.gen_grid_num_edges(n, int(torus)))
    src = np.empty(E, dtype=U32)
    dst = np.empty(E, dtype=U32)
    w = np.empty(E, dtype=U32)
    lib.gen_grid(n, int(torus), seed, int(unit_weights), _p32(src), _p32(dst), _p32(w))
    return EdgeList(n * n, src, dst, w, f"{'torus' if torus else 'grid'}{n}s{seed}")


def torus(n: int, seed: int = 0) -> EdgeList:
    return grid(n, seed=seed, unit_weights=True, torus=True)


def from_pairs(V: int, pairs, weights=None, name: str = "hand") -> EdgeList:
    """Hand-built graphs for pins: pairs = [(u, v), ...]."""
    arr = np.asarray(list(pairs), dtype=np.int64).reshape(-1, 2)
    src = arr[:, 0].astype(U32)
    dst = arr[:, 1].astype(U32)
    w = None if weights is None else np.asarray(weights, dtype=U32)
    return EdgeList(V, src, dst, w, name)


def hash64(seed: int, stream: int, ctr: int) -> int:
    return int(_load().gen_hash(seed, stream, ctr))


def scramble(v: int, bits: int, seed: int) -> int:
    return int(_load().gen_scramble(v, bits, seed))


def pick_source(g: EdgeList, seed: int) -> int:
    """SURVEY.md §8(c) reading #19: first vertex of the splitmix64(seed) sequence with outdeg > 0."""
    lib = _load()
    outdeg = np.bincount(g.src, minlength=g.num_vertices)
    if not (outdeg > 0).any():
        return 0
    j = 0
    while True:
        v = int(lib.gen_splitmix_seq(seed, j) % g.num_vertices)
        if outdeg[v] > 0:
            return v
        j += 1


# SURVEY.md §8(d) configs. C1 is the oracle-sized parity case; C2 the N=1 bench workload.
CONFIGS = {
    "C1": dict(kind="rmat", scale=16, edge_factor=16, seed=1, algs=("bfs", "sssp")),
    "C2": dict(kind="rmat", scale=24, edge_factor=16, seed=2, algs=("bfs",)),
    "C3": dict(kind="grid", n=8192, seed=3, algs=("sssp",)),
    "C4": dict(kind="rmat", scale=26, edge_factor=16, seed=4, algs=("wcc",)),
    "C5": dict(kind="rmat", scale=25, edge_factor=44, seed=5, algs=("pr",)),
}


def make_config(name: str, weighted: bool | None = None) -> EdgeList:
    cfg = CONFIGS[name]
    if cfg["kind"] == "rmat":
        wt = ("sssp" in cfg["algs"]) if weighted is None else weighted
        return rmat(cfg["scale"], cfg["edge_factor"], cfg["seed"], weighted=wt)
    return grid(cfg["n"], seed=cfg["seed"])
