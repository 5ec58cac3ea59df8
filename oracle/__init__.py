"""CPU oracle for GUM's hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline`` leg and
``--impl reference``) may import this package. The product package never imports it; it shares
no code with the CUDA path (they meet only at the seeded edge lists of ``inputs/``).

Each function is the plain definition from SURVEY.md §8(c) (see ``oracle/oracle.c`` header for the
PAPER.md citations). Pins live in ``tests/test_oracle_*.py``.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None

INF = 0xFFFFFFFF


def _load():
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(_LIB_PATH):
        raise RuntimeError(f"{_LIB_PATH} missing: run `make -C {os.path.dirname(_HERE)} oracle`")
    lib = ctypes.CDLL(_LIB_PATH)
    p32 = ctypes.POINTER(ctypes.c_uint32)
    p64 = ctypes.POINTER(ctypes.c_uint64)
    pd = ctypes.POINTER(ctypes.c_double)
    lib.oracle_build_adj.restype = ctypes.c_int
    lib.oracle_build_adj.argtypes = [ctypes.c_uint32, ctypes.c_uint64, p32, p32, p32, p64, p32, p32]
    lib.oracle_bfs.restype = ctypes.c_int
    lib.oracle_bfs.argtypes = [ctypes.c_uint32, p64, p32, ctypes.c_uint32, p32]
    lib.oracle_sssp.restype = ctypes.c_int
    lib.oracle_sssp.argtypes = [ctypes.c_uint32, p64, p32, p32, ctypes.c_uint32, p32]
    lib.oracle_wcc.restype = ctypes.c_int
    lib.oracle_wcc.argtypes = [ctypes.c_uint32, ctypes.c_uint64, p32, p32, p32]
    lib.oracle_pagerank.restype = ctypes.c_int
    lib.oracle_pagerank.argtypes = [ctypes.c_uint32, ctypes.c_uint64, p32, p32, ctypes.c_int, ctypes.c_double,
                                    pd, pd]
    lib.oracle_delta_pagerank.restype = ctypes.c_int
    lib.oracle_delta_pagerank.argtypes = [ctypes.c_uint32, ctypes.c_uint64, p32, p32, ctypes.c_double, ctypes.c_double,
                                          pd, pd, ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(ctypes.c_uint64)]
    lib.oracle_pagerank_pull.restype = ctypes.c_int
    lib.oracle_pagerank_pull.argtypes = [ctypes.c_uint32, ctypes.c_uint64, p32, p32, ctypes.c_int, ctypes.c_double,
                                         ctypes.c_int, pd, pd, ctypes.POINTER(ctypes.c_int)]
    _lib = lib
    return lib


def _p(a, ct):
    if a is None:
        return None
    return a.ctypes.data_as(ctypes.POINTER(ct))


def _u32(a):
    return np.ascontiguousarray(a, dtype=np.uint32)


class Adjacency:
    """The oracle's own out-adjacency (counting sort of the raw edge list by source)."""

    def __init__(self, V, src, dst, w=None):
        lib = _load()
        src, dst = _u32(src), _u32(dst)
        w = None if w is None else _u32(w)
        E = int(src.shape[0])
        self.V = int(V)
        self.row_ptr = np.empty(self.V + 1, dtype=np.uint64)
        self.adj = np.empty(max(E, 1), dtype=np.uint32)
        self.wadj = np.empty(max(E, 1), dtype=np.uint32) if w is not None else None
        rc = lib.oracle_build_adj(self.V, E, _p(src, ctypes.c_uint32), _p(dst, ctypes.c_uint32),
                                  _p(w, ctypes.c_uint32), _p(self.row_ptr, ctypes.c_uint64),
                                  _p(self.adj, ctypes.c_uint32), _p(self.wadj, ctypes.c_uint32))
        if rc != 0:
            raise ValueError(f"oracle_build_adj failed rc={rc}")


def bfs(adj: Adjacency, source: int) -> np.ndarray:
    out = np.empty(adj.V, dtype=np.uint32)
    rc = _load().oracle_bfs(adj.V, _p(adj.row_ptr, ctypes.c_uint64), _p(adj.adj, ctypes.c_uint32), source,
                            _p(out, ctypes.c_uint32))
    if rc != 0:
        raise ValueError(f"oracle_bfs rc={rc}")
    return out


class OracleRangeError(ValueError):
    pass


def sssp(adj: Adjacency, source: int) -> np.ndarray:
    if adj.wadj is None:
        raise ValueError("sssp needs weights")
    out = np.empty(adj.V, dtype=np.uint32)
    rc = _load().oracle_sssp(adj.V, _p(adj.row_ptr, ctypes.c_uint64), _p(adj.adj, ctypes.c_uint32),
                             _p(adj.wadj, ctypes.c_uint32), source, _p(out, ctypes.c_uint32))
    if rc == -3:
        raise OracleRangeError("finite distance >= 2^32-1")
    if rc != 0:
        raise ValueError(f"oracle_sssp rc={rc}")
    return out


def wcc(V, src, dst) -> np.ndarray:
    src, dst = _u32(src), _u32(dst)
    out = np.empty(int(V), dtype=np.uint32)
    rc = _load().oracle_wcc(int(V), int(src.shape[0]), _p(src, ctypes.c_uint32), _p(dst, ctypes.c_uint32),
                            _p(out, ctypes.c_uint32))
    if rc != 0:
        raise ValueError(f"oracle_wcc rc={rc}")
    return out


def pagerank(V, src, dst, iterations=20, damping=0.85, return_residuals=False):
    src, dst = _u32(src), _u32(dst)
    x = np.empty(int(V), dtype=np.float64)
    r = np.empty(max(iterations, 1), dtype=np.float64)
    rc = _load().oracle_pagerank(int(V), int(src.shape[0]), _p(src, ctypes.c_uint32), _p(dst, ctypes.c_uint32),
                                 int(iterations), float(damping), _p(x, ctypes.c_double), _p(r, ctypes.c_double))
    if rc != 0:
        raise ValueError(f"oracle_pagerank rc={rc}")
    if return_residuals:
        return x, r[:iterations]
    return x


def pagerank_pull(V, src, dst, iterations=20, damping=0.85, threads=0, return_residuals=False):
    """OpenMP pull variant of ``pagerank``: same x_K (same terms, same per-vertex sum
    order); returns (x, threads_used) or (x, residuals, threads_used)."""
    src, dst = _u32(src), _u32(dst)
    x = np.empty(int(V), dtype=np.float64)
    r = np.empty(max(iterations, 1), dtype=np.float64)
    used = ctypes.c_int(0)
    rc = _load().oracle_pagerank_pull(int(V), int(src.shape[0]), _p(src, ctypes.c_uint32), _p(dst, ctypes.c_uint32),
                                      int(iterations), float(damping), int(threads), _p(x, ctypes.c_double),
                                      _p(r, ctypes.c_double), ctypes.byref(used))
    if rc != 0:
        raise ValueError(f"oracle_pagerank_pull rc={rc}")
    if return_residuals:
        return x, r[:iterations], used.value
    return x, used.value


def dpr_epsilon(V, tolerance=1e-6, damping=0.85):
    """Residual threshold of delta-PageRank for a target L1 tolerance (reading #27):
    eps = tolerance * (1 - d) / V, so that sum(x* - x) <= V * eps / (1 - d) = tolerance."""
    return tolerance * (1.0 - damping) / float(V)


def delta_pagerank(V, src, dst, damping=0.85, eps=None, tolerance=1e-6, return_state=False, return_work=False):
    """NEXT-4 delta-PageRank (residual push in BSP rounds). Returns x, or (x, r, rounds); return_work adds the
    number of edges pushed along."""
    src, dst = _u32(src), _u32(dst)
    if eps is None:
        eps = dpr_epsilon(V, tolerance, damping)
    x = np.empty(int(V), dtype=np.float64)
    r = np.empty(int(V), dtype=np.float64)
    rounds = ctypes.c_uint32(0)
    work = ctypes.c_uint64(0)
    rc = _load().oracle_delta_pagerank(int(V), int(src.shape[0]), _p(src, ctypes.c_uint32), _p(dst, ctypes.c_uint32),
                                       float(damping), float(eps), _p(x, ctypes.c_double), _p(r, ctypes.c_double),
                                       ctypes.byref(rounds), ctypes.byref(work))
    if rc != 0:
        raise ValueError(f"oracle_delta_pagerank rc={rc}")
    if return_state:
        return (x, r, rounds.value, work.value) if return_work else (x, r, rounds.value)
    return (x, work.value) if return_work else x


def run(alg: str, g, source: int = 0, pr_iterations: int = 20, pr_damping: float = 0.85):
    """Convenience: run one algorithm on an inputs.EdgeList."""
    if alg == "bfs":
        return bfs(Adjacency(g.num_vertices, g.src, g.dst), source)
    if alg == "sssp":
        return sssp(Adjacency(g.num_vertices, g.src, g.dst, g.w), source)
    if alg == "wcc":
        return wcc(g.num_vertices, g.src, g.dst)
    if alg == "pr":
        return pagerank(g.num_vertices, g.src, g.dst, pr_iterations, pr_damping)
    if alg == "dpr":
        return delta_pagerank(g.num_vertices, g.src, g.dst, pr_damping)
    raise ValueError(alg)
