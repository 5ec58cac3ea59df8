"""Thin Python binding of the GUM C ABI (include/gum.h) -- argument marshalling only.

Every step of the hot path runs in ``libgum.so`` (hand-written sm_100a CUDA). This module only
converts numpy arrays / torch tensors to pointers and back. There is no CPU fallback: if the
extension is missing or no GPU is visible, calls raise ``GumError``.

Names follow the ABI: ``build_csr``, ``Context.load_csr``, ``Context.partition``, ``Context.run``,
``Context.result``. PyTorch is optional plumbing: device tensors can be passed to ``load_csr`` /
``result_device``, the torch caching allocator can back device memory (``use_torch_allocator``) and
torch streams can be used (``streams``).
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("GUM_LIB") or os.path.join(_HERE, "libgum.so")  # GUM_LIB: build variants (tuning)

GUM_OK, GUM_EINVAL, GUM_ENOMEM, GUM_ESTATE, GUM_ERANGE, GUM_ECUDA, GUM_ENCCL, GUM_EUNSUP = 0, -1, -2, -3, -4, -5, -6, -7
STATUS_NAMES = {0: "GUM_OK", -1: "GUM_EINVAL", -2: "GUM_ENOMEM", -3: "GUM_ESTATE", -4: "GUM_ERANGE",
                -5: "GUM_ECUDA", -6: "GUM_ENCCL", -7: "GUM_EUNSUP"}
ALGS = {"bfs": 0, "sssp": 1, "wcc": 2, "pr": 3, "dpr": 4}
PARTS = {"seg": 0, "random": 1, "degree": 2}
INF = 0xFFFFFFFF
MAX_WORKERS = 8

CFG_TRACE, CFG_HOST_LOOP, CFG_FORCE_SPARSE, CFG_FORCE_DENSE, CFG_PROFILE, CFG_SPLIT_UNITS = 0x1, 0x2, 0x4, 0x8, 0x10, 0x20
LOAD_DEVICE = 0x1

# exported symbols of include/gum.h (tests check the .so exports exactly these)
ABI_SYMBOLS = ("gum_config_default", "gum_create", "gum_destroy", "gum_last_error", "gum_build_csr",
               "gum_load_csr", "gum_partition", "gum_partition_bounds", "gum_prepare", "gum_run", "gum_result",
               "gum_result_device", "gum_trace", "gum_profile", "gum_fsteal_plan", "gum_version",
               "gum_mp_handshake", "gum_create_mp", "gum_osteal_plan")


class GumError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS_NAMES.get(status, status)}: {msg}")
        self.status = status


ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int, ctypes.c_void_p)
FREE_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int, ctypes.c_void_p)


class gum_config(ctypes.Structure):
    _fields_ = [("num_gpus", ctypes.c_int), ("device_ids", ctypes.POINTER(ctypes.c_int)),
                ("fsteal", ctypes.c_int), ("t1_min_max_edges", ctypes.c_uint64),
                ("t2_min_spread_edges", ctypes.c_uint64), ("osteal", ctypes.c_int),
                ("osteal_active_threshold", ctypes.c_uint64), ("osteal_edges_per_worker", ctypes.c_uint64),
                ("chunk_edges", ctypes.c_uint32), ("pr_iterations", ctypes.c_int), ("pr_damping", ctypes.c_double),
                ("max_iterations", ctypes.c_uint32), ("flags", ctypes.c_uint32), ("sssp_delta", ctypes.c_uint32),
                ("tail_vertices", ctypes.c_uint32), ("pb_block_log2", ctypes.c_uint32),
                ("fsteal_remote_cost", ctypes.c_double), ("bfs_direction_opt", ctypes.c_int),
                ("osteal_sync_edges", ctypes.c_double),
                ("alloc", ALLOC_FN),
                ("free_fn", FREE_FN), ("alloc_user", ctypes.c_void_p), ("streams", ctypes.POINTER(ctypes.c_void_p)),
                ("mirrors", ctypes.c_int), ("hub_cache", ctypes.c_int), ("hub_degree", ctypes.c_uint32),
                ("pr_push", ctypes.c_int), ("dpr_tolerance", ctypes.c_double), ("osteal_migrate", ctypes.c_int)]


EXCHANGE_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p)


class gum_mp_config(ctypes.Structure):
    _fields_ = [("rank", ctypes.c_int), ("world", ctypes.c_int), ("device", ctypes.c_int),
                ("exchange", EXCHANGE_FN), ("user", ctypes.c_void_p)]


class gum_run_stats(ctypes.Structure):
    _fields_ = [("iterations", ctypes.c_uint32), ("ms", ctypes.c_double), ("edges_expanded", ctypes.c_uint64),
                ("edges_frontier", ctypes.c_uint64), ("edges_stolen", ctypes.c_uint64),
                ("chunks_stolen", ctypes.c_uint64), ("chunks_total", ctypes.c_uint64),
                ("remote_updates", ctypes.c_uint64), ("activations", ctypes.c_uint64),
                ("vertices_frontier", ctypes.c_uint64), ("final_owners", ctypes.c_uint32), ("osteal_iteration", ctypes.c_uint32),
                ("tail_iterations", ctypes.c_uint32), ("bodies", ctypes.c_uint32),
                ("pr_last_residual", ctypes.c_double), ("kernel_launches", ctypes.c_uint64),
                ("remote_filtered", ctypes.c_uint64), ("hub_cached_edges", ctypes.c_uint64),
                ("mirror_flush_bytes", ctypes.c_uint64), ("blocked_iterations", ctypes.c_uint32),
                ("tail_overflows", ctypes.c_uint32), ("tail_edges", ctypes.c_uint64), ("tail_vertices", ctypes.c_uint64),
                ("tail_activations", ctypes.c_uint64), ("unit_barriers", ctypes.c_uint32 * MAX_WORKERS),
                ("unit_last_iter", ctypes.c_uint32 * MAX_WORKERS), ("host_launches", ctypes.c_uint64),
                ("osteal_p", ctypes.c_double), ("osteal_p_samples", ctypes.c_uint32), ("pad1", ctypes.c_uint32),
                ("migrated_queue_entries", ctypes.c_uint64)]


class gum_kernel_times(ctypes.Structure):
    _fields_ = [("filter_ms", ctypes.c_double), ("control_ms", ctypes.c_double), ("advance_ms", ctypes.c_double),
                ("finalize_ms", ctypes.c_double), ("init_ms", ctypes.c_double), ("tail_ms", ctypes.c_double),
                ("filter_launches", ctypes.c_uint32), ("control_launches", ctypes.c_uint32),
                ("advance_launches", ctypes.c_uint32), ("finalize_launches", ctypes.c_uint32),
                ("init_launches", ctypes.c_uint32), ("tail_launches", ctypes.c_uint32)]


class gum_iter_trace(ctypes.Structure):
    _fields_ = [("t_start", ctypes.c_uint64 * MAX_WORKERS), ("t_end", ctypes.c_uint64 * MAX_WORKERS),
                ("edges_own", ctypes.c_uint64 * MAX_WORKERS), ("edges_stolen", ctypes.c_uint64 * MAX_WORKERS),
                ("frontier_vertices", ctypes.c_uint64), ("frontier_edges", ctypes.c_uint64),
                ("owners", ctypes.c_uint32), ("steal_ok", ctypes.c_uint32)]


_lib = None


def load_library():
    """Loads libgum.so; raises if it is missing (no fallback path exists)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise GumError(GUM_EUNSUP, f"{LIB_PATH} not built: run `make gum` (or __graft_entry__.build())")
    lib = ctypes.CDLL(LIB_PATH)
    vp, u32, u64, i32 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
    sig = {
        "gum_config_default": (None, [ctypes.POINTER(gum_config)]),
        "gum_create": (i32, [ctypes.POINTER(gum_config), ctypes.POINTER(vp)]),
        "gum_destroy": (None, [vp]),
        "gum_last_error": (ctypes.c_char_p, [vp]),
        "gum_build_csr": (i32, [u32, u64, vp, vp, vp, vp, vp, vp]),
        "gum_load_csr": (i32, [vp, u32, u64, vp, vp, vp, u32]),
        "gum_partition": (i32, [vp, i32, u64]),
        "gum_partition_bounds": (i32, [vp, vp, i32]),
        "gum_prepare": (i32, [vp, i32]),
        "gum_run": (i32, [vp, i32, u32, ctypes.POINTER(gum_run_stats)]),
        "gum_result": (i32, [vp, vp, u64]),
        "gum_result_device": (i32, [vp, vp, u64]),
        "gum_trace": (i32, [vp, vp, u32, ctypes.POINTER(u32)]),
        "gum_profile": (i32, [vp, ctypes.POINTER(gum_kernel_times)]),
        "gum_fsteal_plan": (i32, [vp, i32, ctypes.c_double, vp, ctypes.POINTER(ctypes.c_double)]),
        "gum_version": (i32, []),
        "gum_mp_handshake": (i32, [ctypes.POINTER(gum_config), ctypes.POINTER(gum_mp_config)]),
        "gum_osteal_plan": (i32, [vp, i32, ctypes.c_double, ctypes.c_double, vp, ctypes.POINTER(i32)]),
        "gum_create_mp": (i32, [ctypes.POINTER(gum_config), ctypes.POINTER(gum_mp_config), ctypes.POINTER(vp)]),
    }
    for name, (res, args) in sig.items():
        fn = getattr(lib, name)
        fn.restype = res
        fn.argtypes = args
    _lib = lib
    return lib


def _ptr(a):
    if a is None:
        return None
    if hasattr(a, "data_ptr"):
        return ctypes.c_void_p(a.data_ptr())
    return ctypes.c_void_p(a.ctypes.data)


def _is_cuda(a):
    return hasattr(a, "is_cuda") and a.is_cuda


def build_csr(num_vertices, src, dst, w=None):
    """a1: stable counting sort of an edge multiset into CSR (native, OpenMP). Returns numpy arrays."""
    lib = load_library()
    src = np.ascontiguousarray(src, dtype=np.uint32)
    dst = np.ascontiguousarray(dst, dtype=np.uint32)
    E = int(src.shape[0])
    row_ptr = np.empty(int(num_vertices) + 1, dtype=np.uint64)
    col = np.empty(max(E, 1), dtype=np.uint32)
    wout = None
    if w is not None:
        w = np.ascontiguousarray(w, dtype=np.uint32)
        wout = np.empty(max(E, 1), dtype=np.uint32)
    st = lib.gum_build_csr(int(num_vertices), E, _ptr(src), _ptr(dst), _ptr(w), _ptr(row_ptr), _ptr(col), _ptr(wout))
    if st != GUM_OK:
        raise GumError(st, "gum_build_csr failed (vertex id out of range?)")
    return row_ptr, col[:E], (wout[:E] if wout is not None else None)


@dataclass
class RunStats:
    iterations: int
    ms: float
    edges_expanded: int
    edges_frontier: int
    edges_stolen: int
    chunks_stolen: int
    chunks_total: int
    remote_updates: int
    activations: int
    vertices_frontier: int
    final_owners: int
    osteal_iteration: int
    tail_iterations: int
    bodies: int
    pr_last_residual: float
    kernel_launches: int
    remote_filtered: int = 0
    hub_cached_edges: int = 0
    mirror_flush_bytes: int = 0
    blocked_iterations: int = 0
    tail_overflows: int = 0
    tail_edges: int = 0
    tail_vertices: int = 0
    tail_activations: int = 0
    unit_barriers: list = None
    unit_last_iter: list = None
    host_launches: int = 0
    osteal_p: float = 0.0
    osteal_p_samples: int = 0
    pad1: int = 0
    migrated_queue_entries: int = 0


def make_config(num_gpus=1, device_ids=None, fsteal=True, osteal=True, t1=0, t2=0, osteal_threshold=0,
                osteal_edges_per_worker=0, chunk_edges=2048, pr_iterations=20, pr_damping=0.85, max_iterations=0,
                trace=False, host_loop=False, profile=False, split_units=False, sssp_delta=0, tail_vertices=16384,
                pb_block_log2=0, fsteal_remote_cost=1.0, bfs_direction_opt=False, force_mode=None,
                use_torch_allocator=False, streams=None, osteal_sync_edges=0.0, mirrors=False, hub_cache=False,
                hub_degree=0, pr_push=False, dpr_tolerance=1e-6, osteal_migrate=False):
    """Builds a gum_config (host only). Returns (cfg, keepalive): keepalive holds the ctypes objects the
    config points to and must live as long as the context."""
    lib = load_library()
    keep = []
    cfg = gum_config()
    lib.gum_config_default(ctypes.byref(cfg))
    cfg.num_gpus = int(num_gpus)
    if device_ids is not None:
        ids = (ctypes.c_int * len(device_ids))(*device_ids)
        keep.append(ids)
        cfg.device_ids = ctypes.cast(ids, ctypes.POINTER(ctypes.c_int))
    cfg.fsteal = 2 if fsteal == "planned" else int(bool(fsteal))
    cfg.fsteal_remote_cost = float(fsteal_remote_cost)
    cfg.bfs_direction_opt = int(bool(bfs_direction_opt))
    cfg.osteal = 2 if osteal == "cost" else int(bool(osteal))
    cfg.osteal_sync_edges = float(osteal_sync_edges)
    cfg.t1_min_max_edges = int(t1)
    cfg.t2_min_spread_edges = int(t2)
    cfg.osteal_active_threshold = int(osteal_threshold)
    cfg.osteal_edges_per_worker = int(osteal_edges_per_worker)
    cfg.chunk_edges = int(chunk_edges)
    cfg.pr_iterations = int(pr_iterations)
    cfg.pr_damping = float(pr_damping)
    cfg.max_iterations = int(max_iterations)
    cfg.sssp_delta = int(sssp_delta)
    cfg.tail_vertices = int(tail_vertices)
    cfg.pb_block_log2 = int(pb_block_log2)
    cfg.mirrors = int(bool(mirrors))          # NEXT-1 outer-vertex mirrors
    cfg.hub_cache = int(bool(hub_cache))      # NEXT-1 hub adjacency caching
    cfg.hub_degree = int(hub_degree)          # t4
    cfg.pr_push = int(bool(pr_push))          # PR advance: pull over source blocks (default) or push
    cfg.dpr_tolerance = float(dpr_tolerance)  # delta-PageRank: L1 tolerance (eps = tol * (1-d) / V)
    cfg.osteal_migrate = int(bool(osteal_migrate))  # NEXT-3: evicted fragments' queues generated on the owner
    flags = 0
    if trace:
        flags |= CFG_TRACE
    if host_loop:
        flags |= CFG_HOST_LOOP
    if profile:
        flags |= CFG_PROFILE
    if split_units:
        flags |= CFG_SPLIT_UNITS
    if force_mode == "sparse":
        flags |= CFG_FORCE_SPARSE
    elif force_mode == "dense":
        flags |= CFG_FORCE_DENSE
    cfg.flags = flags
    if use_torch_allocator:
        import torch

        def _alloc(nbytes, device, user):
            try:
                return torch.cuda.caching_allocator_alloc(int(nbytes), device=int(device))
            except Exception:  # noqa: BLE001 - reported to C as a null pointer (GUM_ENOMEM)
                return None

        def _free(ptr, nbytes, device, user):
            torch.cuda.caching_allocator_delete(ptr)

        a, f = ALLOC_FN(_alloc), FREE_FN(_free)
        keep += [a, f]
        cfg.alloc, cfg.free_fn = a, f
    if streams is not None:
        arr = (ctypes.c_void_p * MAX_WORKERS)(*[int(getattr(s, "cuda_stream", s)) for s in streams])
        keep.append(arr)
        cfg.streams = ctypes.cast(arr, ctypes.POINTER(ctypes.c_void_p))
    return cfg, keep


class Context:
    """One GUM context: num_gpus workers/fragments (device_ids None => virtual peers on device 0).

    Multi-process mode (one process per GPU, include/gum.h gum_create_mp): pass
    ``mp=(rank, world, device, exchange)`` with num_gpus == world, where ``exchange`` is a host
    all-gather (see ``paper_conf_icde_menggltyz23_b200.dist.allgather_exchange``). Every later call is
    then collective over the ranks."""

    def __init__(self, num_gpus=1, mp=None, **kw):
        lib = load_library()
        cfg, keep = make_config(num_gpus=num_gpus, **kw)
        self._keep = keep
        self._cfg = cfg
        self._ctx = ctypes.c_void_p()
        if mp is None:
            st = lib.gum_create(ctypes.byref(cfg), ctypes.byref(self._ctx))
            if st != GUM_OK:
                raise GumError(st, "gum_create failed (no CUDA device, bad config or unsupported device mix)")
        else:
            rank, world, device, exchange = mp
            fn = exchange if isinstance(exchange, EXCHANGE_FN) else EXCHANGE_FN(exchange)
            mpc = gum_mp_config(int(rank), int(world), int(device), fn, None)
            self._keep += [fn, mpc]
            st = lib.gum_create_mp(ctypes.byref(cfg), ctypes.byref(mpc), ctypes.byref(self._ctx))
            if st != GUM_OK:
                raise GumError(st, "gum_create_mp failed (handshake mismatch, exchange failure or no device)")
        self.rank = int(mp[0]) if mp is not None else 0
        self.num_gpus = int(num_gpus)
        self.num_vertices = 0
        self._last_alg = None

    # ------------------------------------------------------------------ helpers
    def _check(self, st):
        if st != GUM_OK:
            msg = load_library().gum_last_error(self._ctx)
            raise GumError(st, msg.decode() if msg else "")

    def close(self):
        if getattr(self, "_ctx", None) and self._ctx.value:
            load_library().gum_destroy(self._ctx)
            self._ctx = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:  # noqa: BLE001
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    # ------------------------------------------------------------------ ABI
    def load_csr(self, row_ptr, col, weights=None):
        """Copies the CSR (numpy host arrays, pinned torch CPU tensors, or CUDA tensors on worker 0's device)."""
        dev = _is_cuda(row_ptr)
        if not dev:
            row_ptr = row_ptr if hasattr(row_ptr, "data_ptr") else np.ascontiguousarray(row_ptr, dtype=np.uint64)
            col = col if hasattr(col, "data_ptr") else np.ascontiguousarray(col, dtype=np.uint32)
            if weights is not None and not hasattr(weights, "data_ptr"):
                weights = np.ascontiguousarray(weights, dtype=np.uint32)
        V = int(row_ptr.shape[0]) - 1
        E = int(col.shape[0])
        self._check(load_library().gum_load_csr(self._ctx, V, E, _ptr(row_ptr), _ptr(col), _ptr(weights),
                                                LOAD_DEVICE if dev else 0))
        self.num_vertices = V

    def partition(self, kind="seg", seed=0):
        self._check(load_library().gum_partition(self._ctx, PARTS[kind], int(seed)))

    def bounds(self):
        b = np.zeros(MAX_WORKERS + 1, dtype=np.uint32)
        self._check(load_library().gum_partition_bounds(self._ctx, _ptr(b), MAX_WORKERS + 1))
        return b[: self.num_gpus + 1]

    def prepare(self, alg):
        self._check(load_library().gum_prepare(self._ctx, ALGS[alg]))

    def run(self, alg, source=0) -> RunStats:
        s = gum_run_stats()
        self._check(load_library().gum_run(self._ctx, ALGS[alg], int(source), ctypes.byref(s)))
        self._last_alg = alg
        vals = {k: getattr(s, k) for k, _ in gum_run_stats._fields_}
        for k in ("unit_barriers", "unit_last_iter"):
            vals[k] = list(vals[k])[: self.num_gpus]
        return RunStats(**vals)

    def result(self, out=None):
        dt = np.float64 if self._last_alg in ("pr", "dpr") else np.uint32
        if out is None:
            out = np.empty(self.num_vertices, dtype=dt)
        nbytes = out.nbytes if hasattr(out, "nbytes") else out.numel() * out.element_size()
        self._check(load_library().gum_result(self._ctx, _ptr(out), nbytes))
        return out

    def result_device(self, out):
        self._check(load_library().gum_result_device(self._ctx, _ptr(out), out.numel() * out.element_size()))
        return out

    def profile(self):
        """Per-kernel CUDA-event times of the last run (needs profile=True)."""
        k = gum_kernel_times()
        self._check(load_library().gum_profile(self._ctx, ctypes.byref(k)))
        return {n: getattr(k, n) for n, _ in gum_kernel_times._fields_}

    def trace(self):
        n = ctypes.c_uint32()
        buf = (gum_iter_trace * 65536)()
        self._check(load_library().gum_trace(self._ctx, ctypes.cast(buf, ctypes.c_void_p), 65536, ctypes.byref(n)))
        recs = []
        for i in range(n.value):
            r = buf[i]
            recs.append(dict(t_start=list(r.t_start)[: self.num_gpus], t_end=list(r.t_end)[: self.num_gpus],
                             edges_own=list(r.edges_own)[: self.num_gpus],
                             edges_stolen=list(r.edges_stolen)[: self.num_gpus],
                             frontier_vertices=r.frontier_vertices, frontier_edges=r.frontier_edges,
                             owners=r.owners, steal_ok=r.steal_ok))
        return recs


def mp_handshake(rank, world, exchange, **kw):
    """Host-only multi-process handshake (gum_mp_handshake): returns the gum_status (0 = all ranks agree)."""
    cfg, keep = make_config(num_gpus=kw.pop("num_gpus", world), **kw)
    fn = exchange if isinstance(exchange, EXCHANGE_FN) else EXCHANGE_FN(exchange)
    mpc = gum_mp_config(int(rank), int(world), 0, fn, None)
    return int(load_library().gum_mp_handshake(ctypes.byref(cfg), ctypes.byref(mpc)))


def osteal_plan(loads, remote_cost=1.0, p=0.0):
    """NEXT-3 planner (host helper of the device routine): returns (m, [E(1..n)]) of Alg. 2 / Eq. (4)."""
    n = len(loads)
    l = np.ascontiguousarray(loads, dtype=np.uint64)
    cost = np.zeros(n, dtype=np.float64)
    m = ctypes.c_int()
    st = load_library().gum_osteal_plan(_ptr(l), n, float(remote_cost), float(p), _ptr(cost), ctypes.byref(m))
    if st != GUM_OK:
        raise GumError(st, "gum_osteal_plan: bad arguments")
    return m.value, cost


def fsteal_plan(loads, remote_cost=1.0):
    """NEXT-2 planner (host helper of the device routine): returns (z, X) for Eq. (1) on a uniform fabric."""
    n = len(loads)
    l = np.ascontiguousarray(loads, dtype=np.uint64)
    X = np.zeros(n * n, dtype=np.float64)
    z = ctypes.c_double()
    st = load_library().gum_fsteal_plan(_ptr(l), n, float(remote_cost), _ptr(X), ctypes.byref(z))
    if st != GUM_OK:
        raise GumError(st, "gum_fsteal_plan: bad arguments")
    return z.value, X.reshape(n, n)


def version():
    return load_library().gum_version()
