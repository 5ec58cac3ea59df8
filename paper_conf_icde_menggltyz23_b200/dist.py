"""Process-group plumbing for the multi-process mode (include/gum.h gum_create_mp).

One process per GPU (the paper's one worker per GPU): torch.distributed is used only on the host
to all-gather small byte blobs -- the configuration handshake and the CUDA IPC handles of every rank's
fragment buffers (and, only in the host-driven loop, the ranks' convergence flags). The data path (remote
atomics, frontier steals, the device barriers of the per-rank CUDA-graph loop, OSteal parking and wake-up)
is one-sided device code in libgum.so and never touches the process group.
"""
from __future__ import annotations

import ctypes
import os

from . import EXCHANGE_FN, Context


def host_group():
    """A gloo group over all ranks (the exchange is host memory, whatever the default backend is)."""
    import torch.distributed as dist

    if dist.get_backend() == "gloo":
        return dist.group.WORLD
    return dist.new_group(backend="gloo")


def allgather_bytes(blob: bytes, group=None) -> list[bytes]:
    """Rank-ordered all-gather of equal-length byte strings over `group`."""
    import torch
    import torch.distributed as dist

    t = torch.frombuffer(bytearray(blob), dtype=torch.uint8) if blob else torch.empty(0, dtype=torch.uint8)
    out = [torch.empty(len(blob), dtype=torch.uint8) for _ in range(dist.get_world_size(group))]
    dist.all_gather(out, t, group=group)
    return [o.numpy().tobytes() for o in out]


def allgather_exchange(group=None):
    """The gum_exchange_fn for `group`: all-gathers `bytes` bytes per rank into recv (rank-ordered).
    Returns 0 on success, 1 on any failure (the library reports GUM_ENCCL)."""

    def _fn(send, nbytes, recv, user):
        try:
            parts = allgather_bytes(ctypes.string_at(send, nbytes), group)
            joined = b"".join(parts)
            ctypes.memmove(recv, joined, len(joined))
            return 0
        except Exception:  # noqa: BLE001 - crossing a C callback boundary: report, do not raise
            return 1

    return EXCHANGE_FN(_fn)


def max_over_ranks(x: float, group=None) -> float:
    """Max of a host scalar over ranks (bench.py: the slowest rank's device time is the job's time)."""
    import torch
    import torch.distributed as dist

    t = torch.tensor([float(x)], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())


def mp_context(device=None, group=None, **kw) -> Context:
    """Collective: this rank's context in multi-process mode (rank/world from torch.distributed,
    device = LOCAL_RANK unless given)."""
    import torch.distributed as dist

    group = group if group is not None else host_group()
    rank, world = dist.get_rank(), dist.get_world_size()
    if device is None:
        device = int(os.environ.get("LOCAL_RANK", rank))
    return Context(num_gpus=world, mp=(rank, world, device, allgather_exchange(group)), **kw)
