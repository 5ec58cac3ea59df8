"""Spawns world_size worker processes joined by a gloo process group on 127.0.0.1 and collects each
rank's return value (tests/test_mp_gloo.py on CPU, tests/test_gpu_mp.py on one GPU)."""
import importlib
import multiprocessing as mp
import os
import socket
import sys
import traceback

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, module, case, args, hide_gpu, q):
    try:
        sys.path.insert(0, ROOT)
        if hide_gpu:
            os.environ["CUDA_VISIBLE_DEVICES"] = ""
        import torch.distributed as dist

        dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
        fn = getattr(importlib.import_module(module), case)
        res = fn(rank, world, *args)
        dist.barrier()
        dist.destroy_process_group()
        q.put((rank, "ok", res))
    except Exception:  # noqa: BLE001
        q.put((rank, "err", traceback.format_exc()))


def run(module, case, world=2, args=(), timeout=120, hide_gpu=True):
    """Runs module.case(rank, world, *args) on `world` spawned ranks; returns the results by rank."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, module, case, args, hide_gpu, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = {}
    try:
        for _ in range(world):
            rank, status, res = q.get(timeout=timeout)
            assert status == "ok", f"rank {rank}:\n{res}"
            out[rank] = res
    finally:
        for p in procs:
            p.join(timeout=30)
            if p.is_alive():
                p.kill()
    return [out[r] for r in range(world)]
