"""Multi-process (N>1) host logic on CPU: world_size-2 process groups over gloo (127.0.0.1).

Covers what the one-process-per-GPU path does on the host (include/gum.h gum_mp_handshake /
gum_create_mp, paper_conf_icde_menggltyz23_b200/dist.py): the rank-ordered blob all-gather the library
uses for its IPC-handle and convergence-flag exchanges, the configuration handshake (same status on
every rank, mismatches detected), consistent failure of gum_create_mp without a GPU (no rank hangs),
and bench.py's max-over-ranks timing reduction. The device half (IPC-mapped peers, the signal-pad
barrier) is exercised by tests/test_gpu_mp.py on a GPU.
"""
import pytest

from tests import mp_harness


def _run(case, world=2):
    return mp_harness.run("tests.test_mp_gloo", "case_" + case, world=world)


# ------------------------------------------------------------------------------------------ cases
def _mods():
    import paper_conf_icde_menggltyz23_b200 as gum
    from paper_conf_icde_menggltyz23_b200 import dist as gdist

    return gum, gdist


def case_allgather(rank, world):
    gum, gdist = _mods()
    blobs = gdist.allgather_bytes(bytes([rank] * 5 + [7]))
    return [list(b) for b in blobs]


def case_exchange_callback(rank, world):
    """The C-callable exchange: rank r's block lands at offset r*bytes."""
    import ctypes

    gum, gdist = _mods()
    fn = gdist.allgather_exchange()
    send = (ctypes.c_uint64 * 3)(rank, 100 + rank, 2**40 + rank)
    recv = (ctypes.c_uint64 * (3 * world))()
    rc = fn(ctypes.cast(send, ctypes.c_void_p), ctypes.sizeof(send), ctypes.cast(recv, ctypes.c_void_p), None)
    return rc, list(recv)


def case_handshake_ok(rank, world):
    gum, gdist = _mods()
    return gum.mp_handshake(rank, world, gdist.allgather_exchange(), chunk_edges=1024, osteal_threshold=4096)


def case_handshake_cfg_mismatch(rank, world):
    gum, gdist = _mods()
    return gum.mp_handshake(rank, world, gdist.allgather_exchange(), chunk_edges=1024 if rank == 0 else 2048)


def case_handshake_duplicate_rank(rank, world):
    gum, gdist = _mods()
    return gum.mp_handshake(0, world, gdist.allgather_exchange())


def case_handshake_world_mismatch(rank, world):
    gum, gdist = _mods()
    return gum.mp_handshake(rank, world, gdist.allgather_exchange(), num_gpus=world + 1)


def case_handshake_exchange_failure(rank, world):
    gum, gdist = _mods()
    return gum.mp_handshake(rank, world, gum.EXCHANGE_FN(lambda s, n, r, u: 1))


def case_create_without_gpu(rank, world):
    gum, gdist = _mods()
    try:
        gdist.mp_context(device=0)
    except gum.GumError as e:
        return e.status
    return 0


def case_max_over_ranks(rank, world):
    gum, gdist = _mods()
    import bench

    return gdist.max_over_ranks(1.5 + rank), bench.slowest_rank_ms(10.0 * (rank + 1), world)


# ------------------------------------------------------------------------------------------ tests
def test_allgather_bytes_rank_ordered():
    r = _run("allgather")
    assert r[0] == r[1] == [[0] * 5 + [7], [1] * 5 + [7]]


def test_exchange_callback_layout():
    r = _run("exchange_callback")
    for rc, recv in r:
        assert rc == 0
        assert recv == [0, 100, 2**40, 1, 101, 2**40 + 1]


def test_handshake_agrees():
    assert _run("handshake_ok") == [0, 0]


@pytest.mark.parametrize("case", ["handshake_cfg_mismatch", "handshake_duplicate_rank", "handshake_world_mismatch"])
def test_handshake_mismatch_fails_on_every_rank(case):
    import paper_conf_icde_menggltyz23_b200 as gum

    assert _run(case) == [gum.GUM_EINVAL, gum.GUM_EINVAL]


def test_handshake_exchange_failure_is_enccl():
    import paper_conf_icde_menggltyz23_b200 as gum

    assert _run("handshake_exchange_failure") == [gum.GUM_ENCCL, gum.GUM_ENCCL]


def test_create_mp_without_gpu_fails_consistently():
    """No GPU here: both ranks fail gum_create_mp with the same status and neither hangs (the failure is
    agreed through the exchange), i.e. there is no CPU fallback for the multi-process path either."""
    r = _run("create_without_gpu")
    assert r[0] == r[1] and r[0] < 0


def test_bench_reduces_time_as_max_over_ranks():
    r = _run("max_over_ranks")
    for m, slowest in r:
        assert m == 2.5
        assert slowest == 20.0
