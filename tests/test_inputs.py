"""T1: the seeded input generators (inputs/) -- determinism, structure, statistics."""
import numpy as np

import inputs


def test_rmat_deterministic_and_seeded():
    a = inputs.rmat(10, 8, seed=7)
    b = inputs.rmat(10, 8, seed=7)
    c = inputs.rmat(10, 8, seed=8)
    assert np.array_equal(a.src, b.src) and np.array_equal(a.dst, b.dst) and np.array_equal(a.w, b.w)
    assert not np.array_equal(a.src, c.src)
    assert a.num_edges == (1 << 10) * 8
    assert a.src.max() < 1024 and a.dst.max() < 1024


def test_rmat_weights_range():
    g = inputs.rmat(12, 16, seed=1)
    assert g.w.min() >= 1 and g.w.max() <= 255
    # roughly uniform over [1,255]
    h = np.bincount(g.w, minlength=256)[1:]
    assert h.min() > 0.5 * h.mean()


def test_rmat_quadrant_statistics_unscrambled():
    # Graph500 a,b,c,d = .57,.19,.19,.05: the top src bit is set with prob c+d = .24, top dst bit b+d = .24
    g = inputs.rmat(14, 16, seed=3, scramble=False)
    top = 1 << 13
    ps = ((g.src & top) != 0).mean()
    pd = ((g.dst & top) != 0).mean()
    both = (((g.src & top) != 0) & ((g.dst & top) != 0)).mean()
    assert abs(ps - 0.24) < 0.005 and abs(pd - 0.24) < 0.005 and abs(both - 0.05) < 0.003
    # hubs at low ids without scramble
    deg = np.bincount(g.src, minlength=1 << 14)
    assert deg.argmax() == 0


def test_scramble_is_bijection():
    for bits in (1, 5, 10, 11):
        vals = [inputs.scramble(v, bits, 99) for v in range(1 << bits)]
        assert sorted(vals) == list(range(1 << bits))


def test_scramble_preserves_degree_multiset():
    a = inputs.rmat(11, 8, seed=5, scramble=False, weighted=False)
    b = inputs.rmat(11, 8, seed=5, scramble=True, weighted=False)
    da = np.sort(np.bincount(a.src, minlength=2048))
    db = np.sort(np.bincount(b.src, minlength=2048))
    assert np.array_equal(da, db)


def test_grid_structure():
    n = 17
    g = inputs.grid(n, seed=3)
    assert g.num_vertices == n * n and g.num_edges == 4 * n * (n - 1)
    pairs = {}
    for s, d, w in zip(g.src.tolist(), g.dst.tolist(), g.w.tolist()):
        rs, cs = divmod(s, n)
        rd, cd = divmod(d, n)
        assert abs(rs - rd) + abs(cs - cd) == 1
        pairs[(s, d)] = w
    assert len(pairs) == g.num_edges  # no duplicates
    for (s, d), w in pairs.items():
        assert pairs[(d, s)] == w  # symmetric weights
    assert np.all(np.diff(g.src.astype(np.int64)) >= 0)  # emitted in vertex order


def test_grid_unit_weights():
    g = inputs.grid(9, unit_weights=True)
    assert np.all(g.w == 1)


def test_torus_regular():
    g = inputs.torus(12)
    V = 144
    assert g.num_edges == 4 * V
    assert np.all(np.bincount(g.src, minlength=V) == 4)
    assert np.all(np.bincount(g.dst, minlength=V) == 4)


def test_pick_source_has_outdegree():
    g = inputs.rmat(12, 4, seed=11)
    s = inputs.pick_source(g, 11)
    assert np.bincount(g.src, minlength=g.num_vertices)[s] > 0
    assert s == inputs.pick_source(g, 11)


def test_hash_counter_based():
    assert inputs.hash64(1, 2, 3) == inputs.hash64(1, 2, 3)
    assert inputs.hash64(1, 2, 3) != inputs.hash64(1, 2, 4)
