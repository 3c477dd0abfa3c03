"""The seeded generators (graphgen/) — C fast path == numpy restatement, recipe sizes."""
import numpy as np
import pytest


def test_hash_matches_splitmix64_reference_vector(gg):
    # splitmix64 seeded with 0 yields 0xE220A8397B1DCDAF first (Steele/Vigna reference);
    # h(0, 1) = mix64(0x9E3779B97F4A7C15) is exactly that output.
    assert int(gg.hash_fill(0, 1, 1)[0]) == 0xE220A8397B1DCDAF
    assert int(gg.h_np(0, 1)) == 0xE220A8397B1DCDAF
    a = gg.hash_fill(12345, 1000, 4096)
    assert np.array_equal(a, gg.h_np(12345, np.arange(1000, 1000 + 4096)))


def _eq(a, b):
    assert a.n == b.n
    assert np.array_equal(a.src, b.src) and np.array_equal(a.dst, b.dst)
    assert np.array_equal(a.w, b.w)


def test_grid_c_vs_numpy(gg):
    _eq(gg.grid(7, 5, 99), gg.grid_np(7, 5, 99))
    _eq(gg.grid(1, 6, 3), gg.grid_np(1, 6, 3))
    _eq(gg.grid(6, 1, 3), gg.grid_np(6, 1, 3))


def test_road_c_vs_numpy(gg):
    _eq(gg.road(23, 17, 5, 6), gg.road_np(23, 17, 5, 6))


def test_uniform_c_vs_numpy(gg):
    _eq(gg.uniform(1000, 5000, 1, 2, 3), gg.uniform_np(1000, 5000, 1, 2, 3))


def test_rmat_c_vs_numpy(gg):
    _eq(gg.rmat(10, 16 << 10, 4, 3, 2), gg.rmat_np(10, 16 << 10, 4, 3, 2))
    _eq(gg.rmat(8, 1000, 4, None, 2), gg.rmat_np(8, 1000, 4, None, 2))


def test_rmat_quadrant_probabilities(gg):
    # a=.57, b=c=.19, d=.05 per level: check the top-level bit frequencies
    g = gg.rmat(12, 200000, 44, None, 2)
    top_u = (g.src >> 11) & 1
    top_v = (g.dst >> 11) & 1
    f = np.bincount(top_u * 2 + top_v, minlength=4) / g.m
    assert np.allclose(f, [0.57, 0.19, 0.19, 0.05], atol=0.005)


def test_config_grid64_shape(gg):
    g = gg.config(1)
    assert g.n == 4096 and g.m == 8064
    assert g.w.min() >= 1 and g.w.max() <= 1000


def test_config_small_shapes(gg):
    g = gg.config(2, scale_down=8)
    assert g.n == 1 << 14 and g.m == 4 * g.n
    g = gg.config(4, scale_down=10)
    assert g.n == 1 << 12 and g.m == 16 * g.n
    g = gg.config(5, scale_down=8)
    assert g.m == 2048 * g.n // 16
    g = gg.config(3, scale_down=8)
    W = 4890 >> 4
    assert g.n == W * W
    # about 41.4% of interior cells carry a diagonal
    nd = g.m - ((W - 1) * W * 2)
    assert abs(nd / ((W - 1) ** 2) - 0.414) < 0.02
    d = g.w[(W - 1) * W * 2:]
    assert d.min() >= 1414 * 750 // 1000 and d.max() <= 1414 * 1250 // 1000


@pytest.mark.slow
def test_config_road_full_edge_count(gg):
    m = gg._L().gg_road_m(4890, 4890, gg.field_seed(3, 5), 414)
    assert abs(m - 57.71e6) < 0.05e6  # USA: M = 57.7 M
