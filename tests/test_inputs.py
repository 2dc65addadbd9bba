"""Seeded input generators (paper_conf_ipps_rockis13_b200/inputs.py)."""
import numpy as np

from paper_conf_ipps_rockis13_b200 import inputs


def test_splitmix64_reference_vector():
    # Vigna's splitmix64.c with state 0: first outputs
    z = inputs.splitmix64(0, 3)
    assert int(z[0]) == 0xE220A8397B1DCDAF
    assert int(z[1]) == 0x6E789E6AA1B965F4
    assert int(z[2]) == 0x06C45D188009454F
    assert np.array_equal(inputs.splitmix64(5, 4, offset=2), inputs.splitmix64(5, 6)[2:])


def test_uniform_coords_range_and_determinism():
    c = inputs.uniform_coords(1000, 3)
    assert c.dtype == np.int32 and c.shape == (1000, 2)
    assert c.min() >= 0 and c.max() < (1 << 15)
    assert np.array_equal(c, inputs.uniform_coords(1000, 3))
    assert not np.array_equal(c, inputs.uniform_coords(1000, 4))


def test_lattice_distinct_sites():
    for n in (5, 100, 7397):
        c = inputs.lattice_coords(n, 1)
        assert c.min() >= 0 and c.max() < (1 << 15)
        assert len({(int(x), int(y)) for x, y in c}) == n
    c = inputs.lattice_coords(7397, 1)
    assert np.unique(c[:, 0]).size <= 122 and (np.diff(np.unique(c[:, 0])) % 268 == 0).all()


def test_tours_are_permutations():
    for n in (3, 10, 1002):
        coords = inputs.uniform_coords(n, 2)
        for kind in ("random", "hilbert", "identity"):
            t = inputs.make_tour(kind, coords, 2)
            assert t.dtype == np.int32 and sorted(t.tolist()) == list(range(n))


def test_hilbert_index_is_a_bijection_on_small_grid():
    g = np.arange(16)
    x, y = np.meshgrid(g, g)
    h = inputs.hilbert_index(x.ravel(), y.ravel(), order=4)
    assert sorted(h.tolist()) == list(range(256))
    # consecutive indices are grid neighbours
    order = np.argsort(h)
    pts = np.stack([x.ravel()[order], y.ravel()[order]], 1)
    assert (np.abs(np.diff(pts, axis=0)).sum(1) == 1).all()
