"""Pins of the fp64 stencil oracle — closed forms and a
pure-Python brute force, independent of the oracle's vectorised code."""
import numpy as np

from oracle import stencil as ost


def brute(a, c0, c1):
    nz, ny, nx = a.shape
    out = np.array(a, np.float64)
    for z in range(1, nz - 1):
        for y in range(1, ny - 1):
            for x in range(1, nx - 1):
                s = 0.0
                for dz, dy, dx in ((-1, 0, 0), (1, 0, 0), (0, -1, 0), (0, 1, 0), (0, 0, -1), (0, 0, 1)):
                    s += float(a[z + dz, y + dy, x + dx])
                out[z, y, x] = c1 * s - c0 * float(a[z, y, x])
    return out


def test_constant_field():
    a = np.full((5, 6, 7), 2.5)
    out = ost.stencil(a, 0.75, 0.5)
    assert np.all(out[1:-1, 1:-1, 1:-1] == (6 * 0.5 - 0.75) * 2.5)
    assert np.array_equal(out[0], a[0]) and np.array_equal(out[:, :, -1], a[:, :, -1])


def test_linear_field_closed_form():
    z, y, x = np.meshgrid(np.arange(6), np.arange(5), np.arange(8), indexing="ij")
    a = 3.0 * x - 2.0 * y + 0.5 * z + 1.0                 # discrete Laplacian of a linear field = 0
    c0, c1 = 1.25, 0.375
    out = ost.stencil(a, c0, c1)
    assert np.allclose(out[1:-1, 1:-1, 1:-1], (6 * c1 - c0) * a[1:-1, 1:-1, 1:-1], rtol=0, atol=1e-12)


def test_brute_force_random():
    g = np.random.default_rng(7)
    a = g.uniform(-1, 1, (4, 5, 6))
    assert np.allclose(ost.stencil(a, 0.3, 1.7), brute(a, 0.3, 1.7), rtol=0, atol=1e-14)


def test_degenerate_grids_copy():
    for shape in ((1, 4, 4), (3, 2, 9), (2, 2, 2)):
        a = np.random.default_rng(1).uniform(-1, 1, shape)
        assert np.array_equal(ost.stencil(a, 0.3, 1.7), a)
