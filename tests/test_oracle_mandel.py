"""Pins of the Mandelbrot Streaming oracle (row NEXT-4; PAPER.md Section
IV-A, Listing 1) against things other than itself (CPU only).

* Closed forms of the iteration z <- z^2 + p: p = 0, -1, -2 never leave the
  radius-2 disc (k = niter); p = 1 escapes at k = 2 (1, 2, 5); |p| > 2
  escapes at k = 0; p = 0.25 + 0.5i and others computed by hand.
* Set membership by geometry: points strictly inside the main cardioid or
  the period-2 disc never escape; points outside the radius-2 disc escape
  at once.
* An independent formulation with Python complex numbers and a different
  loop structure, on a coarse image (same IEEE operations, so bit-equal).
* The pixel mapping 255 - floor(k * 255 / niter) and the row/column
  coordinates (row i <-> im = init_b + step * i) on single-point images.
"""
import numpy as np
import pytest

import oracle


@pytest.mark.parametrize("p,k", [(0j, None), (-1 + 0j, None), (-2 + 0j, None),
                                 (1 + 0j, 2), (3 + 0j, 0), (2.5j, 0), (-2.1 + 0j, 0),
                                 (0.5 + 0j, 4), (1j, None), (0.3 + 0.5j, None)])
def test_known_points(p, k):
    niter = 1000
    got = oracle.mandel_iters(p.real, p.imag, niter)
    if k is None:
        # 0, -1 (period 2), -2 (pre-periodic: 0, -2, 2, 2, ...; |z|^2 = 4 is
        # not > 4), i (pre-periodic: i, -1+i, -i, -1+i, ...) and 0.3+0.5i
        # (attracting cycle) never leave the disc
        assert got == niter, p
    else:
        assert got == k, p


def _hand_escape(c, niter):
    # written independently: complex arithmetic, while-loop form
    z, k = 0j, 0
    z = c               # the listing starts at z = p (one step ahead of 0)
    while k < niter:
        if z.real * z.real + z.imag * z.imag > 4.0:
            break
        z = complex(z.real * z.real - z.imag * z.imag + c.real,
                    2 * z.real * z.imag + c.imag)
        k += 1
    return k


def test_point_0_5():
    # p = 0.5: z = 0.5, 0.75, 1.0625, 1.62890625, 3.1533203125: the test at
    # k = 4 sees |z|^2 = 9.94 > 4 -> k = 4
    k = _hand_escape(0.5 + 0j, 100)
    assert oracle.mandel_iters(0.5, 0.0, 100) == k == 4


def test_geometry_membership():
    rng = np.random.default_rng(0)
    niter = 2000
    n_in = n_out = 0
    for _ in range(4000):
        x, y = rng.uniform(-2.5, 1.0), rng.uniform(-1.5, 1.5)
        q = (x - 0.25) ** 2 + y * y
        cardioid = q * (q + (x - 0.25)) < 0.25 * y * y * 0.98      # strictly inside
        bulb = (x + 1) ** 2 + y * y < (1 / 16) * 0.98
        k = oracle.mandel_iters(x, y, niter)
        if cardioid or bulb:
            assert k == niter, (x, y)
            n_in += 1
        if x * x + y * y > 4.0:
            assert k == 0, (x, y)
            n_out += 1
    assert n_in > 500 and n_out > 50


def test_image_vs_complex_formulation():
    dim, niter = 48, 300
    a0, b0, rng_ = -2.125, -1.5, 3.0
    img = oracle.mandel_rows(dim, niter, init_a=a0, init_b=b0, rng=rng_)
    step = rng_ / dim
    for i in range(dim):
        im = b0 + step * i
        for j in range(dim):
            cr = a0 + step * j
            k = _hand_escape(complex(cr, im), niter)
            assert img[i, j] == 255 - (k * 255) // niter, (i, j)


def test_rows_and_mapping():
    dim, niter = 40, 777
    full = oracle.mandel_rows(dim, niter)
    part = oracle.mandel_rows(dim, niter, row0=13, nrows=9)
    assert np.array_equal(part, full[13:22])
    # the pixel at (0, 0) is the point init_a + init_b i
    k = oracle.mandel_iters(oracle.MANDEL_INIT_A, oracle.MANDEL_INIT_B, niter)
    assert full[0, 0] == 255 - (k * 255) // niter
    # inside points map to 0, immediate escapes to 255
    assert (full == 0).any() and (full == 255).any()
    with pytest.raises(ValueError):
        oracle.mandel_rows(dim, niter, row0=35, nrows=9)
