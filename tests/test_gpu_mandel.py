"""GPU parity of row NEXT-4, Mandelbrot Streaming (include/mandel.h through
the C ABI) against the CPU oracle (oracle/mandel_oracle.cpp, Listing 1 of
PAPER.md): bit-identical pixels (the escape counts are integer decisions
taken in binary64 on both sides, operation by operation)."""
import numpy as np
import pytest

import oracle

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def M():
    assert torch.cuda.is_available(), "GPU tests need a B200"
    from paper_conf_ipps_rockenbachsgmtd19_b200 import build
    build.build()
    from paper_conf_ipps_rockenbachsgmtd19_b200 import mandel
    return mandel


def gpu_rows(M, dim, niter, row0=0, nrows=None, **kw):
    nrows = dim - row0 if nrows is None else nrows
    img = torch.full((max(nrows * dim, 1),), 7, dtype=torch.uint8, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
    it = torch.zeros(1, dtype=torch.int64, device="cuda")
    M.rows_device(img, cnt, dim, niter, row0, nrows, iters=it, **kw)
    torch.cuda.synchronize()
    assert it.item() >= 0
    return img.cpu().numpy()[:nrows * dim].reshape(nrows, dim)


@pytest.mark.parametrize("dim,niter", [(1, 1), (7, 3), (64, 1000), (333, 5000), (500, 20000)])
def test_rows_whole_image(M, dim, niter):
    assert np.array_equal(gpu_rows(M, dim, niter), oracle.mandel_rows(dim, niter))


@pytest.mark.parametrize("frame", [(-0.75, 0.1, 0.01), (-1.77, -0.01, 0.02),
                                   (0.25, -0.01, 0.02), (-2.0, -2.0, 4.0)])
def test_rows_zoomed_frames(M, frame):
    # boundary-rich frames (seahorse valley, period-3 bulb, the cusp) where
    # escape counts are long and rounding-sensitive
    a, b, r = frame
    dim, niter = 200, 20000
    want = oracle.mandel_rows(dim, niter, init_a=a, init_b=b, rng=r)
    assert np.array_equal(gpu_rows(M, dim, niter, init_a=a, init_b=b, rng=r), want)


def test_iteration_count(M):
    dim, niter = 50, 500
    img = torch.zeros(dim * dim, dtype=torch.uint8, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
    it = torch.zeros(1, dtype=torch.int64, device="cuda")
    M.rows_device(img, cnt, dim, niter, iters=it)
    torch.cuda.synchronize()
    step = 3.0 / dim
    want = sum(oracle.mandel_iters(-2.125 + step * j, -1.5 + step * i, niter)
               for i in range(dim) for j in range(dim))
    assert it.item() == want


def test_rows_subrange(M):
    dim, niter = 300, 3000
    full = oracle.mandel_rows(dim, niter)
    for row0, n in ((0, 1), (17, 32), (150, 1), (268, 32), (299, 1)):
        assert np.array_equal(gpu_rows(M, dim, niter, row0, n), full[row0:row0 + n])


@pytest.mark.parametrize("batch_rows,spaces", [(32, 1), (32, 2), (32, 4), (7, 3), (1000, 2)])
def test_image_pipeline(M, batch_rows, spaces):
    dim, niter = 400, 4000
    img, ms, it = M.image(dim, niter, batch_rows=batch_rows, spaces=spaces)
    assert ms > 0 and it > 0
    assert np.array_equal(img, oracle.mandel_rows(dim, niter))


def test_paper_workload_sampled_rows(M):
    """The paper's image (2000 x 2000, niter 200,000) through the
    streamed pipeline the bench times (batches of 32 rows, 4 spaces); the
    oracle recomputes sampled rows, including the densest middle rows."""
    dim, niter = 2000, 200000
    img, _, _ = M.image(dim, niter, batch_rows=32, spaces=4)
    for r in (0, 611, 999, 1000, 1385, 1999):
        assert np.array_equal(img[r], oracle.mandel_rows(dim, niter, row0=r, nrows=1)[0]), r


def test_bad_args(M):
    img = torch.zeros(16, dtype=torch.uint8, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
    with pytest.raises(Exception, match="EINVAL"):
        M.rows_device(img, cnt, 4, 100, 3, 2)
    with pytest.raises(Exception, match="EINVAL"):
        M.image(16, 0)
