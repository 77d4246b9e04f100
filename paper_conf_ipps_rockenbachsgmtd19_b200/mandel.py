"""Row NEXT-4: Mandelbrot Streaming (Section IV-A) -- binding of
include/mandel.h (argument marshalling only; the pixels are computed by the
sm_100a kernel in csrc/mandel.cu)."""
from __future__ import annotations

import ctypes

import numpy as np

from . import _native as N

# reading M1: the frame that holds the whole set
INIT_A, INIT_B, RANGE = -2.125, -1.5, 3.0


def rows_device(img, counter, dim: int, niter: int, row0: int = 0, nrows: int | None = None,
                init_a: float = INIT_A, init_b: float = INIT_B, rng: float = RANGE,
                stream=None, iters=None) -> None:
    """Stream-ordered: rows [row0, row0 + nrows) into the device tensor `img`
    (uint8, nrows * dim); `counter`: a device int32/uint32 tensor of >= 1
    element (scratch); `iters` (optional): a device int64 tensor the number of
    computed iterations is added to."""
    nrows = dim - row0 if nrows is None else nrows
    s = 0 if stream is None else (stream if isinstance(stream, int) else stream.cuda_stream)
    N.check(N.lib().mandel_rows_device(s, dim, niter, init_a, init_b, rng, row0, nrows,
                                       img.data_ptr(), counter.data_ptr(),
                                       0 if iters is None else iters.data_ptr()))


def image(dim: int, niter: int, batch_rows: int = 32, spaces: int = 2,
          init_a: float = INIT_A, init_b: float = INIT_B, rng: float = RANGE,
          devices=(0,), out: np.ndarray | None = None):
    """The whole dim x dim image through the streamed pipeline (batches of
    rows, memory spaces round-robin over `devices`).  Returns (img, ms, iters):
    host wall ms of the streamed computation and the iterations computed."""
    img = np.empty((dim, dim), np.uint8) if out is None else out
    assert img.dtype == np.uint8 and img.flags.c_contiguous and img.size == dim * dim
    ids = (ctypes.c_int32 * len(devices))(*devices)
    cfg = N.MandelConfig(dim, niter, init_a, init_b, rng, batch_rows, spaces, len(devices), ids)
    ms = ctypes.c_double(0.0)
    it = ctypes.c_uint64(0)
    N.check(N.lib().mandel_image(ctypes.byref(cfg), img.ctypes.data, ctypes.byref(ms),
                                 ctypes.byref(it)))
    return img, ms.value, it.value
