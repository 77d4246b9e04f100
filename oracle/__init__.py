"""CPU oracle for the GPU Dedup hot path -- TEST INFRASTRUCTURE ONLY.

Plain, slow, sequential implementation of what the path computes (Rockenbach
et al., IPDPSW 2019, Section IV-B), written in C++
(``dedup_oracle.cpp``) and wrapped here with ctypes.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product (``paper_conf_ipps_rockenbachsgmtd19_b200``) never imports it and
shares no code with it.

Pins (see tests/test_oracle_*.py):
  * SHA-1: FIPS 180-4 test vectors, hashlib on every length 0..300 and random
    lengths (fully pinned).
  * Fingerprint: Python big-integer long division at every offset; linearity;
    closed-form special cases (pinned to the stated definition; equality with
    the PARSEC constants is "parity unpinned" -- reading O1 in DESIGN.md).
  * Chunking: brute-force greedy on tiny inputs, all-zero closed form, the
    SURVEY App. A golden stream, invariants (partition, min size, feed
    invariance).
  * Dedup: O(n^2) brute force over digests and bytes, dict re-run.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "dedup_oracle.cpp")
_SRCS = [_SRC, os.path.join(_HERE, "findmatch_oracle.cpp"),   # NEXT-1 LZSS FindMatch
         os.path.join(_HERE, "mandel_oracle.cpp")]      # NEXT-4 Mandelbrot
_LIB = os.path.join(_HERE, "liboracle.so")

# Defaults (SURVEY 8(c) readings O1-O3, O6, O7).
WINDOW = 32
POLY = 0x45C2B6A1
MASK = 0xFFF
VALUE = 0


def build_oracle(force: bool = False) -> str:
    """Compile the oracle shared library with g++ (no CUDA)."""
    if force or not os.path.exists(_LIB) or any(
            os.path.getmtime(_LIB) < os.path.getmtime(s) for s in _SRCS):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(
            ["g++", "-O2", "-std=c++17", "-ffp-contract=off", "-shared", "-fPIC", "-pthread",
             "-o", tmp,
             *_SRCS])
        os.replace(tmp, _LIB)
    return _LIB


class _Params(ctypes.Structure):
    _fields_ = [("window", ctypes.c_uint32), ("poly", ctypes.c_uint32),
                ("anchor_mask", ctypes.c_uint32), ("anchor_value", ctypes.c_uint32),
                ("min_chunk", ctypes.c_uint32), ("max_chunk", ctypes.c_uint32),
                ("literal_window", ctypes.c_uint32)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build_oracle())
        u8p = ctypes.POINTER(ctypes.c_uint8)
        u32p = ctypes.POINTER(ctypes.c_uint32)
        u64p = ctypes.POINTER(ctypes.c_uint64)
        L.oracle_fp_window.argtypes = [u8p, ctypes.c_uint32, ctypes.c_uint32]
        L.oracle_fp_window.restype = ctypes.c_uint32
        L.oracle_rabin_tables.argtypes = [ctypes.c_uint32, ctypes.c_uint32, u32p, u32p]
        L.oracle_rolling_fp.argtypes = [u8p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32, u32p]
        L.oracle_chunk_item.argtypes = [u8p, ctypes.c_uint64, ctypes.POINTER(_Params), u32p,
                                        ctypes.c_uint64]
        L.oracle_chunk_item.restype = ctypes.c_uint64
        L.oracle_sha1.argtypes = [u8p, ctypes.c_uint64, u8p]
        L.oracle_ctx_new.argtypes = [ctypes.POINTER(_Params)]
        L.oracle_ctx_new.restype = ctypes.c_void_p
        L.oracle_ctx_free.argtypes = [ctypes.c_void_p]
        L.oracle_ctx_item.argtypes = [ctypes.c_void_p, ctypes.c_uint64, u8p, ctypes.c_uint64,
                                      u32p, u8p, u8p, u64p, ctypes.c_uint64]
        L.oracle_ctx_item.restype = ctypes.c_uint64
        L.oracle_ctx_counts.argtypes = [ctypes.c_void_p, u64p]
        L.oracle_ctx_items_parallel.argtypes = [ctypes.c_void_p, ctypes.c_uint64, u8p, u64p,
                                                ctypes.c_uint64, ctypes.c_uint32]
        L.oracle_ctx_items_parallel.restype = ctypes.c_void_p
        L.oracle_batch_chunks.argtypes = [ctypes.c_void_p]
        L.oracle_batch_chunks.restype = ctypes.c_uint64
        L.oracle_batch_times.argtypes = [ctypes.c_void_p, ctypes.POINTER(ctypes.c_double)]
        L.oracle_batch_fetch.argtypes = [ctypes.c_void_p, u64p, u32p, u8p, u8p, u64p]
        L.oracle_batch_free.argtypes = [ctypes.c_void_p]
        L.oracle_max_chunks.argtypes = [ctypes.c_uint64, ctypes.c_uint32]
        L.oracle_max_chunks.restype = ctypes.c_uint64
        L.oracle_findmatch.argtypes = [u8p, ctypes.c_uint64, u32p, ctypes.c_uint32, u8p,
                                       ctypes.c_uint32, ctypes.c_uint32, u64p, ctypes.c_uint64,
                                       u32p, u32p]
        L.oracle_findmatch.restype = ctypes.c_int
        L.oracle_findmatch_block_linear.argtypes = [u32p, ctypes.c_uint32, ctypes.c_uint64]
        L.oracle_findmatch_block_linear.restype = ctypes.c_int64
        L.oracle_mandel_rows.argtypes = [ctypes.c_int32, ctypes.c_int32, ctypes.c_double,
                                         ctypes.c_double, ctypes.c_double, ctypes.c_int32,
                                         ctypes.c_int32, u8p]
        L.oracle_mandel_rows.restype = ctypes.c_int
        L.oracle_mandel_iters.argtypes = [ctypes.c_double, ctypes.c_double, ctypes.c_int32]
        L.oracle_mandel_iters.restype = ctypes.c_int32
        _lib = L
    return _lib


def _u8(a):
    a = np.ascontiguousarray(a, dtype=np.uint8)
    return a, a.ctypes.data_as(ctypes.POINTER(ctypes.c_uint8))


@dataclass(frozen=True)
class Params:
    window: int = WINDOW
    poly: int = POLY
    anchor_mask: int = MASK
    anchor_value: int = VALUE
    min_chunk: int = WINDOW
    max_chunk: int = 0
    literal_window: bool = False  # PARSEC rabinwintab with rf_win = 0 (reading O5-L)

    def c(self) -> _Params:
        return _Params(self.window, self.poly, self.anchor_mask, self.anchor_value,
                       self.min_chunk, self.max_chunk, int(self.literal_window))


def fp_window(window_bytes, poly: int = POLY) -> int:
    a, p = _u8(window_bytes)
    return int(lib().oracle_fp_window(p, len(a), poly))


def rabin_tables(poly: int = POLY, window: int = WINDOW):
    R = np.zeros(256, np.uint32)
    Wt = np.zeros(256, np.uint32)
    lib().oracle_rabin_tables(poly, window, R.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)),
                              Wt.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)))
    return R, Wt


def rolling_fp(data, poly: int = POLY, window: int = WINDOW) -> np.ndarray:
    a, p = _u8(data)
    out = np.zeros(len(a), np.uint32)
    lib().oracle_rolling_fp(p, len(a), poly, window,
                            out.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)))
    return out


def chunk_item(data, params: Params = Params()) -> np.ndarray:
    """Item-relative chunk starts (the paper's startPos)."""
    a, p = _u8(data)
    cap = int(lib().oracle_max_chunks(len(a), params.min_chunk))
    out = np.zeros(max(cap, 1), np.uint32)
    prm = params.c()
    k = lib().oracle_chunk_item(p, len(a), ctypes.byref(prm),
                                out.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)), cap)
    assert k <= cap
    return out[:k].copy()


def sha1(data) -> bytes:
    a, p = _u8(data)
    out = (ctypes.c_uint8 * 20)()
    lib().oracle_sha1(p, len(a), out)
    return bytes(out)


@dataclass
class ItemResult:
    seq: int
    item_len: int
    chunk_start: np.ndarray  # u32 [n]
    digest: np.ndarray       # u8 [n, 20]
    is_dup: np.ndarray       # u8 [n]
    first_id: np.ndarray     # u64 [n]


@dataclass
class BatchResult:
    """Results of Stream.items_parallel: item k's chunks are
    [item_first[k], item_first[k + 1]) of the per-chunk arrays."""
    item_first: np.ndarray   # u64 [n_items + 1]
    chunk_start: np.ndarray  # u32 [m] item-relative
    digest: np.ndarray       # u8 [m, 20]
    is_dup: np.ndarray       # u8 [m]
    first_id: np.ndarray     # u64 [m]
    s_chunk_sha: float       # wall seconds, threaded chunking + SHA-1
    s_dedup: float           # wall seconds, sequential dedup
    threads: int

    def item(self, k: int) -> tuple:
        a, b = int(self.item_first[k]), int(self.item_first[k + 1])
        return (self.chunk_start[a:b], self.digest[a:b], self.is_dup[a:b], self.first_id[a:b])


class Stream:
    """Stateful oracle over one dedup stream (global table across items)."""

    def __init__(self, params: Params = Params()):
        self.params = params
        self._prm = params.c()
        self._ctx = lib().oracle_ctx_new(ctypes.byref(self._prm))

    def close(self):
        if self._ctx:
            lib().oracle_ctx_free(self._ctx)
            self._ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def item(self, seq: int, data) -> ItemResult:
        a, p = _u8(data)
        cap = max(int(lib().oracle_max_chunks(len(a), self.params.min_chunk)), 1)
        cs = np.zeros(cap, np.uint32)
        dg = np.zeros((cap, 20), np.uint8)
        dup = np.zeros(cap, np.uint8)
        fid = np.zeros(cap, np.uint64)
        k = lib().oracle_ctx_item(
            self._ctx, seq, p, len(a), cs.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)),
            dg.ctypes.data_as(ctypes.POINTER(ctypes.c_uint8)),
            dup.ctypes.data_as(ctypes.POINTER(ctypes.c_uint8)),
            fid.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)), cap)
        assert k <= cap
        return ItemResult(seq, len(a), cs[:k].copy(), dg[:k].copy(), dup[:k].copy(),
                          fid[:k].copy())

    def items_parallel(self, seq0: int, buf, item_off, threads: int | None = None):
        """Items buf[item_off[k]:item_off[k+1]] (seq = seq0 + k) with chunking
        and SHA-1 on `threads` host threads (default: all cores) and the dedup
        step sequential.  Returns a BatchResult."""
        a, p = _u8(buf)
        off = np.ascontiguousarray(item_off, dtype=np.uint64)
        n = len(off) - 1
        T = threads or os.cpu_count() or 1
        h = lib().oracle_ctx_items_parallel(
            self._ctx, seq0, p, off.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)), n, T)
        try:
            m = int(lib().oracle_batch_chunks(h))
            r = BatchResult(np.zeros(n + 1, np.uint64), np.zeros(m, np.uint32),
                            np.zeros((m, 20), np.uint8), np.zeros(m, np.uint8),
                            np.zeros(m, np.uint64), 0.0, 0.0, T)
            tt = (ctypes.c_double * 2)()
            lib().oracle_batch_times(h, tt)
            r.s_chunk_sha, r.s_dedup = tt[0], tt[1]
            lib().oracle_batch_fetch(
                h, r.item_first.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)),
                r.chunk_start.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)),
                r.digest.ctypes.data_as(ctypes.POINTER(ctypes.c_uint8)),
                r.is_dup.ctypes.data_as(ctypes.POINTER(ctypes.c_uint8)),
                r.first_id.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)))
        finally:
            lib().oracle_batch_free(h)
        return r

    def counts(self) -> dict:
        out = np.zeros(5, np.uint64)
        lib().oracle_ctx_counts(self._ctx, out.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)))
        return dict(zip(["items", "bytes", "chunks", "dup_chunks", "dup_bytes"],
                        (int(x) for x in out)))


def dedup_items(items, params: Params = Params(), first_seq: int = 0):
    """Run the oracle over a list of items (one fresh stream)."""
    s = Stream(params)
    try:
        return [s.item(first_seq + k, it) for k, it in enumerate(items)], s.counts()
    finally:
        s.close()


# ------------------------------------------------------------------ NEXT-1 --
# LZSS FindMatch (Listing 3; readings L1-L6 in
# findmatch_oracle.cpp and DESIGN.md).
LZSS_WINDOW = 4096
LZSS_MAX_CODED = 18


def findmatch(data, starts, window: int = LZSS_WINDOW, max_coded: int = LZSS_MAX_CODED,
              positions=None, skip=None):
    """(length u32[n], offset u32[n]) for every byte of `data` (or the given
    positions).  `starts`: strictly increasing block starts, starts[0] == 0."""
    a, p = _u8(data)
    st = np.ascontiguousarray(starts, dtype=np.uint32)
    u32p = ctypes.POINTER(ctypes.c_uint32)
    pos = None if positions is None else np.ascontiguousarray(positions, dtype=np.uint64)
    n = len(a) if pos is None else len(pos)
    ln = np.zeros(max(n, 1), np.uint32)
    of = np.zeros(max(n, 1), np.uint32)
    sk = None if skip is None else np.ascontiguousarray(skip, dtype=np.uint8)
    rc = lib().oracle_findmatch(
        p, len(a), st.ctypes.data_as(u32p), len(st),
        None if sk is None else sk.ctypes.data_as(ctypes.POINTER(ctypes.c_uint8)),
        window, max_coded,
        None if pos is None else pos.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)), n,
        ln.ctypes.data_as(u32p), of.ctypes.data_as(u32p))
    if rc != 0:
        raise ValueError("oracle_findmatch: bad arguments")
    return ln[:n].copy(), of[:n].copy()


def findmatch_block_linear(starts, idx: int) -> int:
    """Listing 3 lines 4-10 as listed (linear scan): the block index of idx."""
    st = np.ascontiguousarray(starts, dtype=np.uint32)
    return int(lib().oracle_findmatch_block_linear(
        st.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)), len(st), idx))


# ------------------------------------------------------------------ NEXT-4 --
# Mandelbrot Streaming (Section IV-A, Listing 1; readings
# M1-M4 in mandel_oracle.cpp and DESIGN.md).
MANDEL_INIT_A, MANDEL_INIT_B, MANDEL_RANGE = -2.125, -1.5, 3.0


def mandel_rows(dim: int, niter: int, row0: int = 0, nrows: int | None = None,
                init_a: float = MANDEL_INIT_A, init_b: float = MANDEL_INIT_B,
                rng: float = MANDEL_RANGE) -> np.ndarray:
    """Rows [row0, row0 + nrows) of the dim x dim image (uint8 [nrows, dim])."""
    nrows = dim - row0 if nrows is None else nrows
    out = np.zeros((nrows, dim), np.uint8)
    rc = lib().oracle_mandel_rows(dim, niter, init_a, init_b, rng, row0, nrows,
                                  out.ctypes.data_as(ctypes.POINTER(ctypes.c_uint8)))
    if rc != 0:
        raise ValueError("oracle_mandel_rows: bad arguments")
    return out


def mandel_iters(cr: float, im: float, niter: int) -> int:
    """Escape count k of one point (inner loop of Listing 1)."""
    return int(lib().oracle_mandel_iters(cr, im, niter))
