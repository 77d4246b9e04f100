"""Row NEXT-3: the host-side archive writer --
binding of the dedup_archive_* calls of include/dedup.h (argument
marshalling only; the encoder/decoder are C++ in csrc/archive.cpp)."""
from __future__ import annotations

import numpy as np

from . import _native as N


def _p(a):
    return 0 if a is None else a.ctypes.data


def encode(data, starts, digest, is_dup, match_len, match_off, window: int = 4096,
           max_coded: int = 18) -> bytes:
    """One batch's archive records (host numpy arrays; see include/dedup.h)."""
    data = np.ascontiguousarray(data, np.uint8)
    starts = np.ascontiguousarray(starts, np.uint32)
    digest = np.ascontiguousarray(digest, np.uint8)
    is_dup = np.ascontiguousarray(is_dup, np.uint8)
    match_len = np.ascontiguousarray(match_len, np.uint8)
    match_off = np.ascontiguousarray(match_off, np.uint16)
    cap = 29 * len(starts) + len(data) + len(data) // 8 + 64
    out = np.empty(cap, np.uint8)
    n = N.lib().dedup_archive_encode(_p(data), len(data), _p(starts), len(starts), _p(digest),
                                     _p(is_dup), _p(match_len), _p(match_off), window,
                                     max_coded, _p(out), cap)
    if n < 0:
        raise N.DedupError(int(n), "dedup_archive_encode failed")
    return out[:n].tobytes()


class Decoder:
    """Decodes archive records batch by batch (keeps the digest -> chunk map)."""

    def __init__(self, window: int = 4096):
        self._d = N.lib().dedup_archive_decoder_new(window)
        if not self._d:
            raise N.DedupError(N.DEDUP_EINVAL, "dedup_archive_decoder_new failed")

    def decode(self, records: bytes, out_bytes: int) -> np.ndarray:
        src = np.frombuffer(records, np.uint8)
        out = np.empty(max(out_bytes, 1), np.uint8)
        n = N.lib().dedup_archive_decode(self._d, _p(src), len(src), _p(out), out_bytes)
        if n < 0:
            raise N.DedupError(int(n), "dedup_archive_decode failed")
        return out[:n]

    def close(self):
        if self._d:
            N.lib().dedup_archive_decoder_free(self._d)
            self._d = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
