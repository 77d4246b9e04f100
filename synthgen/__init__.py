"""Seeded synthetic byte streams shared by tests, bench and oracle runs.

This module holds NO arithmetic of the dedup method (no Rabin, no SHA-1, no
table logic): only a counter-mode splitmix64 byte generator and the segment
duplication model of SURVEY.md 8(d) "Synthetic inputs".  Both the CUDA path
and the oracle consume its output; neither is imported here.

Stream model:
  * The stream is cut into segments of ``segment`` bytes (256 KiB).
  * Segment j is, with probability ``dup_frac`` (and if a fresh segment
    exists), an exact copy of one of the last ``ring`` (256) FRESH segments,
    chosen uniformly; otherwise it is fresh.
  * Fresh bytes are splitmix64 counter-mode output (8 bytes per word,
    little-endian).  For ``entropy < 8`` each byte is masked to ``entropy``
    bits and mapped through a fixed seeded permutation of 0..255.
  * Items (the paper's fixed 1 MB batches) are consecutive
    ``item_bytes`` slices of the stream; the last one may be shorter.
"""
from __future__ import annotations

import numpy as np

GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)
_DECISION_SALT = 0xD1B54A32D192ED03
_PERM_SALT = 0x2545F4914F6CDD1D

KiB = 1024
MiB = 1024 * 1024


def splitmix64_words(seed: int, first: int, count: int) -> np.ndarray:
    """Words first..first+count-1 of the splitmix64 stream for ``seed``.

    Word i uses state s_i = seed + (i + 1) * GOLDEN (mod 2^64), then the
    standard splitmix64 finaliser.
    """
    idx = np.arange(first + 1, first + 1 + count, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = np.uint64(seed & 0xFFFFFFFFFFFFFFFF) + idx * GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        z = z ^ (z >> np.uint64(31))
    return z


def splitmix64_bytes(seed: int, nbytes: int, first_byte: int = 0) -> np.ndarray:
    """``nbytes`` bytes of the little-endian splitmix64 byte stream."""
    w0 = first_byte // 8
    w1 = (first_byte + nbytes + 7) // 8
    words = splitmix64_words(seed, w0, max(w1 - w0, 0))
    b = words.astype("<u8").view(np.uint8)
    off = first_byte - 8 * w0
    return b[off:off + nbytes].copy()


def _permutation(seed: int) -> np.ndarray:
    keys = splitmix64_words(seed ^ _PERM_SALT, 0, 256)
    return np.argsort(keys, kind="stable").astype(np.uint8)


def make_stream(nbytes: int, seed: int, dup_frac: float = 0.0, entropy: int = 8,
                segment: int = 256 * KiB, ring: int = 256) -> np.ndarray:
    """One synthetic stream of ``nbytes`` bytes (uint8 array)."""
    out = np.empty(nbytes, np.uint8)
    nseg = (nbytes + segment - 1) // segment
    dec = splitmix64_words(seed ^ _DECISION_SALT, 0, 2 * max(nseg, 1))
    perm = _permutation(seed) if entropy < 8 else None
    fresh_pos: list[int] = []      # stream offsets of fresh segments
    fresh_count = 0
    for j in range(nseg):
        lo = j * segment
        hi = min(lo + segment, nbytes)
        u = float(dec[2 * j] >> np.uint64(11)) / float(1 << 53)
        if fresh_pos and u < dup_frac:
            m = min(len(fresh_pos), ring)
            k = int(dec[2 * j + 1] % np.uint64(m))
            src = fresh_pos[len(fresh_pos) - 1 - k]
            n = min(hi - lo, min(src + segment, nbytes) - src)
            out[lo:lo + n] = out[src:src + n]
            if n < hi - lo:  # source was a short final segment: fill fresh
                out[lo + n:hi] = _fresh(seed, fresh_count, segment, hi - lo - n, perm, entropy)
                fresh_count += 1
        else:
            out[lo:hi] = _fresh(seed, fresh_count, segment, hi - lo, perm, entropy)
            fresh_count += 1
            fresh_pos.append(lo)
            if len(fresh_pos) > ring:
                fresh_pos.pop(0)
    return out


def _fresh(seed, fresh_index, segment, n, perm, entropy):
    b = splitmix64_bytes(seed, n, first_byte=fresh_index * segment)
    if entropy < 8:
        b = perm[b & np.uint8((1 << entropy) - 1)]
    return b


def split_items(stream: np.ndarray, item_bytes: int = MiB) -> np.ndarray:
    """Item offsets (n_items + 1, uint64) cutting ``stream`` into fixed items."""
    n = len(stream)
    k = (n + item_bytes - 1) // item_bytes
    off = np.minimum(np.arange(k + 1, dtype=np.uint64) * np.uint64(item_bytes), np.uint64(n))
    return off


def all_zero(nbytes: int) -> np.ndarray:
    return np.zeros(nbytes, np.uint8)


def all_duplicate(nbytes: int, seed: int, item_bytes: int = MiB) -> np.ndarray:
    """Every item is a copy of item 0."""
    base = splitmix64_bytes(seed, min(item_bytes, nbytes))
    reps = (nbytes + item_bytes - 1) // item_bytes
    return np.tile(base, reps)[:nbytes].copy()


_PATTERNS = None


def _patterns():
    """Stored inputs of C5c(ii)/C5d (synthgen/data/c5_patterns.npz, written by
    tools/make_c5_patterns.py with the oracle fingerprint; here they are only
    XORed and tiled)."""
    global _PATTERNS
    if _PATTERNS is None:
        import os
        z = np.load(os.path.join(os.path.dirname(os.path.abspath(__file__)), "data",
                                 "c5_patterns.npz"))
        _PATTERNS = {k: z[k] for k in z.files}
    return _PATTERNS


def constructed_hit(nbytes: int, seed: int = 53) -> np.ndarray:
    """consecutive 32-byte blocks, each the XOR of a seeded
    random subset of the 32 stored hit blocks (bits of one splitmix64 word per
    block); every block's window hits, so every chunk is one 32-byte block and
    almost all of them are distinct.  Trailing bytes (< 32) are zero."""
    basis = _patterns()["hit_basis"]                  # u8 [32, 32]
    nb = nbytes // 32
    # XOR tables over each byte of the selector word: T[i][b] = XOR of the
    # basis blocks 8i + j for the set bits j of b
    T = np.zeros((4, 256, 32), np.uint8)
    for i in range(4):
        for b in range(1, 256):
            low = b & -b
            j = low.bit_length() - 1
            T[i, b] = T[i, b ^ low] ^ basis[8 * i + j]
    T = T.view(np.uint64)                             # [4, 256, 4] (same bytes)
    sel = splitmix64_words(seed, 0, nb).astype(np.uint32)
    out = np.zeros(nbytes, np.uint8)
    blocks = out[:nb * 32].view(np.uint64).reshape(nb, 4)
    for i in range(4):
        blocks ^= T[i][(sel >> np.uint32(8 * i)) & np.uint32(0xFF)]
    return out


def constructed_no_hit(nbytes: int, item_bytes: int = MiB) -> np.ndarray:
    """item k is the k-th stored 64-byte no-hit pattern tiled
    (no window of the item hits: every item is ONE chunk)."""
    pats = _patterns()["nohit_period"]                # u8 [672, 64]
    out = np.empty(nbytes, np.uint8)
    for k, lo in enumerate(range(0, nbytes, item_bytes)):
        hi = min(lo + item_bytes, nbytes)
        p = pats[k % len(pats)]
        out[lo:hi] = np.tile(p, (hi - lo + 63) // 64)[:hi - lo]
    return out


# Named workloads (BASELINE.json configs).
CONFIGS = {
    "C1": dict(nbytes=10 * MiB, seed=1, dup_frac=0.52, entropy=8),
    "C2": dict(nbytes=184 * MiB, seed=2, dup_frac=0.52, entropy=8),
    "C3": dict(nbytes=672 * MiB, seed=3, dup_frac=0.52, entropy=8),
    "C4": dict(nbytes=16 * 1024 * MiB, seed=4, dup_frac=0.0, entropy=8),
    "C5a": dict(nbytes=672 * MiB, seed=51, dup_frac=0.0, entropy=8),
}


# adversarial streams of BASELINE.json configs[4]
ADVERSARIAL = {
    "C5b": lambda n: all_duplicate(n, seed=52),
    "C5c_zero": all_zero,
    "C5c_hit": lambda n: constructed_hit(n, seed=53),
    "C5d": constructed_no_hit,
}


def config_stream(name: str, nbytes: int | None = None) -> np.ndarray:
    if name in ADVERSARIAL:
        return ADVERSARIAL[name](nbytes if nbytes is not None else 672 * MiB)
    cfg = dict(CONFIGS[name])
    if nbytes is not None:
        cfg["nbytes"] = nbytes
    return make_stream(**cfg)
