"""Adversarial input constructors.  They use the ORACLE
fingerprint (test infrastructure), never the CUDA path."""
import numpy as np

import oracle

MASK = 0xFFF


def constructed_hit(nbytes: int, seed: int) -> np.ndarray:
    """Every 32-byte block's window hits (fp & 0xFFF == 0): the last 1.5
    bytes of each block are solved from the fingerprint."""
    rng = np.random.default_rng(seed)
    nb = nbytes // 32
    d = rng.integers(0, 256, nb * 32, dtype=np.uint8).reshape(nb, 32)
    d[:, 30] &= 0xF0
    d[:, 31] = 0
    for k in range(nb):
        f = oracle.fp_window(d[k])
        d[k, 31] = f & 0xFF
        d[k, 30] |= (f >> 8) & 0xF
    out = np.zeros(nbytes, np.uint8)
    out[:nb * 32] = d.reshape(-1)
    return out


def constructed_no_hit(nbytes: int, seed: int, mask: int = MASK) -> np.ndarray:
    """No window anywhere hits: whenever the window ending at byte j hits,
    flip the low bit of byte j (changes that fingerprint by exactly 1)."""
    rng = np.random.default_rng(seed)
    d = rng.integers(0, 256, nbytes, dtype=np.uint8)
    fp = oracle.rolling_fp(d)
    i = 31
    while True:
        h = np.nonzero((fp[i:] & mask) == 0)[0]
        if len(h) == 0:
            break
        j = i + int(h[0])
        d[j] ^= 1
        lo = j - 31
        hi = min(j + 32, nbytes)
        fp[j:hi] = oracle.rolling_fp(d[lo:hi])[31:31 + (hi - j)]
        i = j
    return d
