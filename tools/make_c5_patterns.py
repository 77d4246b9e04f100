"""Writes synthgen/data/c5_patterns.npz: the stored inputs of the adversarial
streams C5c(ii) (constructed-hit) and C5d (constructed no-hit) of SURVEY
8(d), built with the ORACLE fingerprint only (oracle/ is the one module this
script calls for method arithmetic; the generator in synthgen/ then only
XORs and tiles these stored bytes).

  hit_basis   u8[32, 32]: 32 blocks of 32 bytes, each with
              (fp(block) & 0xFFF) == 0 (last 1.5 bytes solved).
              The fingerprint is linear over GF(2), so every XOR of a subset
              of them hits too: a stream of such blocks cuts every 32 bytes.
  nohit_period u8[672, 64]: per item of C5d a 64-byte pattern whose 64 cyclic
              windows of 32 bytes all miss (fp & 0xFFF != 0): the item (the
              pattern tiled) is one chunk.
Run: python tools/make_c5_patterns.py
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402

MASK = 0xFFF


def hit_block(rng):
    d = rng.integers(0, 256, 32, dtype=np.uint8)
    d[30] &= 0xF0
    d[31] = 0
    f = oracle.fp_window(d)
    d[31] = f & 0xFF
    d[30] |= (f >> 8) & 0xF
    assert oracle.fp_window(d) & MASK == 0
    return d


def gf2_rank(rows):
    vals = [int.from_bytes(r.tobytes(), "big") for r in rows]
    rank = 0
    for bit in range(255, -1, -1):
        piv = next((i for i in range(rank, len(vals)) if vals[i] >> bit & 1), None)
        if piv is None:
            continue
        vals[rank], vals[piv] = vals[piv], vals[rank]
        for i in range(len(vals)):
            if i != rank and vals[i] >> bit & 1:
                vals[i] ^= vals[rank]
        rank += 1
    return rank


def nohit_pattern(rng):
    while True:
        p = rng.integers(0, 256, 64, dtype=np.uint8)
        fp = oracle.rolling_fp(np.concatenate([p, p]))
        if np.all(fp[31:95] & MASK != 0):  # the 64 windows of the periodic stream
            return p


def main():
    rng = np.random.default_rng(0xC5)
    basis = np.stack([hit_block(rng) for _ in range(32)])
    assert gf2_rank(basis) == 32
    pats = np.stack([nohit_pattern(rng) for _ in range(672)])
    out = os.path.join(ROOT, "synthgen", "data", "c5_patterns.npz")
    np.savez_compressed(out, hit_basis=basis, nohit_period=pats)
    print(out)


if __name__ == "__main__":
    main()
