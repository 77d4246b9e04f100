"""The adversarial input constructors of SURVEY 8(d) do what their names say,
checked with the oracle (CPU only)."""
import numpy as np

import oracle
import synthgen

MiB = 1 << 20


def test_constructed_hit_cuts_every_32_bytes():
    d = synthgen.constructed_hit(2 * MiB + 40)
    off = synthgen.split_items(d)
    for k in range(len(off) - 1):
        it = d[int(off[k]):int(off[k + 1])]
        s = oracle.chunk_item(it)
        assert np.array_equal(s, np.arange(0, len(it), 32, dtype=np.uint32)), k
    blocks = d[:2 * MiB].reshape(-1, 32)
    assert len(np.unique(blocks, axis=0)) > 0.999 * len(blocks)   # almost all distinct


def test_constructed_no_hit_one_chunk_per_item():
    d = synthgen.constructed_no_hit(5 * MiB + 1000)
    off = synthgen.split_items(d)
    for k in range(len(off) - 1):
        it = d[int(off[k]):int(off[k + 1])]
        assert np.array_equal(oracle.chunk_item(it), [0]), k
        assert not np.any(oracle.rolling_fp(it)[31:] & 0xFFF == 0), k
    assert len({bytes(d[int(off[k]):int(off[k]) + 64]) for k in range(5)}) == 5
