"""Row NEXT-3, the host-side archive writer: the
encoder run on the oracle's chunking, digests, duplicate flags and LZSS
matches must decode back to the exact input stream (CPU only; the GPU
variant is in test_gpu_archive.py)."""
import numpy as np
import pytest

import oracle
import synthgen
from paper_conf_ipps_rockenbachsgmtd19_b200 import archive


def _batch_inputs(data, items_off, stream):
    """Oracle outputs of one batch of whole items (batch-relative arrays)."""
    starts, digests, dups = [], [], []
    for k in range(len(items_off) - 1):
        a, b = int(items_off[k]), int(items_off[k + 1])
        r = stream.item(k, data[a:b])
        starts.append(r.chunk_start.astype(np.int64) + a)
        digests.append(r.digest)
        dups.append(r.is_dup)
    starts = np.concatenate(starts).astype(np.uint32)
    ln, of = oracle.findmatch(data, starts)
    return starts, np.concatenate(digests), np.concatenate(dups), ln, of


@pytest.mark.parametrize("entropy,dup", [(8, 0.5), (3, 0.3), (1, 0.0)])
def test_roundtrip_oracle_inputs(entropy, dup):
    data = synthgen.make_stream(300_000, seed=entropy, dup_frac=dup, entropy=entropy,
                                segment=32 * 1024)
    off = synthgen.split_items(data, 100_000)
    st = oracle.Stream()
    starts, dg, dups, ln, of = _batch_inputs(data, off, st)
    rec = archive.encode(data, starts, dg, dups, ln.astype(np.uint8), of.astype(np.uint16))
    assert rec.count(b"D") >= 0
    dec = archive.Decoder()
    out = dec.decode(rec, len(data))
    assert np.array_equal(out, data)
    if entropy <= 3:
        assert len(rec) < 0.8 * len(data)          # low-entropy data compresses
    n_dup_records = int(dups.sum())
    assert n_dup_records > 0 or dup == 0.0


def test_two_batches_share_references():
    data = synthgen.make_stream(400_000, seed=9, dup_frac=0.7, segment=16 * 1024)
    off = synthgen.split_items(data, 100_000)
    st = oracle.Stream()
    dec = archive.Decoder()
    outs = []
    for lo, hi in ((0, 2), (2, 4)):                 # batch 2 refers to batch 1's chunks
        a, b = int(off[lo]), int(off[hi])
        sub = data[a:b]
        o = off[lo:hi + 1] - off[lo]
        starts, dg, dups, ln, of = _batch_inputs(sub, o, _Shift(st, lo))
        rec = archive.encode(sub, starts, dg, dups, ln.astype(np.uint8), of.astype(np.uint16))
        outs.append(dec.decode(rec, len(sub)))
    assert np.array_equal(np.concatenate(outs), data)


class _Shift:
    """Stream wrapper giving items of a later batch their global seq."""

    def __init__(self, st, base):
        self.st, self.base = st, base

    def item(self, k, it):
        return self.st.item(self.base + k, it)


def test_rejects_bad_input():
    dec = archive.Decoder()
    with pytest.raises(Exception):
        dec.decode(b"D" + b"\x01" * 20, 100)        # reference to an unknown chunk
    with pytest.raises(Exception):
        dec.decode(b"X" * 30, 100)
    with pytest.raises(Exception):
        archive.encode(np.zeros(10, np.uint8), np.array([0], np.uint32), np.zeros(20, np.uint8),
                       np.zeros(1, np.uint8), np.zeros(10, np.uint8), np.zeros(10, np.uint16),
                       window=2048)
