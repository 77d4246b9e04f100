"""Helpers for the GPU parity tests (compare the CUDA path with the oracle)."""
import numpy as np

import oracle
import synthgen


def items_of(data, off):
    return [data[int(off[k]):int(off[k + 1])] for k in range(len(off) - 1)]


def batches(off, batch_bytes, batch_items):
    """Greedy grouping of whole items into GPU batches (item index ranges)."""
    out, k, n = [], 0, len(off) - 1
    while k < n:
        j = k + 1
        while (j < n and j - k < batch_items and
               int(off[j + 1]) - int(off[k]) <= batch_bytes):
            j += 1
        out.append((k, j))
        k = j
    return out


def run_device(d, dev_data, off, batch_bytes, batch_items=4096):
    """Submit items resident on the device in batches; drain everything."""
    got = []
    for k, j in batches(off, batch_bytes, batch_items):
        a, b = int(off[k]), int(off[j])
        chunk = dev_data[a:b]
        if a % 16:                       # the C ABI needs 16-byte aligned batches
            chunk = chunk.clone()
        while True:
            try:
                d.submit_device(chunk, off[k:j + 1] - off[k])
                break
            except Exception as e:  # slot ring full: drain one batch first
                if "EAGAIN" not in str(e):
                    raise
                got.extend(d.drain(wait_ms=-1))
    got.extend(d.drain_all())
    return got


def assert_same(got, want, check_dup=True):
    assert len(got) == len(want)
    for g, w in zip(got, want):
        assert g.seq == w.seq and g.item_len == w.item_len
        assert np.array_equal(g.chunk_start, w.chunk_start), f"chunk_start item {g.seq}"
        assert np.array_equal(g.digest, w.digest), f"digest item {g.seq}"
        if check_dup:
            assert np.array_equal(g.is_dup, w.is_dup), f"is_dup item {g.seq}"
            assert np.array_equal(g.first_id, w.first_id), f"first_id item {g.seq}"


def oracle_results(data, off, params=oracle.Params(), first_seq=0):
    res, counts = oracle.dedup_items(items_of(data, off), params, first_seq)
    return res, counts


def stream(nbytes, seed, dup_frac=0.5, segment=64 * 1024):
    return synthgen.make_stream(nbytes, seed=seed, dup_frac=dup_frac, segment=segment)
