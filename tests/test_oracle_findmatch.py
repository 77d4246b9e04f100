"""Pins of the LZSS FindMatch oracle (row NEXT-1; Listing 3,
P:227-290) against things other than itself (CPU only).

* An independent formulation through Python's substring search: the
  longest L <= min(MAX_CODED, block_end - i) such that block[i:i+L] occurs
  entirely inside block[max(i - W, 0):i] (bytes.find returns the earliest
  occurrence, i.e. the listing's first-found tie-break; "entirely inside"
  is the listing's `current + j < thisBatchI` non-overlap bound).
* Closed forms: a run of one byte value, a periodic block, distinct bytes.
* Decodability: every (length, offset) pair copies the right bytes from the
  right place (offset = position mod W, reading L2).
* Lines 4-10 of the listing as printed (linear scan) vs the oracle's
  block search (reading L5); skip flags (reading L6).
"""
import numpy as np
import pytest

import oracle
import synthgen


def find_ref(block: bytes, i: int, W: int, MC: int):
    """Longest earlier match of block[i:] via bytes.find (earliest occurrence)."""
    lo = max(i - W, 0)
    for L in range(min(MC, len(block) - i), 0, -1):
        c = block.find(block[i:i + L], lo, i)
        if c >= 0:
            return L, c % W
    return 0, 0


def blocks_of(n, starts):
    ends = list(starts[1:]) + [n]
    return list(zip(starts, ends))


def check_against_find(data, starts, W, MC):
    ln, of = oracle.findmatch(data, starts, W, MC)
    b = bytes(data)
    for s, e in blocks_of(len(data), starts):
        blk = b[s:e]
        for i in range(e - s):
            want = find_ref(blk, i, W, MC)
            assert (int(ln[s + i]), int(of[s + i])) == want, (s, i, want)


def _data(n, seed, entropy):
    return synthgen.make_stream(n, seed=seed, dup_frac=0.0, entropy=entropy)


@pytest.mark.parametrize("entropy", [1, 2, 4, 8])
@pytest.mark.parametrize("W,MC", [(64, 18), (256, 18), (4096, 18), (300, 5), (16, 40)])
def test_findmatch_vs_substring_search(entropy, W, MC):
    rng = np.random.default_rng(entropy * 1000 + W + MC)
    n = 3000
    data = _data(n, seed=int(rng.integers(1 << 30)), entropy=entropy)
    cuts = np.sort(rng.choice(np.arange(1, n), size=6, replace=False))
    starts = np.concatenate([[0], cuts]).astype(np.uint32)
    check_against_find(data, starts, W, MC)


def test_findmatch_text_like():
    # repeated words with variations: long matches, many ties
    words = [b"stream", b"parallel", b"gpu", b"dedup", b"batch", b"block ", b"the "]
    rng = np.random.default_rng(5)
    b = b"".join(words[int(k)] for k in rng.integers(0, len(words), 900))
    data = np.frombuffer(b, np.uint8)
    starts = np.array([0, 700, 1900, 1901, 2500], np.uint32)
    check_against_find(data, starts, 4096, 18)
    check_against_find(data, starts, 100, 30)


@pytest.mark.parametrize("W,MC", [(4096, 18), (37, 7), (8, 255)])
def test_findmatch_run_closed_form(W, MC):
    n = 5000
    data = np.full(n, 0x41, np.uint8)
    ln, of = oracle.findmatch(data, [0], W, MC)
    i = np.arange(n)
    c = np.maximum(i - W, 0)
    want = np.minimum(np.minimum(i - c, n - i), MC)
    assert np.array_equal(ln, want)
    assert np.array_equal(of, np.where(want > 0, c % W, 0))


@pytest.mark.parametrize("period", [1, 3, 17, 200])
def test_findmatch_periodic_closed_form(period):
    W, MC, n = 512, 18, 3000
    pat = np.random.default_rng(period).permutation(256)[:period].astype(np.uint8)
    data = np.resize(pat, n)
    ln, of = oracle.findmatch(data, [0], W, MC)
    for i in range(n):
        if i < period:
            assert ln[i] == 0 and of[i] == 0
            continue
        lo = max(i - W, 0)
        c0 = lo + ((i - lo) % period)          # earliest c >= lo with c == i (mod period)
        L = min(i - c0, n - i, MC)
        assert (ln[i], of[i]) == (L, c0 % W), i


def test_findmatch_distinct_bytes():
    data = np.random.default_rng(1).permutation(256).astype(np.uint8)
    ln, of = oracle.findmatch(data, [0, 100])
    assert not ln.any() and not of.any()


@pytest.mark.parametrize("entropy", [2, 8])
def test_findmatch_decodes(entropy):
    W, MC = 1024, 18
    data = _data(20000, seed=9, entropy=entropy)
    starts = np.array([0, 4000, 4001, 9000, 15000], np.uint32)
    ln, of = oracle.findmatch(data, starts, W, MC)
    for s, e in blocks_of(len(data), starts):
        assert ln[s] == 0 and of[s] == 0          # nothing before a block start
        for i in range(1, e - s):
            L, o = int(ln[s + i]), int(of[s + i])
            assert L <= MC and i + L <= e - s
            if L == 0:
                assert o == 0
                continue
            c = i - ((i - o) % W or W)            # the c in [i - W, i) with c % W == o
            assert max(i - W, 0) <= c and c + L <= i
            assert bytes(data[s + c:s + c + L]) == bytes(data[s + i:s + i + L])


def test_findmatch_block_search_matches_listing():
    rng = np.random.default_rng(3)
    starts = np.concatenate([[0], np.sort(rng.choice(np.arange(1, 5000), 40, replace=False))])
    for idx in list(range(0, 5000, 7)) + [int(x) for x in starts]:
        want = int(np.searchsorted(starts, idx, side="right") - 1)
        assert oracle.findmatch_block_linear(starts, idx) == want


def test_findmatch_positions_and_skip():
    data = _data(6000, seed=4, entropy=3)
    starts = np.array([0, 1000, 2500, 4000], np.uint32)
    ln, of = oracle.findmatch(data, starts, 256, 18)
    pos = np.array([5, 999, 1000, 1001, 3000, 5999], np.uint64)
    l2, o2 = oracle.findmatch(data, starts, 256, 18, positions=pos)
    assert np.array_equal(l2, ln[pos.astype(np.int64)])
    assert np.array_equal(o2, of[pos.astype(np.int64)])
    skip = np.array([0, 1, 0, 1], np.uint8)
    l3, o3 = oracle.findmatch(data, starts, 256, 18, skip=skip)
    for s, e in blocks_of(len(data), starts):
        k = list(starts).index(s)
        if skip[k]:
            assert not l3[s:e].any() and not o3[s:e].any()
        else:
            assert np.array_equal(l3[s:e], ln[s:e]) and np.array_equal(o3[s:e], of[s:e])


def test_findmatch_rejects_bad_starts():
    d = np.zeros(10, np.uint8)
    for bad in ([1], [0, 5, 5], [0, 10], []):
        with pytest.raises(ValueError):
            oracle.findmatch(d, bad)
