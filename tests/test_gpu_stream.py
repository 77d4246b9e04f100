"""Row NEXT-2, carry-over chunking (paper_conf_..._b200/stream.py): the whole
stream is one chunking domain, so results must be identical for ANY cut of
the stream into pieces (the north_star invariant "the chunking is identical
when the input is split at arbitrary batch cuts") and equal to the oracle
run on the whole stream as one item."""
import numpy as np
import pytest

import oracle
import synthgen
from tests import adversarial as A

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def run_pieces(data, cuts):
    from paper_conf_ipps_rockenbachsgmtd19_b200.stream import CarryChunker
    dev = torch.from_numpy(data).cuda()
    cc = CarryChunker(0, max_piece=4 << 20, table_capacity=1 << 18)
    parts = []
    try:
        bounds = [0] + list(cuts) + [len(data)]
        for i, (a, b) in enumerate(zip(bounds[:-1], bounds[1:])):
            parts.append(cc.feed(dev[a:b], final=(i == len(bounds) - 2)))
    finally:
        cc.close()
    cat = lambda f: np.concatenate([getattr(p, f) for p in parts])  # noqa: E731
    return cat("offset"), cat("length"), cat("digest"), cat("is_dup"), cat("first_index")


def want_whole(data):
    (r,), _ = oracle.dedup_items([data])
    starts = r.chunk_start.astype(np.uint64)
    lens = np.diff(np.append(starts, np.uint64(len(data))))
    return starts, lens, r.digest, r.is_dup, r.first_id & np.uint64(0xFFFFFFFF)


def check(data, cuts):
    got = run_pieces(data, cuts)
    want = want_whole(data)
    for g, w, name in zip(got, want, ("offset", "length", "digest", "is_dup", "first")):
        assert np.array_equal(g, w), name


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_random_cuts(seed):
    rng = np.random.default_rng(seed)
    data = synthgen.make_stream(3 << 20, seed=seed, dup_frac=0.5, segment=64 * 1024)
    # cuts anywhere: inside windows, tiny pieces, one empty piece
    cuts = sorted(set(rng.integers(1, len(data), 25).tolist()) |
                  {5, 6, 37, 100, 1 << 20, (1 << 20) + 1})
    cuts.insert(3, cuts[2])            # an empty piece
    check(data, cuts)


def test_piece_count_invariance():
    data = synthgen.make_stream(2 << 20, seed=7, dup_frac=0.6, segment=32 * 1024)
    a = run_pieces(data, [])
    b = run_pieces(data, list(range(4096, len(data), 65536 + 13)))
    for x, y in zip(a, b):
        assert np.array_equal(x, y)


def test_adversarial_streams_in_pieces():
    rng = np.random.default_rng(5)
    for data in (np.zeros(300_000, np.uint8),
                 A.constructed_hit(200_000, seed=3),
                 A.constructed_no_hit(300_000, seed=4)):
        cuts = sorted(rng.integers(1, len(data), 7).tolist())
        check(data, cuts)
