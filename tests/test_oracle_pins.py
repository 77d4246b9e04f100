"""Pins of the CPU oracle against things other than itself (CPU only).

SHA-1      -> FIPS 180-4 vectors (tests/golden/sha1_fips180.txt) + hashlib.
Fingerprint-> Python big-integer GF(2) long division (tests/pyref.py) at every
              offset, linearity, closed-form special cases, SURVEY App. A.
Chunking   -> brute-force greedy definition over the long-division fp, the
              all-zero closed form, the App. A golden stream, invariants.
Dedup      -> O(n^2) brute force over digests AND bytes, dict re-run.
"""
import hashlib
import json
import os

import numpy as np
import pytest

import oracle
import synthgen
from tests import pyref

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _fips_vectors():
    out = []
    for line in open(os.path.join(GOLD, "sha1_fips180.txt")):
        if line.startswith("#") or not line.strip():
            continue
        spec, dig = line.rstrip("\n").split("\t")
        if spec.startswith("str:"):
            msg = spec[4:].encode()
        else:
            _, cnt, ch = spec.split(":")
            msg = ch.encode() * int(cnt)
        out.append((msg, dig))
    return out


# ---------------------------------------------------------------- SHA-1 -----
@pytest.mark.parametrize("msg,dig", _fips_vectors())
def test_sha1_fips_vectors(msg, dig):
    assert oracle.sha1(np.frombuffer(msg, np.uint8)).hex() == dig


def test_sha1_all_lengths_vs_hashlib():
    rng = np.random.default_rng(0)
    buf = rng.integers(0, 256, 400, dtype=np.uint8)
    for n in range(0, 301):  # covers padding edges 55/56/63/64/119/120
        assert oracle.sha1(buf[:n]) == hashlib.sha1(buf[:n].tobytes()).digest(), n


def test_sha1_random_lengths_vs_hashlib():
    rng = np.random.default_rng(1)
    for n in list(rng.integers(0, 70000, 40)) + [1 << 20, (4 << 20) - 3]:
        b = rng.integers(0, 256, int(n), dtype=np.uint8)
        assert oracle.sha1(b) == hashlib.sha1(b.tobytes()).digest()


# ---------------------------------------------------------- fingerprint -----
def test_tables_match_survey_appendix():
    g = json.load(open(os.path.join(GOLD, "rabin_survey_appA.json")))
    R, Wt = oracle.rabin_tables()
    for k, v in g["R"].items():
        assert int(R[int(k)]) == int(str(v), 0)
    for k, v in g["Wt"].items():
        assert int(Wt[int(k)]) == int(str(v), 0)


def test_tables_are_polynomial_products():
    # R[b] = b t^32 mod P and Wt[b] = b t^248 mod P by long division
    R, Wt = oracle.rabin_tables()
    for b in range(256):
        assert int(R[b]) == pyref.gf2_mod(b << 32)
        assert int(Wt[b]) == pyref.gf2_mod(b << 248)


def test_rolling_fp_equals_long_division_every_offset():
    rng = np.random.default_rng(2)
    data = rng.integers(0, 256, 2048, dtype=np.uint8)
    roll = oracle.rolling_fp(data)
    b = data.tobytes()
    for i in range(31, len(b)):
        assert int(roll[i]) == pyref.fp(b[i - 31:i + 1]), i
    # the Horner form in the oracle agrees too
    for i in range(31, 400):
        assert oracle.fp_window(data[i - 31:i + 1]) == int(roll[i])


def test_fp_special_cases_and_linearity():
    z = np.zeros(32, np.uint8)
    assert oracle.fp_window(z) == 0
    for bval in (1, 7, 0x80, 0xFF):
        w = z.copy()
        w[31] = bval
        assert oracle.fp_window(w) == bval            # degree < 32 -> itself
    w = z.copy()
    w[27] = 1                                          # t^32 -> poly
    assert oracle.fp_window(w) == pyref.POLY
    rng = np.random.default_rng(3)
    for _ in range(50):
        a = rng.integers(0, 256, 32, dtype=np.uint8)
        c = rng.integers(0, 256, 32, dtype=np.uint8)
        assert oracle.fp_window(a ^ c) == oracle.fp_window(a) ^ oracle.fp_window(c)


def test_w256_post_shift_identity():
    g = json.load(open(os.path.join(GOLD, "rabin_survey_appA.json")))
    assert pyref.gf2_mod(1 << 256) == int(g["W256_1"], 0)


# ------------------------------------------------------------- chunking -----
def test_chunk_golden_stream_appendix_a():
    g = json.load(open(os.path.join(GOLD, "rabin_survey_appA.json")))["golden_stream"]
    d = synthgen.splitmix64_bytes(42, g["nbytes"])
    s = oracle.chunk_item(d)
    assert list(map(int, s)) == g["starts"]
    ends = list(map(int, s[1:])) + [len(d)]
    assert oracle.sha1(d[s[0]:ends[0]]).hex() == g["sha1_chunk0"]
    cat = b"".join(oracle.sha1(d[a:e]) for a, e in zip(map(int, s), ends))
    assert hashlib.sha1(cat).hexdigest() == g["sha1_of_concat_digests"]


def test_chunk_all_zero_closed_form():
    for n in (0, 1, 31, 32, 33, 63, 64, 65, 100, 1000):
        s = list(map(int, oracle.chunk_item(np.zeros(n, np.uint8))))
        assert s == list(range(0, n, 32)), n


@pytest.mark.parametrize("seed", range(12))
def test_chunk_bruteforce_tiny(seed):
    rng = np.random.default_rng(100 + seed)
    n = int(rng.integers(0, 700))
    kind = seed % 3
    if kind == 0:
        d = rng.integers(0, 256, n, dtype=np.uint8)
        mask = 0x1F                        # dense anchors so cuts actually occur
    elif kind == 1:
        d = (rng.random(n) < 0.7).astype(np.uint8) * rng.integers(0, 256, n, dtype=np.uint8)
        mask = 0x7
    else:
        d = rng.integers(0, 4, n, dtype=np.uint8)
        mask = 0x3
    p = oracle.Params(anchor_mask=mask)
    got = list(map(int, oracle.chunk_item(d, p)))
    assert got == pyref.chunk_bruteforce(d.tobytes(), mask=mask)


@pytest.mark.parametrize("min_chunk,max_chunk", [(48, 0), (32, 100), (64, 64), (40, 200)])
def test_chunk_bruteforce_min_max(min_chunk, max_chunk):
    rng = np.random.default_rng(min_chunk * 7 + max_chunk)
    d = rng.integers(0, 256, 900, dtype=np.uint8)
    p = oracle.Params(anchor_mask=0xF, min_chunk=min_chunk, max_chunk=max_chunk)
    got = list(map(int, oracle.chunk_item(d, p)))
    assert got == pyref.chunk_bruteforce(d.tobytes(), mask=0xF, min_chunk=min_chunk,
                                         max_chunk=max_chunk)


def test_chunk_invariants_random_1mib():
    d = synthgen.make_stream(1 << 20, seed=9)
    s = oracle.chunk_item(d).astype(np.int64)
    assert s[0] == 0 and np.all(np.diff(s) > 0)
    sizes = np.diff(np.append(s, len(d)))
    assert np.all(sizes[:-1] >= 32)
    # every non-final cut hits the anchor and no earlier eligible hit exists
    roll = oracle.rolling_fp(d)
    hit = (roll & 0xFFF) == 0                 # hit[i] -> cut candidate at i+1
    for a, e in zip(s[:-1], s[1:]):
        assert hit[e - 1]
        assert not np.any(hit[a + 31:e - 1])
    # mean chunk ~ 32 + 4096 (~4127 B)
    assert 3000 < sizes.mean() < 5500


def test_chunk_restart_equals_position_independent_candidates():
    # reading O5/O6: restart-based chunking == candidates on the true sliding
    # window + greedy min-gap 32 (SURVEY App. A equivalence)
    rng = np.random.default_rng(11)
    d = rng.integers(0, 256, 200000, dtype=np.uint8)
    p = oracle.Params(anchor_mask=0x3FF)
    s = list(map(int, oracle.chunk_item(d, p)))
    hit = (oracle.rolling_fp(d) & 0x3FF) == 0
    g, c, n = [], 0, len(d)
    while c < n:
        g.append(c)
        nz = np.nonzero(hit[c + 31:n - 1])[0]
        c = int(c + 31 + nz[0] + 1) if len(nz) else n
    assert s == g


# ---------------------------------------------------------------- dedup -----
def test_dedup_bruteforce_and_dict():
    items = synthgen.make_stream(3 << 20, seed=5, dup_frac=0.6, segment=64 * 1024)
    off = synthgen.split_items(items, 256 * 1024)
    its = [items[int(off[k]):int(off[k + 1])] for k in range(len(off) - 1)]
    res, counts = oracle.dedup_items(its)
    digs, ids, dup, fid, blobs = [], [], [], [], []
    for r, it in zip(res, its):
        ends = list(map(int, r.chunk_start[1:])) + [len(it)]
        for j, (a, e) in enumerate(zip(map(int, r.chunk_start), ends)):
            blobs.append(it[a:e].tobytes())
            digs.append(r.digest[j].tobytes())
            ids.append((r.seq << 32) | j)
            dup.append(int(r.is_dup[j]))
            fid.append(int(r.first_id[j]))
    assert all(hashlib.sha1(b).digest() == d for b, d in zip(blobs, digs))
    n = len(digs)
    # brute force O(n^2) over digests; first_id points at equal BYTES too
    for k in range(n):
        earlier = [j for j in range(k) if digs[j] == digs[k]]
        assert dup[k] == (1 if earlier else 0)
        want = ids[earlier[0]] if earlier else ids[k]
        assert fid[k] == want
        if earlier:
            assert blobs[earlier[0]] == blobs[k]
    # one non-dup per distinct digest; byte accounting
    assert sum(1 for x in dup if x == 0) == len(set(digs))
    dup_bytes = sum(len(b) for b, x in zip(blobs, dup) if x)
    assert counts["dup_bytes"] == dup_bytes
    assert sum(len(b) for b, x in zip(blobs, dup) if not x) + dup_bytes == counts["bytes"]
    ratio = counts["dup_chunks"] / counts["chunks"]
    assert 0.3 < ratio < 0.8


def test_feed_invariance():
    # a stream fed item by item, or in any grouping, gives identical results
    s = synthgen.make_stream(2 << 20, seed=6, dup_frac=0.5, segment=32 * 1024)
    off = synthgen.split_items(s, 100 * 1024)
    its = [s[int(off[k]):int(off[k + 1])] for k in range(len(off) - 1)]
    a, _ = oracle.dedup_items(its)
    st = oracle.Stream()
    b = [st.item(k, it) for k, it in enumerate(its)]
    for x, y in zip(a, b):
        assert np.array_equal(x.chunk_start, y.chunk_start)
        assert np.array_equal(x.digest, y.digest)
        assert np.array_equal(x.first_id, y.first_id)


def test_tiny_and_empty_items():
    res, _ = oracle.dedup_items([np.zeros(0, np.uint8), np.arange(5, dtype=np.uint8),
                                 np.zeros(0, np.uint8), np.arange(5, dtype=np.uint8)])
    assert [len(r.chunk_start) for r in res] == [0, 1, 0, 1]
    assert res[1].is_dup[0] == 0 and res[3].is_dup[0] == 1
    assert int(res[3].first_id[0]) == (1 << 32)


# ------------------------------------------------ threaded variant (8c.6) --
@pytest.mark.parametrize("threads", [1, 3, 8])
def test_items_parallel_equals_sequential_and_hashlib(threads):
    """The threaded driver (steps 2-3 on T threads, step 4 sequential) gives
    the sequential stream's results item by item, across two calls on one
    stream; every digest is re-checked with hashlib and every dup flag with a
    dict over (digest) in stream order."""
    data = synthgen.make_stream(3 << 20, seed=11, dup_frac=0.5, segment=64 * 1024)
    off = list(synthgen.split_items(data, 200 * 1024))
    off = np.array(off[:5] + [off[4], off[4] + 7] + off[5:], np.uint64)  # empty + tiny item
    items = [data[int(off[k]):int(off[k + 1])] for k in range(len(off) - 1)]
    want, _ = oracle.dedup_items(items)
    s = oracle.Stream()
    h = len(items) // 2
    r1 = s.items_parallel(0, data, off[:h + 1], threads)
    r2 = s.items_parallel(h, data[int(off[h]):], off[h:] - off[h], threads)
    s.close()
    got = [r1.item(k) for k in range(h)] + [r2.item(k) for k in range(len(items) - h)]
    seen = {}
    for k, (w, g) in enumerate(zip(want, got)):
        cs, dg, dup, fid = g
        assert np.array_equal(cs, w.chunk_start) and np.array_equal(dg, w.digest)
        assert np.array_equal(dup, w.is_dup) and np.array_equal(fid, w.first_id)
        ends = list(cs[1:]) + [len(items[k])]
        for j, (a, b) in enumerate(zip(cs, ends)):
            d = hashlib.sha1(items[k][a:b].tobytes()).digest()
            assert bytes(dg[j]) == d
            assert dup[j] == (d in seen)
            assert fid[j] == seen.setdefault(d, (k << 32) | j)


# ------------------------------------- NEXT-2: PARSEC literal window (O5-L) --
@pytest.mark.parametrize("seed", range(6))
def test_literal_window_bruteforce(seed):
    """oracle chunk_item(literal_window) == the greedy definition over the
    closed-form literal hash (big-integer long division, tests/pyref.py) on
    small random inputs, dense masks so that cuts happen often."""
    rng = np.random.default_rng(1000 + seed)
    data = rng.integers(0, 256, 300 + 97 * seed, dtype=np.uint8)
    for mask in (0x3, 0xF, 0x3F):
        got = oracle.chunk_item(data, oracle.Params(anchor_mask=mask, literal_window=True))
        want = pyref.chunk_bruteforce_literal(data.tobytes(), mask=mask)
        assert list(got) == want, mask


def test_literal_window_differs_from_true_window_and_zero_closed_form():
    """The literal hash is history-dependent: on random data it cuts
    elsewhere than the true 32-byte window (reading O5); on all-zero data both
    are the same closed form (cuts every 32 bytes)."""
    data = synthgen.splitmix64_bytes(42, 1 << 17)
    lit = oracle.chunk_item(data, oracle.Params(literal_window=True))
    assert list(lit) != list(oracle.chunk_item(data))
    assert lit[0] == 0 and np.all(np.diff(lit.astype(np.int64)) >= 32)
    z = np.zeros(100, np.uint8)
    assert list(oracle.chunk_item(z, oracle.Params(literal_window=True))) == [0, 32, 64, 96]
