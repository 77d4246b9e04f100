"""Row NEXT-2, carry-over mode behind the C ABI (dedup_config.carry_over,
csrc/carry.cu): the bytes of a dedup stream are ONE chunking domain and every
submitted item is a piece of it, cut anywhere.  Results must equal the oracle
run on the whole stream as one item, for any cut of the stream into pieces
(north_star: "the chunking is identical when the input is split at arbitrary
batch cuts") -- tiny pieces (< 32 bytes: the window straddles several),
empty pieces, pieces without a cut (the open chunk is carried through), cuts
exactly at piece boundaries -- through the host-fed and device-resident
submits, across dedup streams (end_stream submits the closing item)."""
import numpy as np
import pytest

import oracle
import synthgen
from tests import adversarial as A

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

MiB = 1 << 20


def carry_ctx(**kw):
    from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup
    base = dict(batch_bytes=4 * MiB, batch_items=4, slots=4, table_capacity=1 << 18,
                carry_over=True)
    base.update(kw)
    return Dedup(0, **base)


def random_cuts(n, rng, k, tiny=True):
    cuts = set(rng.integers(1, n, k).tolist())
    if tiny:  # clusters of tiny pieces and empty pieces
        for c in rng.integers(64, n - 64, max(1, k // 4)).tolist():
            cuts.update([c, c + 1, c + 5, c + 37])
    pieces = sorted(cuts)
    out = [0] + pieces + [n]
    bounds = list(zip(out[:-1], out[1:]))
    # empty pieces
    for i in rng.integers(0, len(bounds), max(1, k // 8)).tolist():
        a = bounds[i][0]
        bounds.insert(i, (a, a))
    return bounds


def to_stream(got, piece_start):
    """(stream starts, digests, is_dup, first chunk index) of the reported
    chunks, in order; piece_start[seq] = stream offset of item seq."""
    starts, dig, dup, fid_raw, ids = [], [], [], [], []
    for g in got:
        S = piece_start[g.seq]
        for j in range(g.n_chunks):
            starts.append(S + int(g.chunk_start[j]) - (g.carried if j == 0 else 0))
            ids.append((g.seq << 32) | j)
        dig.append(g.digest)
        dup.append(g.is_dup)
        fid_raw.extend(int(x) for x in g.first_id)
    index = {cid: k for k, cid in enumerate(ids)}
    return (np.array(starts, np.int64), np.concatenate(dig) if dig else np.zeros((0, 20)),
            np.concatenate(dup) if dup else np.zeros(0), np.array([index[f] for f in fid_raw]))


def oracle_stream(data):
    (w,), _ = oracle.dedup_items([data])
    return (w.chunk_start.astype(np.int64), w.digest, w.is_dup,
            (w.first_id & 0xFFFFFFFF).astype(np.int64))


def check(got, piece_start, data):
    gs, gd, gu, gf = to_stream(got, piece_start)
    ws, wd, wu, wf = oracle_stream(data)
    assert np.array_equal(gs, ws)
    assert np.array_equal(gd, wd)
    assert np.array_equal(gu, wu)
    assert np.array_equal(gf, wf)


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_carry_random_cuts_host_fed(seed):
    rng = np.random.default_rng(seed)
    data = synthgen.make_stream(6 * MiB + 777, seed=40 + seed, dup_frac=0.5, segment=64 * 1024)
    bounds = random_cuts(len(data), rng, 40)
    got, ps = [], {}
    with carry_ctx() as d:
        seq = 0
        for a, b in bounds:
            seq = submit_until(d, lambda: d.submit([data[a:b]]), got)
            ps[seq] = a
        ps[seq + 1] = len(data)
        submit_until(d, d.end_stream, got)
        got.extend(d.drain_all())
    check(got, ps, data)


def submit_until(d, fn, got):
    while True:
        try:
            return fn()
        except Exception as e:
            if "EAGAIN" not in str(e):
                raise
            got.extend(d.drain(wait_ms=-1))


def run_stream_device(d, data, bounds, got, ps, seq0):
    dev = torch.from_numpy(data).cuda()
    keep = []
    seq = seq0
    for a, b in bounds:
        piece = dev[a:b].clone() if b > a else dev[:0]
        keep.append(piece)
        s = submit_until(d, lambda: d.submit_device(piece, np.array([0, b - a], np.uint64)), got)
        assert s == seq
        ps[seq] = a
        seq += 1
    ps[seq] = len(data)
    submit_until(d, d.end_stream, got)
    return seq + 1, keep


@pytest.mark.parametrize("kind", ["random", "all_zero", "hit", "no_hit"])
def test_carry_device_streams(kind):
    """Two dedup streams back to back through submit_device (the second one
    repeats the first one's bytes: all new again after the fresh table)."""
    rng = np.random.default_rng(7)
    n = 3 * MiB + 123
    if kind == "random":
        data = synthgen.make_stream(n, seed=9, dup_frac=0.5, segment=32 * 1024)
    elif kind == "all_zero":
        data = np.zeros(n, np.uint8)
    elif kind == "hit":
        data = A.constructed_hit(n, 53)
    else:
        data = A.constructed_no_hit(n, 54)
    bounds = random_cuts(n, rng, 30)
    got1, got2, ps1, ps2 = [], [], {}, {}
    with carry_ctx() as d:
        nxt, k1 = run_stream_device(d, data, bounds, got1, ps1, 0)
        got1.extend(d.drain_all())
        nxt2, k2 = run_stream_device(d, data, bounds[::-1][::-1], got2, ps2, nxt)
        got2.extend(d.drain_all())
    check(got1, ps1, data)
    check(got2, ps2, data)


def test_carry_piece_invariance_and_no_cut_pieces():
    """The same stream cut three ways (incl. pieces far shorter than a chunk,
    so most pieces have no cut and carry the open chunk through) gives the
    same stream results."""
    data = synthgen.make_stream(2 * MiB, seed=77, dup_frac=0.3, segment=32 * 1024)
    n = len(data)
    for step in (1000, 4096 * 3 + 1, 1 << 20):
        bounds = [(a, min(a + step, n)) for a in range(0, n, step)]
        got, ps = [], {}
        with carry_ctx(slots=8) as d:
            nxt, keep = run_stream_device(d, data, bounds, got, ps, 0)
            got.extend(d.drain_all())
        check(got, ps, data)


def test_carry_rejects_unsupported_configs():
    from paper_conf_ipps_rockenbachsgmtd19_b200._native import DedupError
    for kw in (dict(max_chunk=65536), dict(min_chunk=64), dict(slots=1)):
        with pytest.raises(DedupError, match="EUNSUPPORTED"):
            carry_ctx(**kw)
    with carry_ctx() as d:
        dev = torch.zeros(64, dtype=torch.uint8, device="cuda")
        with pytest.raises(DedupError, match="EINVAL"):
            d.submit_device(dev, np.array([0, 32, 64], np.uint64))   # two items
