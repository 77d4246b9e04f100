"""GPU tests of the routing ops (row A5: owner split by digest prefix, local
combine) and of the one-process-per-GPU front end of the multi-GPU engine
(dedup_dist_*, world size 1: own share by device copy or NCCL).  G > 1 is tested in
tests/test_gpu_mg.py (G logical ranks on one GPU, the copy transport)."""
import numpy as np
import pytest

import oracle
import synthgen
from tests import gpu_util as U

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

MiB = 1 << 20


def test_route_owner_split_is_by_digest_prefix():
    """Row A5: every routed record lands in its owner's segment."""
    from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup
    rng = np.random.default_rng(3)
    n, G = 5000, 8
    dig = rng.integers(0, 256, (n, 20), dtype=np.uint8)
    ids = np.arange(n, dtype=np.uint64)
    with Dedup(0, batch_bytes=1 << 20, batch_items=4, slots=1, table_capacity=1 << 14) as d:
        td = torch.from_numpy(dig.reshape(-1)).cuda()
        ti = torch.from_numpy(ids.view(np.int64)).cuda()
        tn = torch.tensor([n], dtype=torch.int32, device="cuda")
        send = torch.zeros((n, 4), dtype=torch.int64, device="cuda")
        soff = torch.zeros(G + 1, dtype=torch.int32, device="cuda")
        spos = torch.zeros(n, dtype=torch.int32, device="cuda")
        d.op_route(td, ti, tn, n, G, send, soff, spos)
        torch.cuda.synchronize()
    soff = soff.cpu().numpy()
    raw = send.cpu().numpy().view(np.uint8).reshape(n, 32)
    spos = spos.cpu().numpy()
    own = (dig[:, 0].astype(np.uint64) << 24 | dig[:, 1].astype(np.uint64) << 16 |
           dig[:, 2].astype(np.uint64) << 8 | dig[:, 3].astype(np.uint64)) * G >> 32
    assert soff[0] == 0 and soff[-1] == n
    assert np.array_equal(np.diff(soff), np.bincount(own.astype(np.int64), minlength=G))
    for r in range(n):
        p = spos[r]
        assert soff[own[r]] <= p < soff[own[r] + 1]
        assert np.array_equal(raw[p, :20], dig[r])
        assert raw[p, 24:32].view(np.uint64)[0] == ids[r]


def test_local_combine_representatives():
    """Row A5 local combine: rep[r] = smallest index with an equal digest, on
    duplicate-heavy digests; the local table is left empty (second call on
    different data gives independent answers)."""
    from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup
    rng = np.random.default_rng(11)
    with Dedup(0, batch_bytes=1 << 20, batch_items=4, slots=1, table_capacity=1 << 12) as d:
        for trial, (n, distinct) in enumerate([(5000, 37), (4000, 4000), (3000, 1)]):
            pool = rng.integers(0, 256, (distinct, 20), dtype=np.uint8)
            pick = rng.integers(0, distinct, n)
            dig = pool[pick]
            td = torch.from_numpy(dig.reshape(-1).copy()).cuda()
            tn = torch.tensor([n], dtype=torch.int32, device="cuda")
            rep = torch.full((n,), -1, dtype=torch.int32, device="cuda")
            d.op_local_combine(td, tn, n, rep)
            got = rep.cpu().numpy().astype(np.int64)
            first = {}
            want = np.empty(n, np.int64)
            for r in range(n):
                want[r] = first.setdefault(dig[r].tobytes(), r)
            assert np.array_equal(got, want), trial
            used, _, ovf = d.op_table_status()
            assert ovf == 0


@pytest.fixture(params=["self_copy", "nccl_self"])
def self_path(request, monkeypatch):
    """The rank's own share of the exchange: a device copy (the product
    path), or through NCCL send/recv to itself (DEDUP_MG_NCCL_SELF), which
    is how the NCCL calls of the exchange run at world size 1."""
    if request.param == "nccl_self":
        monkeypatch.setenv("DEDUP_MG_NCCL_SELF", "1")
    else:
        monkeypatch.delenv("DEDUP_MG_NCCL_SELF", raising=False)
    return request.param


@pytest.mark.parametrize("drain", [True, False])
@pytest.mark.parametrize("depth", [1, 3])
def test_native_wave_pipeline_world1(depth, drain, self_path):
    """The one-process-per-GPU front end of the multi-GPU engine (csrc/mg.cpp,
    dedup_dist_*) with one rank: the exchange sends every record to itself
    (a device copy, or NCCL send/recv to itself).  Three dedup streams: the
    first half of the batches, the second half, then the first half again
    from the same device buffers; bit-exact vs the oracle each time.
    drain=False: end_stream with waves in flight (the table reset deferred to
    the next stream's first wave)."""
    assert torch.cuda.is_available()
    from paper_conf_ipps_rockenbachsgmtd19_b200 import dist as D
    data = U.stream(10 * MiB, seed=71 + depth, dup_frac=0.6)
    off = synthgen.split_items(data, MiB // 2)
    n_items = len(off) - 1
    per_batch = 3
    bbytes = per_batch * MiB // 2
    batches = [(k, min(k + per_batch, n_items)) for k in range(0, n_items, per_batch)]
    dev = torch.from_numpy(data).cuda()
    views = [dev[int(off[k]):int(off[j])] for k, j in batches]
    pipe = D.NativeWavePipeline(D.nccl_unique_id(), 1, 0, 0, bbytes, per_batch + 1, 1 << 16,
                                depth=depth)
    split = len(batches) // 2
    plan = [(0, split, 0), (split, len(batches), 0), (0, split, n_items)]  # (lo, hi, seq base)
    got = [[] for _ in plan]
    try:
        def sid_of(seq):  # the three streams' seq ranges are disjoint
            return 2 if seq >= n_items else (0 if seq < batches[split][0] else 1)

        def take(outs, _sid):
            for wave in outs:
                for o in wave:
                    for r in o.items():
                        got[sid_of(r[0])].append(r)
        for sid, (lo, hi, base) in enumerate(plan):
            if sid:
                take(pipe.end_stream(drain=drain), sid - 1)
            for b in range(lo, hi):
                k, j = batches[b]
                take(pipe.submit([(views[b], off[k:j + 1] - off[k], base + k)]), sid)
        take(pipe.flush(), len(plan) - 1)
        torch.cuda.synchronize()
    finally:
        pipe.close()
    for sid, (lo, hi, base) in enumerate(plan):
        k0, k1 = batches[lo][0], batches[hi - 1][1]
        res = sorted(got[sid], key=lambda r: r[0])
        want, _ = oracle.dedup_items([data[int(off[k]):int(off[k + 1])] for k in range(k0, k1)],
                                     first_seq=base + k0)
        assert [g[0] for g in res] == [w.seq for w in want]
        for (seq, cs, dg, dup, fid), w in zip(res, want):
            assert np.array_equal(cs, w.chunk_start), seq
            assert np.array_equal(dg, w.digest), seq
            assert np.array_equal(dup, w.is_dup), seq
            assert np.array_equal(fid, w.first_id), seq


@pytest.mark.parametrize("depth", [2, 4])
def test_native_wave_pipeline_deferred_resets(depth, self_path):
    """end_stream twice in a row with waves in flight (an empty dedup stream
    between two), then a stream that repeats the first one's data: every
    deferred reset lands before the right wave, so the repeat is all-new
    again (bit-exact vs the oracle per stream)."""
    assert torch.cuda.is_available()
    from paper_conf_ipps_rockenbachsgmtd19_b200 import dist as D
    data = U.stream(6 * MiB, seed=97 + depth, dup_frac=0.5)
    off = synthgen.split_items(data, MiB // 2)
    n_items = len(off) - 1
    per_batch = 2
    bbytes = per_batch * MiB // 2
    batches = [(k, min(k + per_batch, n_items)) for k in range(0, n_items, per_batch)]
    dev = torch.from_numpy(data).cuda()
    views = [dev[int(off[k]):int(off[j])] for k, j in batches]
    pipe = D.NativeWavePipeline(D.nccl_unique_id(), 1, 0, 0, bbytes, per_batch + 1, 1 << 16,
                                depth=depth)
    got = {0: [], 1: []}
    try:
        def take(outs):
            for wave in outs:
                for o in wave:
                    for r in o.items():
                        got[0 if r[0] < n_items else 1].append(r)
        for b, (k, j) in enumerate(batches):
            take(pipe.submit([(views[b], off[k:j + 1] - off[k], k)]))
        take(pipe.end_stream(drain=False))
        take(pipe.end_stream(drain=False))  # an empty stream
        for b, (k, j) in enumerate(batches):
            take(pipe.submit([(views[b], off[k:j + 1] - off[k], n_items + k)]))
        take(pipe.flush())
        torch.cuda.synchronize()
    finally:
        pipe.close()
    for sid, base in ((0, 0), (1, n_items)):
        res = sorted(got[sid], key=lambda r: r[0])
        want, _ = oracle.dedup_items([data[int(off[k]):int(off[k + 1])] for k in range(n_items)],
                                     first_seq=base)
        assert [g[0] for g in res] == [w.seq for w in want]
        for (seq, cs, dg, dup, fid), w in zip(res, want):
            assert np.array_equal(cs, w.chunk_start), seq
            assert np.array_equal(dg, w.digest), seq
            assert np.array_equal(dup, w.is_dup), seq
            assert np.array_equal(fid, w.first_id), seq


def test_native_wave_pipeline_rejects_bad_offsets_before_enqueue():
    """Argument checks run before anything is enqueued: a bad
    offset array is EINVAL and the pipeline still works afterwards."""
    from paper_conf_ipps_rockenbachsgmtd19_b200 import dist as D
    from paper_conf_ipps_rockenbachsgmtd19_b200._native import DedupError
    data = U.stream(2 * MiB, seed=5, dup_frac=0.3)
    off = synthgen.split_items(data, MiB // 2)
    dev = torch.from_numpy(data).cuda()
    pipe = D.NativeWavePipeline(D.nccl_unique_id(), 1, 0, 0, 2 * MiB, 8, 1 << 14, depth=2)
    try:
        bad = off.copy()
        bad[1], bad[2] = bad[2], bad[1]          # decreasing
        with pytest.raises(DedupError, match="EINVAL"):
            pipe.submit([(dev, bad, 0)])
        with pytest.raises(DedupError, match="EINVAL"):
            pipe.submit([(dev, off + np.uint64(1), 0)])   # item_off[0] != 0
        got = []
        for outs in (pipe.submit([(dev, off, 0)]), pipe.flush()):
            for wave in outs:
                for o in wave:
                    got.extend(o.items())
    finally:
        pipe.close()
    want, _ = oracle.dedup_items([data[int(off[k]):int(off[k + 1])] for k in range(len(off) - 1)])
    assert [g[0] for g in got] == [w.seq for w in want]
    for (seq, cs, dg, dup, fid), w in zip(got, want):
        assert np.array_equal(cs, w.chunk_start) and np.array_equal(fid, w.first_id), seq


def test_native_wave_pipeline_table_overflow_is_sticky():
    """A full owner shard is reported, not silently turned into wrong dup
    flags: DEDUP_ETABLEFULL, and it stays."""
    from paper_conf_ipps_rockenbachsgmtd19_b200 import dist as D
    from paper_conf_ipps_rockenbachsgmtd19_b200._native import DedupError
    data = U.stream(4 * MiB, seed=9, dup_frac=0.0)
    off = synthgen.split_items(data, MiB)
    dev = torch.from_numpy(data).cuda()
    pipe = D.NativeWavePipeline(D.nccl_unique_id(), 1, 0, 0, 4 * MiB, 8, 16, depth=1)
    try:
        with pytest.raises(DedupError, match="ETABLEFULL"):
            pipe.submit([(dev, off, 0)])
            for _ in range(2):
                pipe.flush()
        with pytest.raises(DedupError, match="ETABLEFULL"):
            pipe.submit([(dev, off, 100)])
    finally:
        pipe.close()
