"""Row NEXT-2, the max_chunk chunker variant on the GPU (csrc/maxchunk.cu):
bit-exact against the oracle's chunk_item with max_chunk (forced cut at
c + max_chunk when no anchor comes first), per op and through the engine."""
import numpy as np
import pytest

import oracle
import synthgen
from tests import adversarial as A
from tests import gpu_util as U

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def make_ctx(max_chunk, min_chunk=32, **kw):
    from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup
    base = dict(batch_bytes=8 << 20, batch_items=512, slots=2, table_capacity=1 << 18,
                max_chunk=max_chunk, min_chunk=min_chunk)
    base.update(kw)
    return Dedup(0, **base)


def gpu_cuts(d, data, off):
    n = len(data)
    dev = torch.from_numpy(np.concatenate([data, np.zeros(16, np.uint8)])).cuda()
    io = torch.from_numpy(np.asarray(off, np.uint64).view(np.int64)).cuda()
    cap = n // 32 + len(off) + 2
    cut = torch.zeros(cap, dtype=torch.int32, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
    d.op_chunk(dev, n, io, len(off) - 1, cut, cap, cnt)
    torch.cuda.synchronize()
    return cut[:int(cnt.item())].cpu().numpy().astype(np.int64)


def oracle_cuts(data, off, M, m=32):
    prm = oracle.Params(max_chunk=M, min_chunk=m)
    out = []
    for k in range(len(off) - 1):
        a, b = int(off[k]), int(off[k + 1])
        out.append(oracle.chunk_item(data[a:b], prm).astype(np.int64) + a)
    return np.concatenate(out) if out else np.zeros(0, np.int64)


@pytest.mark.parametrize("M", [64, 100, 4096, 8191, 65536])
def test_op_chunk_max_chunk_random_items(M):
    rng = np.random.default_rng(M)
    data = synthgen.make_stream(3 << 20, seed=M % 97, dup_frac=0.3, segment=64 * 1024)
    lens = rng.integers(0, 300_000, 40)
    off = np.concatenate([[0], np.cumsum(lens)])
    off = off[off <= len(data)].astype(np.uint64)
    data = data[:int(off[-1])]
    with make_ctx(M) as d:
        assert np.array_equal(gpu_cuts(d, data, off), oracle_cuts(data, off, M))


@pytest.mark.parametrize("M", [64, 1000, 20000])
def test_op_chunk_max_chunk_adversarial(M):
    streams = [np.zeros(200_000, np.uint8),                  # a candidate at every byte
               A.constructed_no_hit(400_000, seed=2),        # forced cuts only
               A.constructed_hit(100_000, seed=3)]
    with make_ctx(M) as d:
        for data in streams:
            off = np.array([0, 12345, 12345, 50000, len(data)], np.uint64)
            assert np.array_equal(gpu_cuts(d, data, off), oracle_cuts(data, off, M))


def test_engine_max_chunk_bit_exact():
    M = 16384
    data = U.stream(6 << 20, seed=23, dup_frac=0.5)
    off = synthgen.split_items(data)
    want, _ = oracle.dedup_items(U.items_of(data, off), oracle.Params(max_chunk=M))
    with make_ctx(M, batch_bytes=2 << 20) as d:
        got = U.run_device(d, torch.from_numpy(data).cuda(), off, 2 << 20)
    U.assert_same(got, want)


@pytest.mark.parametrize("m,M", [(64, 0), (100, 0), (256, 4096), (1000, 1000), (33, 65536)])
def test_op_chunk_min_chunk(m, M):
    """min_chunk > window (every item walked with lower bound c + min_chunk)."""
    rng = np.random.default_rng(m + M)
    data = synthgen.make_stream(2 << 20, seed=m, dup_frac=0.3, segment=64 * 1024)
    lens = rng.integers(0, 200_000, 30)
    off = np.concatenate([[0], np.cumsum(lens)])
    off = off[off <= len(data)].astype(np.uint64)
    data = data[:int(off[-1])]
    with make_ctx(M, m) as d:
        assert np.array_equal(gpu_cuts(d, data, off), oracle_cuts(data, off, M, m))
        z = np.zeros(50_000, np.uint8)
        zo = np.array([0, 777, 50_000], np.uint64)
        assert np.array_equal(gpu_cuts(d, z, zo), oracle_cuts(z, zo, M, m))


def test_engine_min_chunk_bit_exact():
    data = U.stream(4 << 20, seed=29, dup_frac=0.5)
    off = synthgen.split_items(data)
    prm = oracle.Params(min_chunk=512, max_chunk=32768)
    want, _ = oracle.dedup_items(U.items_of(data, off), prm)
    with make_ctx(32768, 512, batch_bytes=2 << 20) as d:
        got = U.run_device(d, torch.from_numpy(data).cuda(), off, 2 << 20)
    U.assert_same(got, want)
