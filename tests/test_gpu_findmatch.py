"""GPU parity of row NEXT-1, LZSS FindMatch (dedup_op_findmatch through the
C ABI) against the CPU oracle (oracle/findmatch_oracle.cpp, Listing 3 of
PAPER.md): bit-exact match lengths and offsets for every byte."""
import numpy as np
import pytest

import oracle
import synthgen

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def cuda():
    assert torch.cuda.is_available(), "GPU tests need a B200"
    from paper_conf_ipps_rockenbachsgmtd19_b200 import build
    build.build()
    return torch.device("cuda:0")


def make_ctx(batch_bytes=8 << 20):
    from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup
    return Dedup(0, batch_bytes=batch_bytes, batch_items=1024, slots=1,
                 table_capacity=1 << 12, host_fed=False)


def gpu_findmatch(d, data, starts, W=4096, MC=18, skip=None, cuda="cuda:0"):
    n = len(data)
    dev = torch.from_numpy(np.concatenate([data, np.zeros(16, np.uint8)])).to(cuda)
    st = torch.from_numpy(np.asarray(starts, np.int64).astype(np.int32)).to(cuda)
    nb = torch.tensor([len(starts)], dtype=torch.int32, device=cuda)
    ln = torch.full((max(n, 1),), 0xAB, dtype=torch.uint8, device=cuda)
    of = torch.full((max(n, 1),), 0x5A5A, dtype=torch.int16, device=cuda)
    sk = None if skip is None else torch.from_numpy(np.asarray(skip, np.uint8)).to(cuda)
    d.op_findmatch(dev, n, st, nb, max(len(starts), 1), ln, of, W, MC, skip=sk)
    torch.cuda.synchronize()
    return ln.cpu().numpy()[:n], of.cpu().numpy().view(np.uint16)[:n]


def assert_parity(d, data, starts, W=4096, MC=18, skip=None):
    gl, go = gpu_findmatch(d, data, starts, W, MC, skip)
    wl, wo = oracle.findmatch(data, starts, W, MC, skip=skip)
    bad = np.nonzero((gl != wl) | (go != wo))[0]
    assert len(bad) == 0, (f"{len(bad)} mismatches, first at {bad[:5]}: gpu "
                           f"{gl[bad[:5]]}/{go[bad[:5]]} oracle {wl[bad[:5]]}/{wo[bad[:5]]}")


def chunk_starts(d, data, item=1 << 20):
    """Block starts from the GPU chunker (the paper's startPos)."""
    n = len(data)
    dev = torch.from_numpy(np.concatenate([data, np.zeros(16, np.uint8)])).to("cuda:0")
    off = synthgen.split_items(data, item).astype(np.int64)
    io = torch.from_numpy(off).cuda()
    cap = n // 32 + len(off) + 2
    cut = torch.zeros(cap, dtype=torch.int32, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
    d.op_chunk(dev, n, io, len(off) - 1, cut, cap, cnt)
    torch.cuda.synchronize()
    k = int(cnt.item())
    return cut[:k].cpu().numpy().astype(np.uint32)


@pytest.mark.parametrize("entropy", [1, 2, 4, 8])
def test_findmatch_random_starts(cuda, entropy):
    rng = np.random.default_rng(entropy)
    n = 150_000 + entropy * 777              # several tiles and a ragged tail
    data = synthgen.make_stream(n, seed=entropy, dup_frac=0.3, entropy=entropy,
                                segment=4096)
    cuts = np.sort(rng.choice(np.arange(1, n), 60, replace=False))
    starts = np.concatenate([[0], cuts]).astype(np.uint32)
    with make_ctx() as d:
        assert_parity(d, data, starts)


@pytest.mark.parametrize("W,MC", [(1, 1), (7, 3), (64, 18), (300, 40), (2048, 255),
                                  (16384, 18)])
def test_findmatch_window_and_length_limits(cuda, W, MC):
    rng = np.random.default_rng(W + MC)
    n = 70_001
    data = synthgen.make_stream(n, seed=W, dup_frac=0.5, entropy=3, segment=2048)
    cuts = np.sort(rng.choice(np.arange(1, n), 9, replace=False))
    starts = np.concatenate([[0], cuts]).astype(np.uint32)
    with make_ctx() as d:
        assert_parity(d, data, starts, W, MC)


def test_findmatch_chunker_blocks(cuda):
    # the paper's pipeline: Rabin startPos -> FindMatch over the whole batch
    data = synthgen.make_stream(3 << 20, seed=11, dup_frac=0.5, segment=64 * 1024)
    with make_ctx() as d:
        starts = chunk_starts(d, data)
        assert starts[0] == 0 and np.all(np.diff(starts.astype(np.int64)) > 0)
        sub = data[:600_000]
        st = starts[starts < len(sub)]
        assert_parity(d, sub, st)


def test_findmatch_runs_and_dense_blocks(cuda):
    with make_ctx() as d:
        run = np.zeros(100_000, np.uint8)
        assert_parity(d, run, np.array([0], np.uint32))              # one long run
        assert_parity(d, run, np.array([0, 5000, 5001, 99_999], np.uint32))
        data = synthgen.make_stream(10_000, seed=3, entropy=1)
        assert_parity(d, data, np.arange(10_000, dtype=np.uint32))   # a block per byte
        assert_parity(d, data, np.arange(0, 10_000, 3, dtype=np.uint32))
        for n in (1, 2, 15, 16, 17, 2047, 2048, 2049):
            assert_parity(d, data[:n], np.array([0], np.uint32))


def test_findmatch_skip_flags(cuda):
    rng = np.random.default_rng(8)
    data = synthgen.make_stream(200_000, seed=8, dup_frac=0.5, entropy=4, segment=8192)
    cuts = np.sort(rng.choice(np.arange(1, len(data)), 40, replace=False))
    starts = np.concatenate([[0], cuts]).astype(np.uint32)
    skip = rng.integers(0, 2, len(starts)).astype(np.uint8)
    with make_ctx() as d:
        assert_parity(d, data, starts, skip=skip)


def test_findmatch_empty_and_bad_args(cuda):
    with make_ctx() as d:
        ln = torch.zeros(16, dtype=torch.uint8, device=cuda)
        of = torch.zeros(16, dtype=torch.int16, device=cuda)
        dev = torch.zeros(32, dtype=torch.uint8, device=cuda)
        st = torch.zeros(1, dtype=torch.int32, device=cuda)
        nb = torch.ones(1, dtype=torch.int32, device=cuda)
        d.op_findmatch(dev, 0, st, nb, 1, ln, of)              # empty batch: no launch
        for W, MC in ((0, 18), (40000, 18), (4096, 0), (4096, 256)):
            with pytest.raises(Exception, match="EINVAL"):
                d.op_findmatch(dev, 16, st, nb, 1, ln, of, W, MC)


def test_findmatch_full_batch_sampled(cuda):
    """The bench's configuration: a 64 MiB batch of the C2 stream with its
    Rabin blocks; oracle on sampled positions (block starts/ends included)."""
    data = synthgen.config_stream("C2", nbytes=64 << 20)
    with make_ctx(batch_bytes=64 << 20) as d:
        starts = chunk_starts(d, data)
        gl, go = gpu_findmatch(d, data, starts)
    rng = np.random.default_rng(0)
    pos = np.concatenate([rng.integers(0, len(data), 20000), starts.astype(np.int64),
                          starts[1:].astype(np.int64) - 1, [len(data) - 1]])
    pos = np.unique(pos).astype(np.uint64)
    wl, wo = oracle.findmatch(data, starts, positions=pos)
    p = pos.astype(np.int64)
    assert np.array_equal(gl[p], wl) and np.array_equal(go[p], wo)
