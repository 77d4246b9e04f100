"""GPU parity: the CUDA path through the C ABI vs the CPU oracle, bit-exact
on every output (chunk starts, digests, dup flags, first-occurrence ids)."""
import hashlib

import numpy as np
import pytest

import oracle
import synthgen
from tests import adversarial as A
from tests import gpu_util as U

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def cuda():
    assert torch.cuda.is_available(), "GPU tests need a B200"
    from paper_conf_ipps_rockenbachsgmtd19_b200 import build
    build.build()
    return torch.device("cuda:0")


# The engine tests run through dedup_init on every engine of include/dedup.h:
# the single-GPU engine, and the multi-GPU engine (csrc/mg.cpp) with one rank
# over NCCL, with 2 / 4 logical ranks on this GPU (copy transport) and with 2 /
# 8 logical ranks exchanging through the owners' shards (p2p transport: remote
# insert / lookup kernels; on one GPU the peer pointers are local).
ENGINES = ["single", "nccl1", "copy2", "copy4", "p2p2", "p2p8"]


def make_ctx(engine="single", **kw):
    from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup
    base = dict(batch_bytes=8 << 20, batch_items=1024, slots=3, table_capacity=1 << 18)
    base.update(kw)
    if engine != "single":
        G = {"nccl1": 1, "copy2": 2, "copy4": 4, "p2p2": 2, "p2p8": 8}[engine]
        transport = 1 if engine == "nccl1" else (3 if engine.startswith("p2p") else 2)
        base.update(num_devices=G, device_ids=[0] * G, transport=transport,
                    slots=min(base["slots"], 4))
    return Dedup(0, **base)


# ------------------------------------------------------------ SHA-1 op -----
def test_op_sha1_all_lengths_and_alignments(cuda):
    rng = np.random.default_rng(0)
    lens = list(range(1, 301)) + list(rng.integers(1, 20000, 200)) + [65536, 1 << 20]
    cuts = np.concatenate([[0], np.cumsum(lens)[:-1]]).astype(np.int64)
    total = int(np.sum(lens))
    data = rng.integers(0, 256, total, dtype=np.uint8)
    with make_ctx(batch_bytes=4 << 20) as d:
        dev = torch.from_numpy(data).to(cuda)
        cut = torch.from_numpy(cuts.astype(np.int32)).to(cuda)
        n = torch.tensor([len(lens)], dtype=torch.int32, device=cuda)
        dig = torch.zeros(len(lens) * 20, dtype=torch.uint8, device=cuda)
        d.op_sha1(dev, total, cut, n, len(lens), dig)
        torch.cuda.synchronize()
        got = dig.cpu().numpy().reshape(-1, 20)
    for k, (a, L) in enumerate(zip(cuts, lens)):
        assert got[k].tobytes() == hashlib.sha1(data[a:a + L].tobytes()).digest(), (k, L, a % 16)


def test_op_sha1_single_chunk_at_buffer_end(cuda):
    # chunk ends exactly at an unpadded buffer end (guarded tail loads)
    rng = np.random.default_rng(1)
    for total in (1, 15, 16, 17, 55, 56, 64, 119, 4097):
        data = rng.integers(0, 256, total, dtype=np.uint8)
        with make_ctx(batch_bytes=1 << 16) as d:
            dev = torch.from_numpy(data).to(cuda)
            cut = torch.zeros(1, dtype=torch.int32, device=cuda)
            n = torch.ones(1, dtype=torch.int32, device=cuda)
            dig = torch.zeros(20, dtype=torch.uint8, device=cuda)
            d.op_sha1(dev, total, cut, n, 1, dig)
            torch.cuda.synchronize()
            assert dig.cpu().numpy().tobytes() == hashlib.sha1(data.tobytes()).digest()


# ------------------------------------------------------------ chunk op -----
def run_op_chunk(d, data, off, cuda):
    nbytes = len(data)
    dev = torch.from_numpy(np.concatenate([data, np.zeros(16, np.uint8)])).to(cuda)
    offt = torch.from_numpy(off.astype(np.int64)).to(cuda)
    cap = nbytes // 32 + len(off) + 2
    cut = torch.zeros(cap, dtype=torch.int32, device=cuda)
    n = torch.zeros(1, dtype=torch.int32, device=cuda)
    d.op_chunk(dev, nbytes, offt, len(off) - 1, cut, cap, n)
    torch.cuda.synchronize()
    k = int(n.item())
    assert k <= cap
    return cut[:k].cpu().numpy().astype(np.int64)


def oracle_cuts(data, off, params):
    out = []
    for k in range(len(off) - 1):
        a, b = int(off[k]), int(off[k + 1])
        out.extend(int(x) + a for x in oracle.chunk_item(data[a:b], params))
    return np.array(out, np.int64)


@pytest.mark.parametrize("mask", [0xFFF, 0x3F, 0x3, 0x0])
def test_op_chunk_edge_items(cuda, mask):
    rng = np.random.default_rng(mask)
    lens = [0, 1, 31, 32, 33, 63, 64, 65, 0, 4095, 4096, 4097, 8191, 8192, 8193, 100000,
            0, 0, 3, 70000, 1 << 18]
    data = rng.integers(0, 256, sum(lens), dtype=np.uint8)
    off = np.concatenate([[0], np.cumsum(lens)]).astype(np.uint64)
    p = oracle.Params(anchor_mask=mask)
    with make_ctx(anchor_mask=mask) as d:
        got = run_op_chunk(d, data, off, cuda)
    assert np.array_equal(got, oracle_cuts(data, off, p))


def test_op_chunk_anchor_value_and_poly(cuda):
    rng = np.random.default_rng(5)
    data = rng.integers(0, 256, 300000, dtype=np.uint8)
    off = np.array([0, 100, 150000, 300000], np.uint64)
    p = oracle.Params(anchor_mask=0x1FF, anchor_value=0x0A5, poly=0x04C11DB7)
    with make_ctx(anchor_mask=0x1FF, anchor_value=0x0A5, poly=0x04C11DB7) as d:
        got = run_op_chunk(d, data, off, cuda)
    assert np.array_equal(got, oracle_cuts(data, off, p))


@pytest.mark.parametrize("seed", range(4))
def test_op_chunk_random_items_many_tiles(cuda, seed):
    rng = np.random.default_rng(10 + seed)
    lens = list(rng.integers(0, 200000, 30)) + list(rng.integers(0, 64, 30))
    rng.shuffle(lens)
    data = (rng.integers(0, 256, int(sum(lens)), dtype=np.uint8)
            if seed % 2 == 0 else (rng.random(int(sum(lens))) < 0.3).astype(np.uint8))
    off = np.concatenate([[0], np.cumsum(lens)]).astype(np.uint64)
    mask = [0xFFF, 0x7F, 0x1F, 0xFF][seed]
    with make_ctx(anchor_mask=mask) as d:
        got = run_op_chunk(d, data, off, cuda)
    assert np.array_equal(got, oracle_cuts(data, off, oracle.Params(anchor_mask=mask)))


def test_op_chunk_all_zero(cuda):
    with make_ctx() as d:
        for n in (100, 8192 * 3 + 17, 1 << 20):
            data = np.zeros(n, np.uint8)
            off = np.array([0, n], np.uint64)
            got = run_op_chunk(d, data, off, cuda)
            assert np.array_equal(got, np.arange(0, n, 32))


def test_op_chunk_many_tiny_items(cuda):
    rng = np.random.default_rng(3)
    lens = rng.integers(0, 40, 5000)
    data = np.zeros(int(lens.sum()), np.uint8)
    off = np.concatenate([[0], np.cumsum(lens)]).astype(np.uint64)
    with make_ctx(batch_items=8192) as d:
        got = run_op_chunk(d, data, off, cuda)
    assert np.array_equal(got, oracle_cuts(data, off, oracle.Params()))


# ------------------------------------------------------------ table op -----
def test_op_table_min_id_semantics(cuda):
    rng = np.random.default_rng(7)
    n = 50000
    uniq = rng.integers(0, 256, (9000, 20), dtype=np.uint8)
    pick = rng.integers(0, 9000, n)
    dig = uniq[pick]
    ids = rng.permutation(n).astype(np.uint64) * 3 + 1
    with make_ctx() as d:
        tdig = torch.from_numpy(dig.reshape(-1)).to(cuda)
        tid = torch.from_numpy(ids.view(np.int64)).to(cuda)
        tn = torch.tensor([n], dtype=torch.int32, device=cuda)
        fid = torch.zeros(n, dtype=torch.int64, device=cuda)
        dup = torch.zeros(n, dtype=torch.uint8, device=cuda)
        d.op_table_reset()
        d.op_table(tdig, tid, tn, n, fid, dup)
        torch.cuda.synchronize()
        used, slots, ovf = d.op_table_status()
    fid = fid.cpu().numpy().view(np.uint64)
    best = {}
    for k in range(n):
        key = dig[k].tobytes()
        best[key] = min(best.get(key, 1 << 64), int(ids[k]))
    want = np.array([best[dig[k].tobytes()] for k in range(n)], np.uint64)
    assert np.array_equal(fid, want)
    assert np.array_equal(dup.cpu().numpy(), (want != ids).astype(np.uint8))
    assert used == len(best) and ovf == 0


# -------------------------------------------------------- full pipeline ----
@pytest.mark.parametrize("engine", ENGINES)
def test_engine_c1_bit_exact_device(cuda, engine):
    data = synthgen.config_stream("C1")
    off = synthgen.split_items(data)
    want, counts = U.oracle_results(data, off)
    assert 0.3 < counts["dup_chunks"] / counts["chunks"] < 0.7
    with make_ctx(engine, batch_bytes=4 << 20) as d:
        got = U.run_device(d, torch.from_numpy(data).to(cuda), off, 4 << 20)
        st = d.stats()
    U.assert_same(got, want)
    assert st["chunks"] == counts["chunks"] and st["dup_chunks"] == counts["dup_chunks"]
    assert st["dup_bytes"] == counts["dup_bytes"] and st["bytes"] == counts["bytes"]


@pytest.mark.parametrize("engine", ENGINES)
def test_engine_c1_host_fed(cuda, engine):
    data = synthgen.config_stream("C1")
    off = synthgen.split_items(data)
    want, _ = U.oracle_results(data, off)
    with make_ctx(engine, batch_bytes=3 << 20) as d:
        items = U.items_of(data, off)
        got = []
        for k in range(0, len(items), 3):
            d.submit(items[k:k + 3])
            got.extend(d.drain(wait_ms=-1))
        got.extend(d.drain_all())
        # pinned zero-copy buffer path
        pin = d.host_empty(len(data))
        pin[:] = data
        d.end_stream()
        s0 = d.submit_buffer(pin[:int(off[5])], off[:6])
        got2 = d.drain_all()
    U.assert_same(got, want)
    want2, _ = U.oracle_results(data, off[:6], first_seq=s0)
    U.assert_same(got2, want2)


@pytest.mark.parametrize("engine", ENGINES)
@pytest.mark.parametrize("batch_mb", [1, 2, 8])
def test_batch_size_invariance(cuda, batch_mb, engine):
    data = U.stream(12 << 20, seed=21, dup_frac=0.5)
    off = synthgen.split_items(data)
    want, _ = U.oracle_results(data, off)
    with make_ctx(engine, batch_bytes=batch_mb << 20, slots=2) as d:
        got = U.run_device(d, torch.from_numpy(data).to(cuda), off, batch_mb << 20)
    U.assert_same(got, want)


@pytest.mark.parametrize("engine", ENGINES)
def test_full_batches_not_a_tile_multiple(cuda, engine):
    """Batches of exactly batch_bytes where batch_bytes is not a multiple of
    the scan's 8 KiB selection tile: the last, partial tile of every batch is
    written whole into the candidate bitmap (sized in whole tiles), and the
    results stay bit-exact (run under compute-sanitizer memcheck by
    tools/gpu_sanitize.sh)."""
    bb = 1_000_003
    data = U.stream(4 * bb, seed=33, dup_frac=0.5)
    off = np.array([0, bb, 2 * bb, 2 * bb + 5, 3 * bb, 4 * bb], np.uint64)
    want, _ = U.oracle_results(data, off)
    with make_ctx(engine, batch_bytes=bb, batch_items=4, slots=2) as d:
        got = U.run_device(d, torch.from_numpy(data).to(cuda), off, bb, 4)
    U.assert_same(got, want)


@pytest.mark.parametrize("engine", ENGINES)
def test_tiny_and_empty_items_pipeline(cuda, engine):
    rng = np.random.default_rng(4)
    lens = [0, 5, 0, 5, 31, 32, 33, 0, 64, 1000, 0, 5]
    base = rng.integers(0, 256, 2000, dtype=np.uint8)
    data = np.concatenate([base[:L] for L in lens]) if sum(lens) else np.zeros(0, np.uint8)
    off = np.concatenate([[0], np.cumsum(lens)]).astype(np.uint64)
    want, _ = U.oracle_results(data, off)
    with make_ctx(engine, batch_bytes=1 << 16, batch_items=4) as d:
        got = U.run_device(d, torch.from_numpy(np.concatenate([data, np.zeros(16, np.uint8)]))
                           .to(cuda), off, 1 << 16, 4)
    U.assert_same(got, want)


@pytest.mark.parametrize("engine", ENGINES)
@pytest.mark.parametrize("kind", ["all_zero", "hit", "no_hit", "all_dup"])
def test_adversarial_streams(cuda, kind, engine):
    n = 4 << 20
    if kind == "all_zero":
        data = np.zeros(n, np.uint8)
    elif kind == "hit":
        data = A.constructed_hit(n, 53)
    elif kind == "no_hit":
        data = A.constructed_no_hit(n, 54)
    else:
        data = synthgen.all_duplicate(n, 52)
    off = synthgen.split_items(data)
    want, _ = U.oracle_results(data, off)
    with make_ctx(engine, batch_bytes=2 << 20) as d:
        got = U.run_device(d, torch.from_numpy(data).to(cuda), off, 2 << 20)
    U.assert_same(got, want)
    if kind in ("all_zero", "hit"):
        assert all(np.all(np.diff(g.chunk_start) == 32) for g in got)
    if kind == "no_hit":
        assert all(g.n_chunks == 1 for g in got)


@pytest.mark.parametrize("engine", ENGINES)
def test_table_chain_orders_batches(cuda, engine):
    """Batch 0 = one 1 MiB no-anchor item (a long sequential SHA-1 chain) +
    small item B; batch 1 = a copy of B, submitted right behind it.  Batch 1's
    lookup must wait for batch 0's inserts: B' is a duplicate of B."""
    long_item = A.constructed_no_hit(1 << 20, 77)
    b = np.random.default_rng(8).integers(0, 256, 100, dtype=np.uint8)
    d0 = torch.from_numpy(np.concatenate([long_item, b, np.zeros(12, np.uint8)])).to(cuda)
    d1 = torch.from_numpy(np.concatenate([b, np.zeros(12, np.uint8)])).to(cuda)
    with make_ctx(engine, batch_bytes=2 << 20, slots=4) as d:
        for rep in range(4):
            s0 = d.submit_device(d0, np.array([0, 1 << 20, (1 << 20) + 100], np.uint64))
            d.submit_device(d1, np.array([0, 100], np.uint64))
            got = d.drain_all()
            assert [g.seq for g in got] == [s0, s0 + 1, s0 + 2]
            assert got[2].is_dup[0] == 1 and int(got[2].first_id[0]) == ((s0 + 1) << 32)
            assert got[0].n_chunks == 1 and got[0].is_dup[0] == 0
            d.end_stream()


@pytest.mark.parametrize("engine", ENGINES)
def test_end_stream_fresh_table(cuda, engine):
    data = U.stream(6 << 20, seed=31, dup_frac=0.6)
    off = synthgen.split_items(data)
    with make_ctx(engine, batch_bytes=2 << 20) as d:
        dev = torch.from_numpy(data).to(cuda)
        got1 = U.run_device(d, dev, off, 2 << 20)
        d.end_stream()
        got2 = U.run_device(d, dev, off, 2 << 20)
        d.end_stream()
        got3 = U.run_device(d, dev, off, 2 << 20)
    want1, _ = U.oracle_results(data, off)
    U.assert_same(got1, want1)
    for g in (got2, got3):
        want, _ = U.oracle_results(data, off, first_seq=g[0].seq)
        U.assert_same(g, want)


@pytest.mark.parametrize("engine", ENGINES)
def test_full_size_c2_bench_config(cuda, engine):
    """BASELINE configs[1] (184 MiB) in the launch configuration bench.py
    times: full bit-exact comparison with the oracle (~3 s of CPU)."""
    import bench
    data = synthgen.config_stream("C2")
    off = synthgen.split_items(data)
    want, counts = U.oracle_results(data, off)
    with make_ctx(engine, **bench.engine_kwargs(len(data))) as d:
        got = U.run_device(d, torch.from_numpy(data).to(cuda), off, bench.BATCH_BYTES,
                           bench.BATCH_ITEMS)
    U.assert_same(got, want)


@pytest.mark.parametrize("engine", ENGINES)
def test_pageable_items_bounce_copied(cuda, engine):
    """Pageable host items go through the slot's page-locked bounce buffer, so
    the caller may overwrite them as soon as submit returns (include/dedup.h
    dedup_submit_batch), on every engine."""
    data = U.stream(6 << 20, seed=91, dup_frac=0.5)
    off = synthgen.split_items(data)
    want, _ = U.oracle_results(data, off)
    scratch = data.copy()
    got = []
    with make_ctx(engine, batch_bytes=2 << 20, slots=2) as d:
        for k in range(0, len(off) - 1, 2):
            j = min(k + 2, len(off) - 1)
            items = [scratch[int(off[i]):int(off[i + 1])] for i in range(k, j)]
            while True:
                try:
                    d.submit(items)
                    break
                except Exception as e:
                    if "EAGAIN" not in str(e):
                        raise
                    got.extend(d.drain(wait_ms=-1))
            scratch[int(off[k]):int(off[j])] = 0xA5   # reuse the buffer at once
        got.extend(d.drain_all())
    U.assert_same(got, want)
