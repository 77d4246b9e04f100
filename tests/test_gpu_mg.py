"""GPU parity of the multi-GPU engine (csrc/mg.cpp) behind the streaming C ABI:
dedup_init with num_devices = G.  On the one-GPU test box the G logical ranks
share device 0 and exchange through the in-process copy transport (each rank
pulls its records / replies from the other ranks' buffers with the gather
kernel); G = 1 with transport = NCCL runs the NCCL code path through
ncclCommInitAll.  The protocol (waves of one batch per rank, local rows as
one CUDA graph per slot, owner shards by digest prefix, insert-all-then-
lookup per wave, deferred table resets, padded partial waves, results merged
in seq order) is the code bench.py --gpus N runs.  Every output is compared
with the sequential oracle (results identical for any G)."""
import numpy as np
import pytest

import oracle
import synthgen
from tests import gpu_util as U

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

MiB = 1 << 20


def mg(G, depth, batch_bytes=MiB, batch_items=8, host_fed=False, transport=0, **kw):
    from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup
    return Dedup(0, num_devices=G, device_ids=[0] * G, slots=depth, batch_bytes=batch_bytes,
                 batch_items=batch_items, host_fed=host_fed, transport=transport,
                 table_capacity=kw.pop("table_capacity", 1 << 16), **kw)


def ragged_stream(nbytes, seed, dup_frac=0.6):
    """C1-like bytes cut into items of 256 KiB with empty and tiny items
    interleaved (item boundaries are forced cuts)."""
    data = U.stream(nbytes, seed=seed, dup_frac=dup_frac)
    off = list(synthgen.split_items(data, MiB // 4))
    k = len(off) // 3
    off = off[:k] + [off[k]] + [off[k] + 7, off[k] + 40] + off[k + 1:]
    return data, np.array(off, np.uint64)


def oracle_stream(data, off, k0=0, k1=None, first_seq=0):
    k1 = len(off) - 1 if k1 is None else k1
    want, _ = oracle.dedup_items([data[int(off[k]):int(off[k + 1])] for k in range(k0, k1)],
                                 first_seq=first_seq)
    return want


def submit_device_batches(d, dev, off, k0, k1, batch_bytes, batch_items, got):
    for k, j in U.batches(off[k0:k1 + 1] - off[k0], batch_bytes, batch_items):
        a, b = int(off[k0 + k]), int(off[k0 + j])
        chunk = dev[a:b] if a % 16 == 0 else dev[a:b].clone()
        while True:
            try:
                d.submit_device(chunk, off[k0 + k:k0 + j + 1] - off[k0 + k])
                break
            except Exception as e:
                if "EAGAIN" not in str(e):
                    raise
                got.extend(d.drain(wait_ms=-1))


@pytest.mark.parametrize("transport", [2, 3])
@pytest.mark.parametrize("G,depth", [(2, 1), (2, 3), (4, 2), (8, 3), (3, 4)])
def test_mg_loopback_device_matches_oracle(G, depth, transport):
    """Device-resident batches through G ranks: two dedup streams (an
    end_stream between them with waves in flight) then the first stream's
    bytes again (all new again after the reset); every output bit-exact."""
    data, off = ragged_stream(8 * MiB, seed=100 + 7 * G + depth)
    dev = torch.from_numpy(data).cuda()
    n = len(off) - 1
    h = n // 2
    got = []
    with mg(G, depth, transport=transport) as d:
        submit_device_batches(d, dev, off, 0, h, MiB, 8, got)
        d.end_stream()
        submit_device_batches(d, dev, off, h, n, MiB, 8, got)
        d.end_stream()
        submit_device_batches(d, dev, off, 0, h, MiB, 8, got)
        got.extend(d.drain_all())
        st = d.stats()
    want = (oracle_stream(data, off, 0, h) + oracle_stream(data, off, h, n, first_seq=h) +
            oracle_stream(data, off, 0, h, first_seq=n))
    U.assert_same(got, want)
    assert st["num_devices"] == G and st["items"] == len(want)
    assert st["chunks"] == sum(len(w.chunk_start) for w in want)
    assert st["dup_chunks"] == sum(int(w.is_dup.sum()) for w in want)


@pytest.mark.parametrize("G,transport", [(2, 2), (5, 2), (3, 3)])
def test_mg_loopback_host_fed_matches_oracle(G, transport):
    """Host items (dedup_submit_batch, pinned and pageable buffers) through G
    ranks, submissions of several batches per call and drains in between
    (partial waves padded with empty batches)."""
    from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup  # noqa: F401
    data, off = ragged_stream(6 * MiB, seed=200 + G)
    items = U.items_of(data, off)
    got = []
    with mg(G, 3, host_fed=True, transport=transport) as d:
        pin = d.host_empty(len(data))
        pin[:] = data
        k = 0
        step = 5
        while k < len(items):
            j = min(k + step, len(items))
            while True:
                try:
                    if (k // step) % 2:
                        d.submit(items[k:j])                        # pageable
                    else:
                        d.submit_buffer(pin[int(off[k]):int(off[j])], off[k:j + 1] - off[k])
                    break
                except Exception as e:
                    if "EAGAIN" not in str(e):
                        raise
                    got.extend(d.drain(wait_ms=-1))
            if (k // step) % 3 == 2:
                got.extend(d.drain(wait_ms=-1))                       # mid-wave drain
            k = j
        got.extend(d.drain_all())
    U.assert_same(got, oracle_stream(data, off))


@pytest.mark.parametrize("transport", [0, 3])
def test_mg_all_duplicate_sends_one_record_per_digest(transport):
    """C5b-like: every item equal.  The local combine sends one record per
    distinct digest per batch; a2a bytes count what left each rank."""
    item = U.stream(MiB // 2, seed=77, dup_frac=0.0)
    data = np.tile(item, 12)
    off = synthgen.split_items(data, MiB // 2)
    dev = torch.from_numpy(data).cuda()
    G = 4
    got = []
    with mg(G, 2, batch_bytes=MiB, batch_items=2, transport=transport) as d:
        submit_device_batches(d, dev, off, 0, len(off) - 1, MiB, 2, got)
        got.extend(d.drain_all())
        st = d.stats()
    want = oracle_stream(data, off)
    U.assert_same(got, want)
    distinct = len({bytes(x) for x in want[0].digest})
    batches = (len(off) - 1) // 2
    # records that left their rank: at most one per distinct digest per batch
    assert st["a2a_bytes"] <= batches * distinct * 40
    assert st["a2a_bytes"] > 0


@pytest.mark.parametrize("nccl_self", [False, True])
def test_mg_nccl_world1_matches_oracle(nccl_self, monkeypatch):
    """transport = NCCL with one rank (ncclCommInitAll on device 0): the NCCL
    code path of the engine end to end.  The rank's own share of the
    exchange is a device copy; with DEDUP_MG_NCCL_SELF it goes through NCCL
    send/recv to itself (counts on their own communicator, grouped send/recv
    of records and replies)."""
    if nccl_self:
        monkeypatch.setenv("DEDUP_MG_NCCL_SELF", "1")
    else:
        monkeypatch.delenv("DEDUP_MG_NCCL_SELF", raising=False)
    data, off = ragged_stream(6 * MiB, seed=303)
    dev = torch.from_numpy(data).cuda()
    n = len(off) - 1
    got = []
    with mg(1, 3, transport=1) as d:
        submit_device_batches(d, dev, off, 0, n // 2, MiB, 8, got)
        d.end_stream()
        submit_device_batches(d, dev, off, n // 2, n, MiB, 8, got)
        got.extend(d.drain_all())
    U.assert_same(got, oracle_stream(data, off, 0, n // 2) +
                  oracle_stream(data, off, n // 2, n, first_seq=n // 2))


def test_mg_join_brackets_all_work():
    """dedup_join makes a stream wait for every submitted batch (padding the
    partial wave): after join + synchronize every item is drainable at once."""
    data, off = ragged_stream(3 * MiB, seed=404)
    dev = torch.from_numpy(data).cuda()
    got = []
    with mg(3, 4) as d:
        submit_device_batches(d, dev, off, 0, len(off) - 1, MiB, 8, got)
        d.join()
        torch.cuda.synchronize()
        got.extend(d.drain(wait_ms=0))
        assert d.pending() == 0
    U.assert_same(got, oracle_stream(data, off))


@pytest.mark.parametrize("transport", [2, 3])
def test_mg_table_overflow_is_sticky(transport):
    """A full shard is DEDUP_ETABLEFULL (sticky), never wrong dup flags."""
    from paper_conf_ipps_rockenbachsgmtd19_b200._native import DedupError
    data = U.stream(48 * MiB, seed=505, dup_frac=0.0)      # ~12 k distinct chunks
    off = synthgen.split_items(data, MiB // 2)
    dev = torch.from_numpy(data).cuda()
    with mg(2, 2, table_capacity=16, transport=transport) as d:  # 2 shards of 4096 slots
        with pytest.raises(DedupError, match="ETABLEFULL"):
            got = []
            submit_device_batches(d, dev, off, 0, len(off) - 1, MiB, 8, got)
            d.drain_all()
        with pytest.raises(DedupError, match="ETABLEFULL"):
            d.drain(wait_ms=0)


def test_mg_rejects_op_layer_and_bad_config():
    from paper_conf_ipps_rockenbachsgmtd19_b200._native import DedupError
    with pytest.raises(DedupError):
        mg(2, 2, owner_rank=1, num_owners=2)
    with pytest.raises(DedupError):
        mg(2, 2, transport=1)           # NCCL needs distinct devices
    with pytest.raises(DedupError):
        mg(2, 2, transport=4)           # no such transport
    with mg(2, 1) as d:
        cut = torch.zeros(16, dtype=torch.int32, device="cuda")
        with pytest.raises(DedupError, match="EUNSUPPORTED"):
            d.op_chunk(cut, 0, cut, 0, cut, 16, cut)
        assert d.next_device() == 0
