"""GPU parity of the multi-GPU routing (rows A5-A8) on ONE GPU: G logical
ranks, each a ctx owning one digest-table shard (owner_rank r of G), run the
real route / owner / scatter kernels; the all-to-all is replaced by
in-process tensor copies (dist.loopback_all_to_all).  Results must equal the
sequential oracle bit for bit, for any G (grouping invariance)."""
import numpy as np
import pytest

import oracle
import synthgen
from tests import gpu_util as U

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

MiB = 1 << 20


@pytest.mark.parametrize("G", [1, 2, 4])
def test_loopback_routing_matches_oracle(G):
    assert torch.cuda.is_available()
    from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup
    from paper_conf_ipps_rockenbachsgmtd19_b200 import dist as D
    data = U.stream(10 * MiB, seed=41 + G, dup_frac=0.6)
    off = synthgen.split_items(data, MiB // 2)
    n_items = len(off) - 1
    per_batch = 3
    batches = [(k, min(k + per_batch, n_items)) for k in range(0, n_items, per_batch)]
    dev = torch.from_numpy(data).cuda()
    cuda = torch.device("cuda", 0)
    bbytes = per_batch * MiB // 2
    ctxs = [Dedup(0, batch_bytes=bbytes, batch_items=per_batch + 1, slots=1,
                  table_capacity=1 << 16, host_fed=False, owner_rank=r, num_owners=G)
            for r in range(G)]
    try:
        states = [D.RankState(c, bbytes, per_batch + 1, cuda, G) for c in ctxs]
        got = []
        for w in range(0, len(batches), G):
            work = []
            for r in range(G):
                b = w + r
                if b < len(batches):
                    k, j = batches[b]
                    work.append((dev[int(off[k]):int(off[j])], off[k:j + 1] - off[k], k))
                else:
                    work.append((dev[:0], np.zeros(1, np.uint64), n_items))
            for res in D.loopback_waves(states, work):
                got.extend(res.items())
        torch.cuda.synchronize()
    finally:
        for c in ctxs:
            c.close()
    got.sort(key=lambda r: r[0])
    want, _ = oracle.dedup_items([data[int(off[k]):int(off[k + 1])] for k in range(n_items)])
    assert [g[0] for g in got] == [w.seq for w in want]
    for (seq, cs, dg, dup, fid), w in zip(got, want):
        assert np.array_equal(cs, w.chunk_start), seq
        assert np.array_equal(dg, w.digest), seq
        assert np.array_equal(dup, w.is_dup), seq
        assert np.array_equal(fid, w.first_id), seq


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
