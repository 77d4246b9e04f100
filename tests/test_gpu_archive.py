"""Row NEXT-3 end to end on the GPU: the CUDA engine's chunk starts, digests
and duplicate flags plus the GPU FindMatch matches, encoded by the host
archive writer, must decode to the exact input stream."""
import numpy as np
import pytest

import synthgen

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def test_gpu_pipeline_archive_roundtrip():
    assert torch.cuda.is_available()
    from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup, archive
    MiB = 1 << 20
    data = synthgen.make_stream(6 * MiB, seed=17, dup_frac=0.5, entropy=4, segment=128 * 1024)
    off = synthgen.split_items(data, MiB)
    dec = archive.Decoder()
    out = []
    with Dedup(0, batch_bytes=2 * MiB, batch_items=4, slots=4, table_capacity=1 << 16) as d:
        items = [data[int(off[k]):int(off[k + 1])] for k in range(len(off) - 1)]
        for k in range(0, len(items), 2):         # one 2 MiB batch per submit
            d.submit(items[k:k + 2])
        res = d.drain_all()
    with Dedup(0, batch_bytes=2 * MiB, batch_items=4, slots=1, table_capacity=1 << 10,
               host_fed=False) as fm:
        for lo in range(0, len(res), 2):          # archive batches of 2 items
            rs = res[lo:lo + 2]
            a = int(off[lo])
            b = int(off[lo + len(rs)])
            sub = data[a:b]
            starts = np.concatenate([r.chunk_start.astype(np.int64) + int(off[lo + i]) - a
                                     for i, r in enumerate(rs)]).astype(np.uint32)
            dg = np.concatenate([r.digest for r in rs])
            dups = np.concatenate([r.is_dup for r in rs])
            dv = torch.from_numpy(np.concatenate([sub, np.zeros(16, np.uint8)])).cuda()
            st = torch.from_numpy(starts.astype(np.int32)).cuda()
            nb = torch.tensor([len(starts)], dtype=torch.int32, device="cuda")
            ln = torch.zeros(len(sub), dtype=torch.uint8, device="cuda")
            of = torch.zeros(len(sub), dtype=torch.int16, device="cuda")
            fm.op_findmatch(dv, len(sub), st, nb, len(starts), ln, of, skip=torch.from_numpy(
                dups).cuda())                      # duplicates are not compressed
            torch.cuda.synchronize()
            rec = archive.encode(sub, starts, dg, dups, ln.cpu().numpy(),
                                 of.cpu().numpy().view(np.uint16))
            out.append(dec.decode(rec, len(sub)))
    assert np.array_equal(np.concatenate(out), data)
    assert sum(int(r.is_dup.sum()) for r in res) > 0
