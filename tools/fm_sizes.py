"""Isolated LZSS FindMatch throughput (row NEXT-1) on 64 MiB batches."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synthgen  # noqa: E402
from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup  # noqa: E402

MiB = 1 << 20
mb = int(os.environ.get("MB", "64"))
nb = mb * MiB
reps = 5
d = Dedup(0, batch_bytes=nb, batch_items=mb + 1, slots=1, table_capacity=1 << 12, host_fed=False)
for name, data in [("C2", synthgen.config_stream("C2", nbytes=nb)),
                   ("entropy4", synthgen.make_stream(nb, seed=5, dup_frac=0.5, entropy=4)),
                   ("entropy2", synthgen.make_stream(nb, seed=6, dup_frac=0.5, entropy=2))]:
    dev = torch.from_numpy(np.concatenate([data, np.zeros(16, np.uint8)])).cuda()
    off = torch.from_numpy(synthgen.split_items(data).astype(np.int64)).cuda()
    cap = nb // 32 + mb + 2
    cut = torch.zeros(cap, dtype=torch.int32, device="cuda")
    n = torch.zeros(1, dtype=torch.int32, device="cuda")
    d.op_chunk(dev, nb, off, len(off) - 1, cut, cap, n)
    ln = torch.zeros(nb, dtype=torch.uint8, device="cuda")
    of = torch.zeros(nb, dtype=torch.int16, device="cuda")
    d.op_findmatch(dev, nb, cut, n, cap, ln, of)
    torch.cuda.synchronize()
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
    ev[0].record()
    for _ in range(reps):
        d.op_findmatch(dev, nb, cut, n, cap, ln, of)
    ev[1].record()
    torch.cuda.synchronize()
    ms = ev[0].elapsed_time(ev[1]) / reps
    L = ln.cpu().numpy()
    print(f"{name}: {mb} MiB, {int(n.item())} blocks: findmatch {ms * 1e3:.1f} us -> "
          f"{nb / ms / 1e6:.1f} GB/s; mean len {L.mean():.2f}, len>=3 {np.mean(L >= 3):.3f}",
          flush=True)
