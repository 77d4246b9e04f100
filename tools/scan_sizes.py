"""Isolated chunk-stage cost vs batch size via the op API (for ncu launch lists)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synthgen  # noqa: E402
from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup  # noqa: E402

MiB = 1 << 20
sizes = [int(x) for x in os.environ.get("SIZES", "64,256,1024").split(",")]
data = synthgen.make_stream(max(sizes) * MiB, seed=3, dup_frac=0.5)
dev = torch.from_numpy(data).cuda()
d = Dedup(0, batch_bytes=max(sizes) * MiB, batch_items=max(sizes) + 1, slots=1,
          table_capacity=1 << 16, host_fed=False)
for mb in sizes:
    nb = mb * MiB
    off = torch.from_numpy(np.minimum(np.arange(mb + 1, dtype=np.uint64) * MiB, nb).view(np.int64)).cuda()
    cap = nb // 32 + mb + 2
    cut = torch.zeros(cap, dtype=torch.int32, device="cuda")
    n = torch.zeros(1, dtype=torch.int32, device="cuda")
    for rep in range(3):
        d.op_chunk(dev, nb, off, mb, cut, cap, n)
    torch.cuda.synchronize()
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
    ev[0].record()
    for rep in range(5):
        d.op_chunk(dev, nb, off, mb, cut, cap, n)
    ev[1].record()
    torch.cuda.synchronize()
    ms = ev[0].elapsed_time(ev[1]) / 5
    print(f"{mb} MiB: chunk stage {ms * 1e3:.1f} us -> {nb / ms / 1e6:.1f} GB/s, chunks {int(n.item())}",
          flush=True)
