"""Row NEXT-2 max_chunk: isolated chunk stage (op_chunk) on C2 tiled 4x,
max_chunk 0 (32-state machine) vs M (walk per item)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synthgen  # noqa: E402
from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup  # noqa: E402

data = synthgen.config_stream("C2")
off1 = synthgen.split_items(data)
copies = 4
nb1 = len(data)
dd = torch.from_numpy(data).cuda().repeat(copies)
nb = nb1 * copies
offs = np.concatenate([off1[:-1] + k * nb1 for k in range(copies)] + [np.array([nb], off1.dtype)])
io = torch.from_numpy(offs.astype(np.int64)).cuda()
cap = nb // 32 + len(offs) + 2
for M in (0, 65536, 16384, 4096):
    d = Dedup(0, batch_bytes=nb, batch_items=len(offs), slots=1, table_capacity=1 << 10,
              host_fed=False, max_chunk=M)
    cut = torch.zeros(cap, dtype=torch.int32, device="cuda")
    n = torch.zeros(1, dtype=torch.int32, device="cuda")
    d.op_chunk(dd, nb, io, len(offs) - 1, cut, cap, n)
    torch.cuda.synchronize()
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
    ev[0].record()
    for _ in range(3):
        d.op_chunk(dd, nb, io, len(offs) - 1, cut, cap, n)
    ev[1].record()
    torch.cuda.synchronize()
    us = ev[0].elapsed_time(ev[1]) * 1e3 / 3
    print(f"max_chunk {M}: {int(n.item())} chunks, chunk stage {us:.0f} us -> "
          f"{nb / us / 1e3:.0f} GB/s", flush=True)
    d.close()
