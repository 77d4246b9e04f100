"""Row NEXT-2 carry-over mode: C2 (184 MiB) fed in pieces of PIECE_MB."""
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synthgen  # noqa: E402
from paper_conf_ipps_rockenbachsgmtd19_b200.stream import CarryChunker  # noqa: E402

data = synthgen.config_stream("C2")
dev = torch.from_numpy(data).cuda()
for mb in (16, 64):
    piece = mb << 20
    cc = CarryChunker(0, max_piece=piece, table_capacity=1 << 18)
    cc.feed(dev[:piece])
    cc.close()
    cc = CarryChunker(0, max_piece=piece, table_capacity=1 << 18)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    n = 0
    for a in range(0, len(data), piece):
        n += len(cc.feed(dev[a:a + piece], final=a + piece >= len(data)).offset)
    torch.cuda.synchronize()
    dt = time.perf_counter() - t0
    cc.close()
    print(f"pieces of {mb} MiB: {len(data) / dt / 1e9:.1f} GB/s, {n} chunks", flush=True)
