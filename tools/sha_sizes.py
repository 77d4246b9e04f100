"""Isolated SHA-1 stage throughput via the op API: uniform 4 KiB chunks (no
tail) and the real chunking of the same data (geometric lengths + tail)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synthgen  # noqa: E402
from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup  # noqa: E402

MiB = 1 << 20
mb = int(os.environ.get("MB", "256"))
cases = os.environ.get("CASES", "uniform,real").split(",")
reps = int(os.environ.get("REPS", "5"))
nb = mb * MiB
data = synthgen.make_stream(nb, seed=3, dup_frac=0.5)
dev = torch.from_numpy(data).cuda()
lane = int(os.environ.get("LANE", "0"))  # SHA-1 bytes per lane (grid size); 0 = default
d = Dedup(0, batch_bytes=nb, batch_items=mb + 1, slots=1, table_capacity=1 << 16, host_fed=False,
          sha_lane_bytes=lane)
cap = nb // 32 + mb + 2
for case in cases:
    cut = torch.zeros(cap, dtype=torch.int32, device="cuda")
    n = torch.zeros(1, dtype=torch.int32, device="cuda")
    if case in ("uniform", "jitter", "capped"):
        rng = np.random.default_rng(1)
        if case == "uniform":
            lens = np.full(nb // 4096 + 1, 4096)
        elif case == "jitter":      # lengths uniform in [2K, 6K): desynchronised switches
            lens = rng.integers(2048, 6144, nb // 2048)
        else:                       # geometric like C2 but no chunk above 12 KiB (no tail)
            lens = np.minimum(32 + rng.geometric(1 / 4096, nb // 1024), 12288)
        c = np.concatenate([[0], np.cumsum(lens)])
        c = c[c < nb]
        cut[:len(c)] = torch.from_numpy(c.astype(np.int32)).cuda()
        n[0] = len(c)
    else:
        off = torch.from_numpy(np.minimum(np.arange(mb + 1, dtype=np.uint64) * MiB, nb).view(np.int64)).cuda()
        d.op_chunk(dev, nb, off, mb, cut, cap, n)
    dig = torch.zeros(cap * 20, dtype=torch.uint8, device="cuda")
    for _ in range(2):
        d.op_sha1(dev, nb, cut, n, cap, dig)
    torch.cuda.synchronize()
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
    ev[0].record()
    for _ in range(reps):
        d.op_sha1(dev, nb, cut, n, cap, dig)
    ev[1].record()
    torch.cuda.synchronize()
    ms = ev[0].elapsed_time(ev[1]) / reps
    k = int(n.item())
    cp = cut[:k].cpu().numpy().astype(np.int64)
    lens = np.diff(np.append(cp, nb))
    print(f"{case} lane={lane}: {mb} MiB, {k} chunks (max {lens.max()} B): sha1 {ms * 1e3:.1f} us -> "
          f"{nb / ms / 1e6:.1f} GB/s", flush=True)
