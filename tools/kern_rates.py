"""Isolated rates of the two dominant kernels on the C3 stream, as bench.py
measures them (chunk stage: one op_chunk over the stream; SHA-1: STREAMS
contexts launching the same SHA-1 work concurrently), without bench.py's
extra rows.  For A/B runs of library variants (DEDUP_LIB=...)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synthgen  # noqa: E402
from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup  # noqa: E402

streams = int(os.environ.get("STREAMS", "4"))
reps = int(os.environ.get("REPS", "3"))
lane = int(os.environ.get("LANE", "0"))
data = synthgen.config_stream("C3")
off = synthgen.split_items(data)
dd = torch.from_numpy(data).cuda()
nb, n_items = int(off[-1]), len(off) - 1
item_off = torch.from_numpy(off.astype(np.int64)).cuda()
cap = nb // 32 + n_items + 2
ctxs = [Dedup(0, batch_bytes=nb, batch_items=n_items + 1, slots=1, table_capacity=1 << 12,
              host_fed=False, sha_lane_bytes=lane) for _ in range(streams)]
cut = torch.zeros(cap, dtype=torch.int32, device="cuda")
n = torch.zeros(1, dtype=torch.int32, device="cuda")
digs = [torch.zeros(cap * 20, dtype=torch.uint8, device="cuda") for _ in range(streams)]
sts = [torch.cuda.Stream() for _ in range(streams)]
ev = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
for trial in range(2):
    ctxs[0].op_chunk(dd, nb, item_off, n_items, cut, cap, n)
    ctxs[0].op_sha1(dd, nb, cut, n, cap, digs[0])
    torch.cuda.synchronize()
    ev[0].record()
    for _ in range(reps):
        ctxs[0].op_chunk(dd, nb, item_off, n_items, cut, cap, n)
    ev[1].record()
    for k in range(streams):
        sts[k].wait_event(ev[1])
        for _ in range(reps):
            ctxs[k].op_sha1(dd, nb, cut, n, cap, digs[k], stream=sts[k].cuda_stream)
        torch.cuda.current_stream().wait_stream(sts[k])
    ev[2].record()
    ev[2].synchronize()
    chunk_us = ev[0].elapsed_time(ev[1]) * 1e3 / reps
    sha_us = ev[1].elapsed_time(ev[2]) * 1e3 / (reps * streams)
    print(f"[{os.environ.get('DEDUP_LIB', 'default')}] chunk stage {nb / chunk_us / 1e3:.1f} GB/s, "
          f"sha1 ({streams} streams) {nb / sha_us / 1e3:.1f} GB/s", flush=True)
