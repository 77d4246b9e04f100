"""Diagnostics: host cost of the C ABI calls and isolated batch latency."""
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synthgen  # noqa: E402
from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup  # noqa: E402

MiB = 1 << 20
data = synthgen.config_stream("C2")
off = synthgen.split_items(data)
dev = torch.from_numpy(data).cuda()
for bmb in (8, 32, 64):
    nb = bmb
    sub_off = off[:nb + 1].copy()
    d = Dedup(0, batch_bytes=bmb * MiB, batch_items=max(64, bmb), slots=32,
              table_capacity=1 << 17)
    x = dev[:bmb * MiB]
    # isolated latency
    lat = []
    for i in range(8):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        d.submit_device(x, sub_off)
        d.drain_raw(wait_ms=-1)
        lat.append(time.perf_counter() - t0)
        d.end_stream()
    # host submit cost
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for i in range(16):
        d.submit_device(x, sub_off)
    t_sub = (time.perf_counter() - t0) / 16
    t0 = time.perf_counter()
    n = 0
    while d.pending():
        n += d.drain_raw(wait_ms=-1)
    t_drain = time.perf_counter() - t0
    s = d.stats()
    print(f"batch {bmb} MiB: isolated latency med {1e3 * np.median(lat):.3f} ms "
          f"(min {1e3 * min(lat):.3f}); host submit {1e6 * t_sub:.1f} us/batch; "
          f"16 batches drained in {1e3 * t_drain:.2f} ms "
          f"-> {16 * bmb * MiB / (t_drain + 16 * t_sub) / 1e9:.1f} GB/s", flush=True)
    d.close()
