"""Host cost of submit: Python wrapper vs raw ctypes call."""
import ctypes
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup  # noqa: E402
from paper_conf_ipps_rockenbachsgmtd19_b200 import _native as N  # noqa: E402

MiB = 1 << 20
x = torch.zeros(32 * MiB, dtype=torch.uint8, device="cuda")
off = (np.arange(33, dtype=np.uint64) * MiB)
d = Dedup(0, batch_bytes=32 * MiB, batch_items=64, slots=40, table_capacity=1 << 17)
L = N.lib()
torch.cuda.synchronize()
# python wrapper
t0 = time.perf_counter()
for i in range(32):
    d.submit_device(x, off)
t1 = time.perf_counter()
d.drain_all()
# raw ctypes
offp = off.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64))
st = torch.cuda.current_stream().cuda_stream
seq = ctypes.c_uint64()
ptr = x.data_ptr()
t2 = time.perf_counter()
for i in range(32):
    L.dedup_submit_device(d.ctx, ptr, 32 * MiB, off.ctypes.data, 32, st, ctypes.byref(seq))
t3 = time.perf_counter()
d.drain_all()
print(f"python submit {1e6 * (t1 - t0) / 32:.1f} us, raw C submit {1e6 * (t3 - t2) / 32:.1f} us")
s = d.stats()
print(f"per batch: host graph launch {1e3 * s['ms_host_launch'] / s['batches']:.1f} us, "
      f"host parse {1e3 * s['ms_host_parse'] / s['batches']:.1f} us over {s['batches']} batches")
