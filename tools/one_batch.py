"""Runs a few device-resident batches of the C3 stream (for ncu launch lists
and full captures of the hot kernels)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synthgen  # noqa: E402
from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup  # noqa: E402

MiB = 1 << 20
bmb = int(os.environ.get("BATCH_MB", "64"))
nbat = int(os.environ.get("NBATCH", "3"))
data = synthgen.config_stream(os.environ.get("WORKLOAD", "C3"))
off = synthgen.split_items(data)
dev = torch.from_numpy(data).cuda()
d = Dedup(0, batch_bytes=bmb * MiB, batch_items=max(64, bmb), slots=4, table_capacity=1 << 19)
for b in range(nbat):
    k = (b * bmb) % (len(off) - 1 - bmb)
    d.submit_device(dev[int(off[k]):int(off[k + bmb])], off[k:k + bmb + 1] - off[k])
    d.drain_all()
torch.cuda.synchronize()
print(d.stats())
