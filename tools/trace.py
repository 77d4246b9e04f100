"""Per-batch event timeline (DEDUP_TRACE=1) of a steady device-resident run."""
import os
import sys

os.environ["DEDUP_TRACE"] = "1"
import torch  # noqa: E402

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synthgen  # noqa: E402
from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup  # noqa: E402

MiB = 1 << 20
bmb = int(os.environ.get("BATCH_MB", "64"))
slots = int(os.environ.get("SLOTS", "16"))
n = int(os.environ.get("NBATCH", "48"))
data = synthgen.config_stream("C2")
off = synthgen.split_items(data)
dev = torch.from_numpy(data).cuda()
d = Dedup(0, batch_bytes=bmb * MiB, batch_items=max(64, bmb), slots=slots, table_capacity=1 << 17)
nb = (len(off) - 1) // bmb
for b in range(n):
    k = (b % nb) * bmb
    while True:
        try:
            d.submit_device(dev[int(off[k]):int(off[k + bmb])], off[k:k + bmb + 1] - off[k])
            break
        except Exception as e:
            if "EAGAIN" not in str(e):
                raise
            if d.drain_raw(wait_ms=0) == 0:
                d.drain_raw(wait_ms=-1)
d.drain_all()
torch.cuda.synchronize()
