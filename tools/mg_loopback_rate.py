"""Multi-GPU engine throughput with G logical ranks sharing GPU 0 (loopback),
copy vs p2p transport: the C3 stream, device-resident, PASSES passes as new
dedup streams.  On one GPU this measures the protocol's overhead (kernels,
barriers), not NVLink."""
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import synthgen  # noqa: E402
from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup  # noqa: E402

G = int(os.environ.get("G", "2"))
passes = int(os.environ.get("PASSES", "10"))
data = synthgen.config_stream("C3")
off = synthgen.split_items(data)
dd = torch.from_numpy(data).cuda()
plan = bench.plan_batches(off)
subs = bench.device_subs(dd, off, plan)
for transport in (2, 3):
    with Dedup(0, num_devices=G, device_ids=[0] * G, transport=transport, slots=8,
               batch_bytes=bench.BATCH_BYTES, batch_items=bench.BATCH_ITEMS,
               table_capacity=len(data) // 2048) as d:
        submit = lambda b: d.submit_device(subs[b][0], subs[b][1])  # noqa: E731
        bench.submit_pass(d, submit, len(plan))
        bench.drain_all(d)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(passes):
            bench.submit_pass(d, submit, len(plan))
        bench.drain_all(d)
        torch.cuda.synchronize()
        dt = time.perf_counter() - t0
        print(f"G={G} transport={transport}: {passes * len(data) / dt / 1e9:.1f} GB/s "
              f"(wall clock, {passes} passes of C3)", flush=True)
