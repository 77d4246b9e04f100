"""Evidence of transfer / compute overlap (the paper's "memory spaces",
P:181-185) without nsys: a host-fed run of the C3 stream through
dedup_submit_batch with DEDUP_TRACE=1 (per-batch CUDA-event timeline on the
device clock: H2D of the items, scan, selection, SHA-1, table, pack into
pinned host memory), then per batch the share of its H2D interval during
which another batch's kernels were running, and the share of the whole run
during which both the copy engine and the SMs were busy.

Run under gpurun:  python tools/overlap_trace.py > gpurun_out/overlap.txt
"""
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r'''
import os, sys
os.environ["DEDUP_TRACE"] = "1"
os.environ["DEDUP_TIME_EVERY"] = "1"
sys.path.insert(0, sys.argv[1])
import numpy as np, torch
import bench, synthgen
from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup
data = synthgen.config_stream("C3")
off = synthgen.split_items(data)
plan = bench.plan_batches(off)
with Dedup(0, **bench.engine_kwargs(len(data))) as d:
    pin = d.host_empty(len(data)); pin[:] = data
    sub = lambda b: d.submit_buffer(pin[int(off[plan[b][0]]):int(off[plan[b][1]])],
                                    off[plan[b][0]:plan[b][1] + 1] - off[plan[b][0]])
    for p in range(3):
        bench.submit_pass(d, sub, len(plan))
    bench.drain_all(d)
    torch.cuda.synchronize()
'''


def union(iv):
    iv = sorted(iv)
    out = []
    for a, b in iv:
        if out and a <= out[-1][1]:
            out[-1][1] = max(out[-1][1], b)
        else:
            out.append([a, b])
    return out


def overlap(a, b, segs):
    return sum(max(0.0, min(b, y) - max(a, x)) for x, y in segs)


def main():
    r = subprocess.run([sys.executable, "-c", CHILD, ROOT], capture_output=True, text=True)
    rows = []
    for line in r.stderr.splitlines():
        if not line.startswith("trace "):
            continue
        kv = dict(re.findall(r"(\w+)=([0-9.]+)", line))
        rows.append({k: float(v) for k, v in kv.items()})
    if not rows:
        print(r.stderr[-3000:])
        sys.exit(1)
    h2d = [(x["host"], x["start"]) for x in rows]
    comp = [(x["h2d"], x["table"]) for x in rows]     # scan .. table (kernels)
    t0 = min(a for a, _ in h2d)
    t1 = max(x["done"] for x in rows)
    per = []
    for i, (a, b) in enumerate(h2d):
        others = union([c for j, c in enumerate(comp) if j != i])
        per.append(overlap(a, b, others) / max(b - a, 1e-9))
    cu, hu = union(comp), union(h2d)
    both = sum(overlap(a, b, cu) for a, b in hu)
    print(f"batches {len(rows)}, run {t1 - t0:.2f} ms on the device clock")
    print(f"H2D busy {sum(b - a for a, b in hu):.2f} ms, kernels busy {sum(b - a for a, b in cu):.2f} ms,"
          f" both at once {both:.2f} ms")
    print(f"per-batch share of its H2D during which other batches' kernels ran: "
          f"median {sorted(per)[len(per) // 2]:.3f}, min {min(per):.3f}")
    print("first batches (ms from the run start): host start h2d scan chunk sha table done")
    for x in rows[:6]:
        print("  seq %6d  " % x["seq"] + " ".join(f"{x[k] - t0:7.2f}" for k in
                                                 ("host", "start", "h2d", "scan", "chunk", "sha",
                                                  "table", "done")))


if __name__ == "__main__":
    main()
