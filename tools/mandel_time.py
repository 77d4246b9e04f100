"""Row NEXT-4: streamed Mandelbrot image (2000 x 2000, niter 200,000: the
paper's workload) under several batch / memory-space settings."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockenbachsgmtd19_b200 import mandel as M  # noqa: E402

M.image(200, 1000, 32, 2)  # warm-up
cfgs = [tuple(int(x) for x in c.split("x")) for c in
        os.environ.get("CFGS", "32x2,32x4,128x4,256x4,256x8,400x4,500x2,1000x2,2000x1").split(",")]
for b, s in cfgs:
    img, ms, it = M.image(2000, 200000, b, s)
    print(f"batch_rows {b} spaces {s}: {ms:.2f} ms, {it} iterations, {it / ms / 1e9:.3f} T iter/s",
          flush=True)
