"""The bench's C2 batch-size sweep alone (tools for A/B)."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import synthgen  # noqa: E402

data = synthgen.config_stream("C2")
off = synthgen.split_items(data)
dd = torch.from_numpy(data).cuda()
print(json.dumps(bench.batch_sweep(dd, off, sizes=(1, 4, 16, 32, 64))), flush=True)
