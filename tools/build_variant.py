"""Builds the library with extra -D flags into build/ab/<name>.so for GPU A/B
runs (select with DEDUP_LIB=...).  Usage: build_variant.py NAME -DX=1 ..."""
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockenbachsgmtd19_b200 import build as B  # noqa: E402

name, defs = sys.argv[1], sys.argv[2:]
out = os.path.join(B.ROOT, "build", "ab", name + ".so")
os.makedirs(os.path.dirname(out), exist_ok=True)
subprocess.check_call([B.NVCC, *B.FLAGS, *defs, "-o", out, *B.sources()])
print(out)
