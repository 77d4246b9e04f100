"""Build kernel variants of libdedup_b200.so under build/variants/ (timing A/B only).
usage: python tools/build_variants.py name:-DFOO=1,-DBAR=0 [name2:...]"""
import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockenbachsgmtd19_b200 import build as b  # noqa: E402

os.makedirs("build/variants", exist_ok=True)


def one(spec):
    name, _, defs = spec.partition(":")
    flags = [d for d in defs.split(",") if d]
    out = f"build/variants/libdedup_{name}.so"
    subprocess.check_call([b.NVCC, *b.FLAGS, *flags, "-o", out, *b.sources()])
    return out


with ThreadPoolExecutor(4) as ex:
    for o in ex.map(one, sys.argv[1:]):
        print(o)
