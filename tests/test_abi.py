"""CPU checks of the C ABI boundary: the library loads, exports every symbol
include/dedup.h declares, and validates configs before touching the GPU."""
import ctypes
import os
import re

import pytest

from paper_conf_ipps_rockenbachsgmtd19_b200 import _native as N
from paper_conf_ipps_rockenbachsgmtd19_b200 import build as B

HDR = os.path.join(os.path.dirname(os.path.dirname(__file__)), "include", "dedup.h")


@pytest.fixture(scope="module")
def L():
    B.build()
    return N.lib()


def declared():
    src = open(HDR).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(dedup_[a-z_0-9]+)\s*\(", src)))


def test_header_symbols_exported(L):
    names = declared()
    assert len(names) >= 20
    assert set(names) == set(N.EXPORTS)
    for n in names:
        assert hasattr(L, n), n


def test_mandel_header_symbols_exported(L):
    src = open(os.path.join(os.path.dirname(HDR), "mandel.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = sorted(set(re.findall(r"\b(mandel_[a-z_0-9]+)\s*\(", src)))
    assert set(names) == set(N.MANDEL_EXPORTS)
    for n in names:
        assert hasattr(L, n), n


def test_mandel_validates_before_the_gpu(L):
    c = N.MandelConfig(0, 100, -2.0, -1.5, 3.0, 32, 2, 1, None)
    assert L.mandel_image(ctypes.byref(c), None, None, None) == N.DEDUP_EINVAL
    buf = (ctypes.c_uint8 * 16)()
    for dim, niter, spaces in ((0, 100, 2), (4, 0, 2), (4, 1 << 24, 2), (4, 100, 0)):
        c = N.MandelConfig(dim, niter, -2.0, -1.5, 3.0, 32, spaces, 1, None)
        assert L.mandel_image(ctypes.byref(c), buf, None, None) == N.DEDUP_EINVAL
    assert L.mandel_rows_device(None, 10, 100, -2.0, -1.5, 3.0, 5, 6, None, None, None) == \
        N.DEDUP_EINVAL


def test_sm100a_only_cubin():
    B.build()
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", B.LIB],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_struct_layouts_match_header(L):
    # sizes that the header fixes (the C side checks struct_size)
    assert ctypes.sizeof(N.Config) == 96  # 10 u32, 2 u64, 4 u32, 6 reserved u32
    assert ctypes.sizeof(N.Record) == 32
    c = N.Config()
    L.dedup_config_default(ctypes.byref(c))
    assert c.struct_size == ctypes.sizeof(N.Config)
    assert (c.window, c.poly, c.anchor_mask, c.anchor_value, c.min_chunk, c.max_chunk) == \
        (32, 0x45C2B6A1, 0xFFF, 0, 32, 0)


@pytest.mark.parametrize("fields,status", [
    (dict(window=48, min_chunk=48), N.DEDUP_EUNSUPPORTED),
    (dict(max_chunk=48), N.DEDUP_EUNSUPPORTED),
    (dict(max_chunk=16), N.DEDUP_EINVAL),         # max_chunk < min_chunk
    (dict(window=48), N.DEDUP_EINVAL),          # min_chunk < window
    (dict(slots=0), N.DEDUP_EINVAL),
    (dict(batch_bytes=0), N.DEDUP_EINVAL),
    (dict(num_owners=0), N.DEDUP_EINVAL),
    (dict(owner_rank=2, num_owners=2), N.DEDUP_EINVAL),
    (dict(struct_size=4), N.DEDUP_EINVAL),
])
def test_config_validation_without_gpu(L, fields, status):
    c = N.Config()
    L.dedup_config_default(ctypes.byref(c))
    for k, v in fields.items():
        setattr(c, k, v)
    ctx = ctypes.c_void_p()
    assert L.dedup_init(ctypes.byref(c), ctypes.byref(ctx)) == status
    assert not ctx.value


def test_null_args(L):
    assert L.dedup_init(None, None) == N.DEDUP_EINVAL
    assert L.dedup_drain(None, 0, 0, None, None) == N.DEDUP_EINVAL
    L.dedup_destroy(None)
    assert L.dedup_last_error(None) == b"null ctx"


def test_product_does_not_import_oracle():
    pkg = os.path.dirname(N.__file__)
    for root, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cpp", ".h")):
                s = open(os.path.join(root, f)).read()
                assert "oracle" not in re.sub(r"(#|//).*", "", s).replace("oracle.", "x"), f
