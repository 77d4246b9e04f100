"""ctypes declarations of include/dedup.h (argument marshalling only).

Loads the in-tree ``libdedup_b200.so``.  There is no fallback: if the library
is missing or cannot be loaded, importing this module raises.
"""
from __future__ import annotations

import ctypes
import os

PKG = os.path.dirname(os.path.abspath(__file__))
# DEDUP_LIB selects an alternative build of the same library (kernel-variant
# experiments under tools/); default: the in-tree build.
LIB_PATH = os.environ.get("DEDUP_LIB", os.path.join(PKG, "libdedup_b200.so"))

DEDUP_OK = 0
DEDUP_EINVAL = -1
DEDUP_EAGAIN = -2
DEDUP_ENOMEM = -3
DEDUP_ETABLEFULL = -4
DEDUP_EUNSUPPORTED = -5
DEDUP_ECUDA = -6
DEDUP_ETIMEDOUT = -7
DEDUP_ENCCL = -8

STATUS_NAMES = {0: "OK", -1: "EINVAL", -2: "EAGAIN", -3: "ENOMEM", -4: "ETABLEFULL",
                -5: "EUNSUPPORTED", -6: "ECUDA", -7: "ETIMEDOUT", -8: "ENCCL"}

# every symbol declared in include/dedup.h (checked by tests/test_abi.py)
EXPORTS = [
    "dedup_config_default", "dedup_init", "dedup_destroy", "dedup_last_error",
    "dedup_submit_batch", "dedup_submit_device", "dedup_join", "dedup_end_stream", "dedup_drain",
    "dedup_pending", "dedup_next_device", "dedup_stats", "dedup_host_alloc", "dedup_host_free",
    "dedup_op_chunk", "dedup_op_chunk_meta", "dedup_op_sha1", "dedup_op_table_insert_lookup",
    "dedup_op_table_reset", "dedup_op_table_status", "dedup_op_local_combine",
    "dedup_op_route", "dedup_op_owner",
    "dedup_op_scatter", "dedup_op_findmatch", "dedup_kernel_launches",
    "dedup_archive_encode", "dedup_archive_decoder_new", "dedup_archive_decoder_free",
    "dedup_archive_decode",
    "dedup_nccl_unique_id", "dedup_dist_create", "dedup_dist_destroy", "dedup_dist_last_error",
    "dedup_dist_submit", "dedup_dist_flush", "dedup_dist_join", "dedup_dist_end_stream",
    "dedup_dist_result", "dedup_dist_kernel_launches", "dedup_dist_a2a_bytes",
    "dedup_dist_last_counts", "dedup_probe_int_rates",
]
# every symbol declared in include/mandel.h (row NEXT-4)
MANDEL_EXPORTS = ["mandel_rows_device", "mandel_image"]


class WaveResult(ctypes.Structure):
    _fields_ = [
        ("first_seq", ctypes.c_uint64), ("n_items", ctypes.c_uint32),
        ("n_chunks", ctypes.c_uint32),
        ("item_off", ctypes.POINTER(ctypes.c_uint64)),
        ("item_first_chunk", ctypes.POINTER(ctypes.c_uint32)),
        ("chunk_start", ctypes.POINTER(ctypes.c_uint32)),
        ("digest", ctypes.POINTER(ctypes.c_uint8)),
        ("first_id", ctypes.POINTER(ctypes.c_uint64)),
        ("is_dup", ctypes.POINTER(ctypes.c_uint8)),
    ]


class MandelConfig(ctypes.Structure):
    _fields_ = [
        ("dim", ctypes.c_int32), ("niter", ctypes.c_int32),
        ("init_a", ctypes.c_double), ("init_b", ctypes.c_double), ("range", ctypes.c_double),
        ("batch_rows", ctypes.c_uint32), ("spaces", ctypes.c_uint32),
        ("num_devices", ctypes.c_uint32), ("device_ids", ctypes.POINTER(ctypes.c_int32)),
    ]


class Config(ctypes.Structure):
    _fields_ = [
        ("struct_size", ctypes.c_uint32), ("window", ctypes.c_uint32),
        ("poly", ctypes.c_uint32), ("anchor_mask", ctypes.c_uint32),
        ("anchor_value", ctypes.c_uint32), ("min_chunk", ctypes.c_uint32),
        ("max_chunk", ctypes.c_uint32), ("device", ctypes.c_int32),
        ("slots", ctypes.c_uint32), ("batch_items", ctypes.c_uint32),
        ("batch_bytes", ctypes.c_uint64), ("table_capacity", ctypes.c_uint64),
        ("owner_rank", ctypes.c_uint32), ("num_owners", ctypes.c_uint32),
        ("host_fed", ctypes.c_uint32), ("sha_lane_bytes", ctypes.c_uint32),
        ("num_devices", ctypes.c_uint32), ("transport", ctypes.c_uint32),
        ("device_ids", ctypes.POINTER(ctypes.c_int32)), ("carry_over", ctypes.c_uint32),
        ("reserved", ctypes.c_uint32 * 1),
    ]


class ItemResult(ctypes.Structure):
    _fields_ = [
        ("seq", ctypes.c_uint64), ("item_len", ctypes.c_uint64),
        ("n_chunks", ctypes.c_uint32), ("carried", ctypes.c_uint32),
        ("chunk_start", ctypes.POINTER(ctypes.c_uint32)),
        ("digest", ctypes.POINTER(ctypes.c_uint8)),
        ("is_dup", ctypes.POINTER(ctypes.c_uint8)),
        ("first_id", ctypes.POINTER(ctypes.c_uint64)),
    ]


class Stats(ctypes.Structure):
    _fields_ = [(n, ctypes.c_uint64) for n in (
        "items", "bytes", "chunks", "dup_chunks", "dup_bytes", "unique_chunks",
        "batches", "table_used", "table_slots", "kernel_launches")] + [
        ("num_owners", ctypes.c_uint32), ("owner_rank", ctypes.c_uint32)] + [
        (n, ctypes.c_double) for n in ("ms_h2d", "ms_scan", "ms_select", "ms_sha1", "ms_table",
                                       "ms_d2h", "ms_host_launch", "ms_host_parse")] + [
        ("sha1_blocks", ctypes.c_uint64), ("timed_batches", ctypes.c_uint64),
        ("timed_bytes", ctypes.c_uint64), ("timed_sha1_blocks", ctypes.c_uint64),
        ("waves", ctypes.c_uint64), ("a2a_bytes", ctypes.c_uint64), ("ms_a2a", ctypes.c_double),
        ("num_devices", ctypes.c_uint32), ("reserved_", ctypes.c_uint32)]


class IntRates(ctypes.Structure):
    _fields_ = [(n, ctypes.c_double) for n in (
        "lop3", "shf", "iadd3", "imad", "imad_hi", "prmt", "lea_hi", "mix_lop3_imad")] + [
        ("num_sms", ctypes.c_int32), ("clock_mhz_attr", ctypes.c_int32)]


class Record(ctypes.Structure):
    _fields_ = [("digest", ctypes.c_uint8 * 20), ("pad", ctypes.c_uint32),
                ("id", ctypes.c_uint64)]


_lib = None


def lib():
    """The loaded C library (raises if it is missing: no CPU fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(
            f"{LIB_PATH} is missing: build it with `python -m "
            "paper_conf_ipps_rockenbachsgmtd19_b200.build` (there is no CPU fallback)")
    L = ctypes.CDLL(LIB_PATH)
    vp, u32, u64, i32, st = (ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int32,
                             ctypes.c_int32)
    P = ctypes.POINTER
    sig = {
        "dedup_config_default": (None, [P(Config)]),
        "dedup_init": (st, [P(Config), P(vp)]),
        "dedup_destroy": (None, [vp]),
        "dedup_last_error": (ctypes.c_char_p, [vp]),
        "dedup_submit_batch": (st, [vp, u32, P(vp), P(u64), P(u64)]),
        "dedup_submit_device": (st, [vp, vp, u64, vp, u32, vp, P(u64)]),
        "dedup_join": (st, [vp, vp]),
        "dedup_end_stream": (st, [vp]),
        "dedup_drain": (st, [vp, u32, i32, P(ItemResult), P(u32)]),
        "dedup_pending": (u64, [vp]),
        "dedup_next_device": (i32, [vp]),
        "dedup_stats": (st, [vp, P(Stats)]),
        "dedup_host_alloc": (vp, [vp, ctypes.c_size_t]),
        "dedup_host_free": (None, [vp, vp]),
        "dedup_op_chunk": (st, [vp, vp, vp, u64, vp, u32, vp, u64, vp]),
        "dedup_op_chunk_meta": (st, [vp, vp, vp, u32, vp, vp, u64, u64, vp, vp, vp]),
        "dedup_op_sha1": (st, [vp, vp, vp, u64, vp, vp, u64, vp]),
        "dedup_op_findmatch": (st, [vp, vp, vp, u64, vp, vp, u64, vp, u32, u32, vp, vp]),
        "dedup_op_table_insert_lookup": (st, [vp, vp, vp, vp, vp, u64, vp, vp]),
        "dedup_op_table_reset": (st, [vp, vp]),
        "dedup_op_table_status": (st, [vp, vp, P(u64), P(u64), P(i32)]),
        "dedup_op_local_combine": (st, [vp, vp, vp, vp, u64, vp]),
        "dedup_op_route": (st, [vp, vp, vp, vp, vp, u64, vp, u32, vp, vp, vp]),
        "dedup_op_owner": (st, [vp, vp, vp, u64, vp]),
        "dedup_op_scatter": (st, [vp, vp, vp, vp, vp, vp, vp, u64, vp, vp]),
        "dedup_kernel_launches": (u64, [vp]),
        "dedup_archive_encode": (ctypes.c_int64, [vp, u64, vp, u32, vp, vp, vp, vp, u32, u32,
                                                  vp, u64]),
        "dedup_archive_decoder_new": (vp, [u32]),
        "dedup_archive_decoder_free": (None, [vp]),
        "dedup_archive_decode": (ctypes.c_int64, [vp, vp, u64, vp, u64]),
        "dedup_nccl_unique_id": (st, [vp]),
        "dedup_dist_create": (st, [P(Config), vp, i32, i32, u32, u64, u32, P(vp)]),
        "dedup_dist_destroy": (None, [vp]),
        "dedup_dist_last_error": (ctypes.c_char_p, [vp]),
        "dedup_dist_submit": (st, [vp, vp, u64, vp, u32, u64, vp, P(u32)]),
        "dedup_dist_flush": (st, [vp, P(u32)]),
        "dedup_dist_join": (st, [vp, vp]),
        "dedup_dist_kernel_launches": (u64, [vp]),
        "dedup_dist_a2a_bytes": (u64, [vp]),
        "dedup_dist_end_stream": (st, [vp]),
        "dedup_dist_result": (st, [vp, P(WaveResult)]),
        "dedup_dist_last_counts": (st, [vp, P(u32), P(u32), P(u64)]),
        "dedup_probe_int_rates": (st, [i32, P(IntRates)]),
        "mandel_rows_device": (st, [vp, i32, i32, ctypes.c_double, ctypes.c_double,
                                    ctypes.c_double, i32, i32, vp, vp, vp]),
        "mandel_image": (st, [P(MandelConfig), vp, P(ctypes.c_double), P(u64)]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _lib = L
    return L


class DedupError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS_NAMES.get(status, status)}: {msg}")
        self.status = status


def check(status: int, ctx=None):
    if status != DEDUP_OK:
        msg = lib().dedup_last_error(ctx).decode() if ctx else "invalid argument"
        raise DedupError(status, msg)
