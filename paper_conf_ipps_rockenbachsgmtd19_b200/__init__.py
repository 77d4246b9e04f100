"""B200-native GPU Dedup hot path (Rockenbach et al., IPDPSW 2019, Sec. IV-B).

Rabin content-defined chunking -> SHA-1 per chunk -> global duplicate check,
as hand-written sm_100a CUDA kernels behind the C ABI of include/dedup.h.
This package is the thin Python binding (argument marshalling only).
"""
import os as _os

# Up to 32 hardware work queues so that the per-slot streams of the engine run
# concurrently; only effective if set before CUDA is initialised.
_os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")

from ._native import DedupError, lib  # noqa: F401
from .api import Dedup, ItemResult, probe_int_rates, result_from_c  # noqa: F401

__all__ = ["Dedup", "DedupError", "ItemResult", "lib", "probe_int_rates", "result_from_c"]
