"""B200-native Suffix kNN Search under Sakoe-Chiba-banded DTW (SMiLer's Search
Step, Zhou & Tung, SIGMOD'15).

The product is libsmiler.so (C ABI, include/smiler.h) built from csrc/ with
nvcc for sm_100a; `smiler` is its thin ctypes binding.  PyTorch is only used by
callers (bench.py, the multi-GPU driver) for device memory, streams and
process groups.
"""
from .smiler import (Index, KnnOpts, KnnStats, SmilerError, Stream, smiler_stream_create, smiler_stream_free,
                     smiler_stream_step, smiler_abi_version, smiler_dtw,  # noqa: F401
                     smiler_free, smiler_index_build, smiler_index_build_shard, smiler_index_envelope,
                     smiler_knn, smiler_knn_step, smiler_lower_bounds, smiler_lower_bounds_ex, smiler_merge_topk,
                     smiler_predict,
                     LB_KINDS)

__all__ = ["Index", "KnnOpts", "KnnStats", "SmilerError", "Stream", "smiler_stream_create", "smiler_stream_free",
           "smiler_stream_step", "smiler_abi_version", "smiler_dtw", "smiler_free",
           "smiler_index_build", "smiler_index_build_shard", "smiler_index_envelope", "smiler_knn", "smiler_knn_step",
           "smiler_lower_bounds", "smiler_lower_bounds_ex", "smiler_merge_topk", "LB_KINDS",
           "smiler_predict"]
