"""B200-native ECL-MST hot path (Fallin, Gonzalez, Seo, Burtscher, SC'23).

The compute lives in libeclmst.so (hand-written CUDA for sm_100a, C ABI in
include/ecl_mst.h).  This package is its thin Python binding: the functions
carry the C names and only marshal torch tensors / streams.

    from paper_conf_sc_fallingsb23_b200 import ecl_mst_device
    in_mst, total, ws = ecl_mst_device(n, nindex, nlist, eweight)
"""
from ._native import (  # noqa: F401
    EXPORTED,
    EclMstError,
    EclMstOptions,
    EclMstStats,
    default_options,
    ecl_mst,
    ecl_mst_device,
    ecl_mst_dist_device,
    ecl_mst_dist_finalize,
    ecl_mst_dist_init,
    ecl_mst_dist_shard_chunks,
    ecl_mst_dist_unique_id,
    ecl_mst_dist_workspace_bytes,
    ecl_mst_read_stats,
    ecl_mst_read_trace,
    ecl_mst_kernel_times,
    ecl_mst_release_host_cache,
    ecl_mst_workspace_bytes,
    lib_path,
    load,
)

__all__ = [
    "ecl_mst", "ecl_mst_device", "ecl_mst_read_stats", "ecl_mst_read_trace", "ecl_mst_kernel_times", "ecl_mst_workspace_bytes",
    "ecl_mst_release_host_cache", "default_options", "EclMstError", "EclMstOptions",
    "EclMstStats", "load", "lib_path", "EXPORTED", "ecl_mst_dist_device", "ecl_mst_dist_init",
    "ecl_mst_dist_finalize", "ecl_mst_dist_shard_chunks", "ecl_mst_dist_unique_id",
    "ecl_mst_dist_workspace_bytes", "dist",
]
from . import dist  # noqa: E402,F401
