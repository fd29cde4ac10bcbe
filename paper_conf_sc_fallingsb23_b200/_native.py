"""ctypes binding of libeclmst.so (include/ecl_mst.h) -- argument marshalling only.

Every step of the MSF runs in the library's CUDA kernel; this module only
checks tensor dtypes/devices, passes raw pointers and the current CUDA stream,
and converts status codes into exceptions.  There is no CPU fallback: if the
shared library is missing, importing the package's functions raises.
"""
from __future__ import annotations

import ctypes
import os

import torch

from . import build as _build

MAX_ROUNDS = 128
ABI_VERSION = 3          # include/ecl_mst.h ECL_MST_ABI_VERSION

OK = 0
ERR_INVALID = -1
ERR_TOO_LARGE = -2
ERR_CUDA = -3
ERR_WORKSPACE = -4
ERR_INPUT = -5
ERR_ROUNDS = -6


class EclMstOptions(ctypes.Structure):
    _fields_ = [
        ("filter", ctypes.c_int32),
        ("threshold_mode", ctypes.c_int32),
        ("threshold", ctypes.c_int32),
        ("path_halving", ctypes.c_int32),
        ("atomic_guards", ctypes.c_int32),
        ("flatten", ctypes.c_int32),
        ("max_ctas", ctypes.c_int32),
        ("trace", ctypes.c_int32),
        ("seed", ctypes.c_uint64),
        ("threshold_samples", ctypes.c_int32),
        ("populate_order", ctypes.c_int32),
        ("refilter", ctypes.c_int32),
        ("filter_c", ctypes.c_int32),
        ("giant_bitmap", ctypes.c_int32),
        ("relabel", ctypes.c_int32),
        ("populate_mode", ctypes.c_int32),
        ("both_directions", ctypes.c_int32),
        ("tuple_layout", ctypes.c_int32),
        ("drive", ctypes.c_int32),
        ("dist_loop", ctypes.c_int32),
    ]


class EclMstStats(ctypes.Structure):
    _fields_ = [
        ("status", ctypes.c_int32),
        ("filtered", ctypes.c_int32),
        ("threshold", ctypes.c_int32),
        ("rounds", ctypes.c_int32),
        ("phase2_round", ctypes.c_int32),
        ("grid", ctypes.c_int32),
        ("block", ctypes.c_int32),
        ("refilters", ctypes.c_int32),
        ("relabels", ctypes.c_int32),
        ("reserved", ctypes.c_int32),
        ("total_weight", ctypes.c_int64),
        ("msf_edges", ctypes.c_int64),
        ("canonical_edges", ctypes.c_int64),
        ("heavy_edges", ctypes.c_int64),
        ("live", ctypes.c_int64 * MAX_ROUNDS),
        ("winners", ctypes.c_int64 * MAX_ROUNDS),
        ("t_ns", ctypes.c_int64 * (2 * MAX_ROUNDS + 4)),
    ]


class EclMstError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"ecl_mst error {code}: {msg}")
        self.code = code


_lib = None


def lib_path() -> str:
    # ECLMST_LIB: load an alternative build of the same library (A/B experiments)
    return os.environ.get("ECLMST_LIB", _build.LIB)


def load(build_if_missing: bool = False):
    """Load libeclmst.so.  Raises if it is missing (no fallback path)."""
    global _lib
    if _lib is not None:
        return _lib
    path = lib_path()
    if not os.path.exists(path):
        if not build_if_missing or path != _build.LIB:
            raise ImportError(f"libeclmst.so not built ({path}); run `python -m "
                              f"paper_conf_sc_fallingsb23_b200.build` or __graft_entry__.build()")
        _build.build()
    L = ctypes.CDLL(path)
    vp, i32, i64, sz = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_size_t
    L.ecl_mst_abi_version.restype = ctypes.c_int
    L.ecl_mst_last_error.restype = ctypes.c_char_p
    L.ecl_mst_default_options.argtypes = [ctypes.POINTER(EclMstOptions)]
    L.ecl_mst_workspace_bytes.restype = sz
    L.ecl_mst_workspace_bytes.argtypes = [i64, i64]
    L.ecl_mst_workspace_bytes_ex.restype = sz
    L.ecl_mst_workspace_bytes_ex.argtypes = [i64, i64, ctypes.POINTER(EclMstOptions)]
    L.ecl_mst_device.restype = ctypes.c_int
    L.ecl_mst_device.argtypes = [i32, i64, vp, vp, vp, vp, vp, vp, sz, ctypes.POINTER(EclMstOptions), vp]
    L.ecl_mst_read_stats.restype = ctypes.c_int
    L.ecl_mst_read_stats.argtypes = [vp, ctypes.POINTER(EclMstStats), vp]
    L.ecl_mst.restype = i64
    L.ecl_mst.argtypes = [i32, vp, vp, vp, vp]
    L.ecl_mst_release_host_cache.restype = None
    L.ecl_mst_read_trace.restype = ctypes.c_int
    L.ecl_mst_read_trace.argtypes = [vp, vp, sz, vp]
    L.ecl_mst_kernel_times.restype = ctypes.c_int
    L.ecl_mst_kernel_times.argtypes = [vp, i32]
    L.ecl_mst_dist_unique_id.restype = ctypes.c_int
    L.ecl_mst_dist_unique_id.argtypes = [vp]
    L.ecl_mst_dist_init.restype = ctypes.c_int
    L.ecl_mst_dist_init.argtypes = [vp, i32, i32, ctypes.POINTER(ctypes.c_void_p)]
    L.ecl_mst_dist_finalize.restype = ctypes.c_int
    L.ecl_mst_dist_finalize.argtypes = [vp]
    L.ecl_mst_dist_shard_chunks.restype = i64
    L.ecl_mst_dist_shard_chunks.argtypes = [i64, i32, i32]
    L.ecl_mst_dist_workspace_bytes.restype = sz
    L.ecl_mst_dist_workspace_bytes.argtypes = [i64, i64, i32, i32]
    L.ecl_mst_dist_device.restype = ctypes.c_int
    L.ecl_mst_dist_device.argtypes = [vp, i32, i32, i64, vp, vp, vp, vp, vp, vp, sz,
                                      ctypes.POINTER(EclMstOptions), vp]
    if L.ecl_mst_abi_version() != ABI_VERSION:
        raise ImportError("libeclmst.so ABI version mismatch")
    _lib = L
    return L


EXPORTED = ["ecl_mst_abi_version", "ecl_mst_last_error", "ecl_mst_default_options",
            "ecl_mst_workspace_bytes", "ecl_mst_workspace_bytes_ex", "ecl_mst_device", "ecl_mst_read_stats", "ecl_mst",
            "ecl_mst_release_host_cache", "ecl_mst_read_trace", "ecl_mst_kernel_times",
            "ecl_mst_dist_unique_id", "ecl_mst_dist_init", "ecl_mst_dist_finalize",
            "ecl_mst_dist_shard_chunks", "ecl_mst_dist_workspace_bytes", "ecl_mst_dist_device"]


def _err(code):
    msg = load().ecl_mst_last_error().decode(errors="replace")
    raise EclMstError(code, msg)


def default_options(**kw) -> EclMstOptions:
    o = EclMstOptions()
    load().ecl_mst_default_options(ctypes.byref(o))
    for k, v in kw.items():
        if not hasattr(o, k):
            raise KeyError(k)
        setattr(o, k, v)
    return o


def ecl_mst_workspace_bytes(n: int, M: int, options=None) -> int:
    if options is None:
        b = load().ecl_mst_workspace_bytes(int(n), int(M))
    else:
        b = load().ecl_mst_workspace_bytes_ex(int(n), int(M), ctypes.byref(options))
    if b == 0:
        raise EclMstError(ERR_TOO_LARGE, f"graph too large (n={n}, M={M})")
    return int(b)


def _check(t, dtype, name, device=None):
    if not isinstance(t, torch.Tensor):
        raise TypeError(f"{name} must be a torch.Tensor")
    if t.dtype != dtype:
        raise TypeError(f"{name} must be {dtype}, got {t.dtype}")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")
    if device is not None and t.device != device:
        raise ValueError(f"{name} must live on {device}, got {t.device}")


def _stream_ptr(stream):
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


def ecl_mst_device(n, nindex, nlist, eweight, in_mst_out=None, total_weight_out=None,
                   workspace=None, options=None, stream=None):
    """Run the MSF hot path on device tensors (async on `stream`).

    Returns (in_mst uint8[M], total_weight int64[1], workspace uint8[...]).
    """
    dev = nlist.device
    if dev.type != "cuda":
        raise ValueError("ecl_mst_device needs CUDA tensors (no CPU fallback)")
    _check(nindex, torch.int64, "nindex", dev)
    _check(nlist, torch.int32, "nlist", dev)
    _check(eweight, torch.int32, "eweight", dev)
    n = int(n)
    M = int(nlist.numel())
    if nindex.numel() != n + 1 or eweight.numel() != M:
        raise ValueError("nindex must have n+1 entries and eweight M entries")
    if in_mst_out is None:
        in_mst_out = torch.empty(M, dtype=torch.uint8, device=dev)
    if total_weight_out is None:
        total_weight_out = torch.empty(1, dtype=torch.int64, device=dev)
    _check(in_mst_out, torch.uint8, "in_mst_out", dev)
    _check(total_weight_out, torch.int64, "total_weight_out", dev)
    if in_mst_out.numel() != M:
        raise ValueError("in_mst_out must have M entries")
    opts = options if options is not None else default_options()
    need = ecl_mst_workspace_bytes(n, M, opts)
    if workspace is None or workspace.numel() < need:
        workspace = torch.empty(need, dtype=torch.uint8, device=dev)
    _check(workspace, torch.uint8, "workspace", dev)
    with torch.cuda.device(dev):
        rc = load().ecl_mst_device(n, M, nindex.data_ptr(), nlist.data_ptr(), eweight.data_ptr(),
                                   in_mst_out.data_ptr(), total_weight_out.data_ptr(),
                                   workspace.data_ptr(), workspace.numel(), ctypes.byref(opts),
                                   _stream_ptr(stream))
    if rc != OK:
        _err(rc)
    return in_mst_out, total_weight_out, workspace


def ecl_mst_read_stats(workspace, stream=None) -> dict:
    """Synchronise and return the statistics of the last run on `workspace`."""
    st = EclMstStats()
    with torch.cuda.device(workspace.device):
        rc = load().ecl_mst_read_stats(workspace.data_ptr(), ctypes.byref(st), _stream_ptr(stream))
    if rc != OK:
        _err(rc)
    R = max(int(st.rounds), 0)
    return {
        "status": st.status, "filtered": bool(st.filtered), "threshold": st.threshold,
        "rounds": st.rounds, "phase2_round": st.phase2_round, "grid": st.grid, "block": st.block,
        "refilters": st.refilters, "relabels": st.relabels,
        "total_weight": st.total_weight, "msf_edges": st.msf_edges,
        "canonical_edges": st.canonical_edges, "heavy_edges": st.heavy_edges,
        "live": list(st.live[:R]), "winners": list(st.winners[:R]),
        "t_ns": list(st.t_ns[: 2 * R + 4]),
    }


TRACE_CTAS = 4096


def ecl_mst_read_trace(workspace, stats, stream=None):
    """Per-CTA stage end times of the last traced run: int64 [slots, grid] (ns)."""
    slots = 2 * MAX_ROUNDS + 4
    out = torch.zeros(slots * TRACE_CTAS, dtype=torch.int64)
    with torch.cuda.device(workspace.device):
        rc = load().ecl_mst_read_trace(workspace.data_ptr(), out.data_ptr(), out.numel(), _stream_ptr(stream))
    if rc != OK:
        _err(rc)
    return out.view(slots, TRACE_CTAS)[:, : stats["grid"]]


# ---- edge-sharded multi-GPU path ----

def ecl_mst_dist_unique_id() -> bytes:
    """128-byte NCCL unique id (create on one rank, broadcast to the others)."""
    buf = ctypes.create_string_buffer(128)
    rc = load().ecl_mst_dist_unique_id(buf)
    if rc != OK:
        _err(rc)
    return buf.raw


def ecl_mst_dist_init(uid, rank: int, world: int):
    """Handle for ecl_mst_dist_device (uid None: world 1 without NCCL)."""
    h = ctypes.c_void_p()
    ubuf = ctypes.create_string_buffer(bytes(uid), 128) if uid is not None else None
    rc = load().ecl_mst_dist_init(ubuf, int(rank), int(world), ctypes.byref(h))
    if rc != OK:
        _err(rc)
    return h


def ecl_mst_dist_finalize(handle):
    load().ecl_mst_dist_finalize(handle)


def ecl_mst_dist_shard_chunks(M: int, shard: int, nshards: int) -> int:
    return int(load().ecl_mst_dist_shard_chunks(int(M), int(shard), int(nshards)))


def ecl_mst_dist_workspace_bytes(n: int, M: int, local_shards: int = 1, world: int = 1) -> int:
    b = load().ecl_mst_dist_workspace_bytes(int(n), int(M), int(local_shards), int(world))
    if b == 0:
        raise EclMstError(ERR_TOO_LARGE, f"graph too large (n={n}, M={M})")
    return int(b)


def ecl_mst_dist_device(handle, n, nindex, nlist, eweight, local_shards=1, world=1, in_mst_out=None,
                        total_weight_out=None, workspace=None, options=None, stream=None):
    """Sharded hot path on this rank's GPU (full replicated CSR in, full mask out)."""
    dev = nlist.device
    if dev.type != "cuda":
        raise ValueError("ecl_mst_dist_device needs CUDA tensors (no CPU fallback)")
    _check(nindex, torch.int64, "nindex", dev)
    _check(nlist, torch.int32, "nlist", dev)
    _check(eweight, torch.int32, "eweight", dev)
    n = int(n)
    M = int(nlist.numel())
    if nindex.numel() != n + 1 or eweight.numel() != M:
        raise ValueError("nindex must have n+1 entries and eweight M entries")
    if in_mst_out is None:
        in_mst_out = torch.empty(M, dtype=torch.uint8, device=dev)
    if total_weight_out is None:
        total_weight_out = torch.empty(1, dtype=torch.int64, device=dev)
    _check(in_mst_out, torch.uint8, "in_mst_out", dev)
    _check(total_weight_out, torch.int64, "total_weight_out", dev)
    if in_mst_out.numel() != M or total_weight_out.numel() < 1:
        raise ValueError("in_mst_out must have M entries and total_weight_out at least one")
    need = ecl_mst_dist_workspace_bytes(n, M, local_shards, world)
    if workspace is None or workspace.numel() < need:
        workspace = torch.empty(need, dtype=torch.uint8, device=dev)
    _check(workspace, torch.uint8, "workspace", dev)
    opts = options if options is not None else default_options()
    with torch.cuda.device(dev):
        rc = load().ecl_mst_dist_device(handle, int(local_shards), n, M, nindex.data_ptr(), nlist.data_ptr(),
                                        eweight.data_ptr(), in_mst_out.data_ptr(), total_weight_out.data_ptr(),
                                        workspace.data_ptr(), workspace.numel(), ctypes.byref(opts),
                                        _stream_ptr(stream))
    if rc != OK:
        _err(rc)
    return in_mst_out, total_weight_out, workspace


KERNEL_STAGES = ["init", "populate1", "rounds1", "flatten", "populate2", "rounds2", "finalize"]


def ecl_mst_kernel_times():
    """Per-stage device times (ms) of the last call made with options.trace & 2."""
    out = (ctypes.c_float * len(KERNEL_STAGES))()
    rc = load().ecl_mst_kernel_times(out, len(KERNEL_STAGES))
    if rc < 0:
        _err(rc)
    return dict(zip(KERNEL_STAGES, list(out)[:rc]))


def ecl_mst(n, nindex, nlist, eweight, in_mst_out):
    """Host-pointer convenience call ("memcpy" variant): CPU tensors in,
    in_mst_out (CPU uint8[M]) filled, total weight returned."""
    for t, dt, nm in ((nindex, torch.int64, "nindex"), (nlist, torch.int32, "nlist"),
                      (eweight, torch.int32, "eweight"), (in_mst_out, torch.uint8, "in_mst_out")):
        _check(t, dt, nm)
        if t.device.type != "cpu":
            raise ValueError(f"{nm} must be a host tensor")
    # the library reads nindex[n] and then M = nindex[n] entries of every
    # array from these host pointers: check the sizes here, before it does
    n = int(n)
    if n < 0 or nindex.numel() != n + 1:
        raise ValueError("nindex must have n+1 entries")
    M = int(nindex[-1]) if n > 0 else 0
    if M < 0 or M > nlist.numel() or nlist.numel() != eweight.numel() or in_mst_out.numel() < M:
        raise ValueError(f"nindex[n] = {M} must satisfy 0 <= M <= nlist.numel() == eweight.numel() "
                         f"<= in_mst_out.numel()")
    total = load().ecl_mst(int(n), nindex.data_ptr(), nlist.data_ptr(), eweight.data_ptr(),
                           in_mst_out.data_ptr())
    if total == -(1 << 63):
        err = load().ecl_mst_last_error().decode(errors="replace")
        code = ERR_INPUT if "inconsistent" in err else ERR_ROUNDS if "round slots" in err else ERR_CUDA
        raise EclMstError(code, err)
    return int(total)


def ecl_mst_release_host_cache():
    load().ecl_mst_release_host_cache()
