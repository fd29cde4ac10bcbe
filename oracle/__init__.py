"""CPU oracle for the minimum spanning forest -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg and
``--impl reference``) may import this package.  The product path
(paper_conf_sc_fallingsb23_b200) never imports it and shares no code with it.

The arithmetic lives in kruskal.c (plain C, single thread); see its header for
the definition it follows and the PAPER.md passages it cites.  This module only
compiles it with gcc and marshals numpy arrays through ctypes.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "kruskal.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile kruskal.c -> liboracle.so (gcc -O3 -march=native, as P:305)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O3", "-march=native", "-std=c11", "-fPIC", "-shared",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            build()
            lib = ctypes.CDLL(_LIB)
            lib.oracle_kruskal.restype = ctypes.c_int
            lib.oracle_kruskal.argtypes = [ctypes.c_int32, ctypes.c_void_p, ctypes.c_void_p,
                                           ctypes.c_void_p, ctypes.c_void_p,
                                           ctypes.POINTER(ctypes.c_int64),
                                           ctypes.POINTER(ctypes.c_int64)]
            lib.oracle_components.restype = ctypes.c_int64
            lib.oracle_components.argtypes = [ctypes.c_int32, ctypes.c_void_p, ctypes.c_void_p]
            lib.oracle_edge_in_msf.restype = ctypes.c_int
            lib.oracle_edge_in_msf.argtypes = [ctypes.c_int32, ctypes.c_void_p, ctypes.c_void_p,
                                               ctypes.c_void_p, ctypes.c_int64]
            _lib = lib
    return _lib


def kruskal(n, nindex, nlist, eweight):
    """MSF by serial Kruskal over the canonical (u < v) CSR entries.

    Returns (mask uint8[M], total_weight int, forest_edge_count int).
    """
    nindex = np.ascontiguousarray(nindex, dtype=np.int64)
    nlist = np.ascontiguousarray(nlist, dtype=np.int32)
    eweight = np.ascontiguousarray(eweight, dtype=np.int32)
    M = int(nlist.shape[0])
    mask = np.zeros(M, dtype=np.uint8)
    total = ctypes.c_int64(0)
    count = ctypes.c_int64(0)
    rc = _load().oracle_kruskal(int(n), nindex.ctypes.data, nlist.ctypes.data,
                                eweight.ctypes.data, mask.ctypes.data,
                                ctypes.byref(total), ctypes.byref(count))
    if rc != 0:
        raise ValueError(f"oracle_kruskal rejected the input (rc={rc})")
    return mask, int(total.value), int(count.value)


def components(n, nindex, nlist):
    """Number of connected components (one union-find scan of the CSR)."""
    nindex = np.ascontiguousarray(nindex, dtype=np.int64)
    nlist = np.ascontiguousarray(nlist, dtype=np.int32)
    c = _load().oracle_components(int(n), nindex.ctypes.data, nlist.ctypes.data)
    if c < 0:
        raise ValueError("oracle_components rejected the input")
    return int(c)


def edge_in_msf(n, nindex, nlist, eweight, edge_id):
    """Is canonical CSR entry edge_id in the MSF? (cycle-property definition)."""
    nindex = np.ascontiguousarray(nindex, dtype=np.int64)
    nlist = np.ascontiguousarray(nlist, dtype=np.int32)
    eweight = np.ascontiguousarray(eweight, dtype=np.int32)
    r = _load().oracle_edge_in_msf(int(n), nindex.ctypes.data, nlist.ctypes.data, eweight.ctypes.data,
                                   int(edge_id))
    if r < 0:
        raise ValueError(f"entry {edge_id} is not a canonical edge")
    return bool(r)


def kruskal_graph(g):
    """Convenience: run on a synth.Graph (tensors copied to host numpy)."""
    n, nindex, nlist, eweight = g.numpy()
    return kruskal(n, nindex, nlist, eweight)
