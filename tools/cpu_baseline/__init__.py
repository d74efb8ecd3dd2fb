"""Multi-core CPU baseline (OpenMP pull PageRank, omp_pagerank.c) for bench.py; measurement only."""
import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB = os.path.join(_HERE, "libomp_pr.so")


def omp_pagerank(n, src, dst, iters=20, damping=0.85, threads=0):
    """(ranks float64[n], ms_build, ms_iters) on all host cores (threads <= 0) or `threads`."""
    lib = ctypes.CDLL(LIB)
    lib.omp_pagerank.restype = ctypes.c_int
    lib.omp_pagerank.argtypes = [ctypes.c_uint32, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int,
                                 ctypes.c_double, ctypes.c_int, ctypes.c_void_p, ctypes.POINTER(ctypes.c_double),
                                 ctypes.POINTER(ctypes.c_double)]
    src = np.ascontiguousarray(src, dtype=np.uint32)
    dst = np.ascontiguousarray(dst, dtype=np.uint32)
    x = np.empty(max(n, 1), dtype=np.float64)
    mb, mi = ctypes.c_double(), ctypes.c_double()
    rc = lib.omp_pagerank(n, len(src), src.ctypes.data, dst.ctypes.data, iters, damping, threads, x.ctypes.data,
                          ctypes.byref(mb), ctypes.byref(mi))
    if rc != 0:
        raise MemoryError("omp_pagerank: allocation failed")
    return x[:n], mb.value, mi.value


def omp_bfs(n, src, dst, source=0, threads=0):
    """(levels uint32[n], ms_build, ms_run): level-synchronous OpenMP BFS on all host cores."""
    lib = ctypes.CDLL(LIB)
    lib.omp_bfs.restype = ctypes.c_int
    lib.omp_bfs.argtypes = [ctypes.c_uint32, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint32,
                            ctypes.c_int, ctypes.c_void_p, ctypes.POINTER(ctypes.c_double),
                            ctypes.POINTER(ctypes.c_double)]
    src = np.ascontiguousarray(src, dtype=np.uint32)
    dst = np.ascontiguousarray(dst, dtype=np.uint32)
    lv = np.empty(max(n, 1), dtype=np.uint32)
    mb, mr = ctypes.c_double(), ctypes.c_double()
    if lib.omp_bfs(n, len(src), src.ctypes.data, dst.ctypes.data, source, threads, lv.ctypes.data,
                   ctypes.byref(mb), ctypes.byref(mr)) != 0:
        raise MemoryError("omp_bfs: allocation failed")
    return lv[:n], mb.value, mr.value
