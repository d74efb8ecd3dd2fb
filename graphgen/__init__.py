"""Seeded synthetic-input generator (host side), shared by the oracle and the tests.

Holds none of the method's arithmetic: it only draws COO edge lists (R-MAT over
Philox4x32-10, spec in rmat.c and DESIGN.md) and builds tiny hand-made graphs.
The CUDA product path has its own, independent implementation of the same
generator (csrc/gen.cu); GPU tests check the two are bit-identical.
"""
from __future__ import annotations

import ctypes
import os
from concurrent.futures import ThreadPoolExecutor

import numpy as np

from .configs import CONFIGS, GraphRecipe, recipe  # noqa: F401

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None


def _lib():
    global _LIB
    if _LIB is None:
        import sys
        sys.path.insert(0, os.path.dirname(_HERE))
        from tools.native_build import build_c_shared
        so = build_c_shared([os.path.join(_HERE, "rmat.c")], os.path.join(_HERE, "libgraphgen.so"))
        lib = ctypes.CDLL(so)
        lib.gg_philox4x32_10.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]
        lib.gg_philox4x32_10.restype = None
        lib.gg_rmat_range.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64,
                                      ctypes.c_double, ctypes.c_double, ctypes.c_double,
                                      ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint32,
                                      ctypes.c_uint32, ctypes.c_void_p, ctypes.c_void_p,
                                      ctypes.c_void_p]
        lib.gg_rmat_range.restype = ctypes.c_int
        _LIB = lib
    return _LIB


def philox4x32_10(ctr, key) -> tuple[int, int, int, int]:
    c = np.asarray(ctr, dtype=np.uint32)
    k = np.asarray(key, dtype=np.uint32)
    o = np.zeros(4, dtype=np.uint32)
    _lib().gg_philox4x32_10(c.ctypes.data, k.ctypes.data, o.ctypes.data)
    return tuple(int(x) for x in o)


def rmat(n: int, m: int, a: float, b: float, c: float, seed: int, wseed: int = 0,
         wmin: int = 1, wmax: int = 64, weighted: bool = True, threads: int | None = None):
    """R-MAT COO (src, dst, w or None) as uint32 numpy arrays, edge e at index e."""
    src = np.empty(m, dtype=np.uint32)
    dst = np.empty(m, dtype=np.uint32)
    w = np.empty(m, dtype=np.uint32) if weighted else None
    if m == 0:
        return src, dst, w
    lib = _lib()
    threads = threads or min(os.cpu_count() or 1, 64)
    nchunk = max(1, min(threads * 4, m // 65536 + 1))
    bounds = [m * i // nchunk for i in range(nchunk + 1)]
    wp = w.ctypes.data if w is not None else None

    def work(i):
        return lib.gg_rmat_range(n, bounds[i], bounds[i + 1], a, b, c, seed, wseed, wmin, wmax,
                                 src.ctypes.data, dst.ctypes.data, wp)

    with ThreadPoolExecutor(max_workers=threads) as ex:
        rcs = list(ex.map(work, range(nchunk)))
    if any(rcs):
        raise RuntimeError("graphgen.rmat: invalid arguments or attempt cap exceeded")
    return src, dst, w


def generate(rec: "GraphRecipe", weighted: bool | None = None):
    """COO for a named recipe (see configs.py)."""
    wt = rec.weighted if weighted is None else weighted
    return rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, rec.wmin, rec.wmax, wt)


def random_small(n: int, m: int, seed: int, wmax: int = 64, self_loops: bool = True):
    """Uniform random multigraph for tiny brute-force cases (numpy PCG64)."""
    rng = np.random.default_rng(seed)
    src = rng.integers(0, n, m, dtype=np.uint32) if n else np.zeros(0, np.uint32)
    dst = rng.integers(0, n, m, dtype=np.uint32) if n else np.zeros(0, np.uint32)
    w = rng.integers(1, wmax + 1, m, dtype=np.uint32)
    if not self_loops and m:
        keep = src != dst
        src, dst, w = src[keep], dst[keep], w[keep]
    return src, dst, w
