"""CPU ORACLE -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / `--impl
reference` legs may import this package.  The product package
(paper_conf_asplos_sabetq018_b200) never imports it and shares no code with it.

ctypes wrapper over oracle/oracle.c (plain single-threaded C; each function
cites the PAPER.md passage it follows).  Pinned by tests/test_oracle.py; see
DESIGN.md "Oracle pins".  Nothing here is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import sys

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None

BFS, SSSP, CC, SSWP, PR = 0, 1, 2, 3, 4
ALGOS = {"bfs": BFS, "sssp": SSSP, "cc": CC, "sswp": SSWP, "pr": PR}
INF = 0xFFFFFFFF

_P = ctypes.c_void_p
_U32, _U64, _I64 = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int64


def _lib():
    global _LIB
    if _LIB is None:
        sys.path.insert(0, os.path.dirname(_HERE))
        from tools.native_build import build_c_shared
        so = build_c_shared([os.path.join(_HERE, "oracle.c")], os.path.join(_HERE, "liboracle.so"))
        lib = ctypes.CDLL(so)
        sig = {
            "or_csr_build": (ctypes.c_int, [_U32, _U64, _P, _P, _P, _P, _P, _P]),
            "or_virtual_count": (_U64, [_U32, _P, _U64, _P]),
            "or_virtual_emit": (None, [_U32, _P, _P]),
            "or_vnode_edges": (_U64, [_P, _P, _P, _U64, _U64, ctypes.c_int, _U64, _P]),
            "or_bfs": (ctypes.c_int, [_U32, _P, _P, _U32, _P]),
            "or_sssp": (ctypes.c_int, [_U32, _P, _P, _P, _U32, _P]),
            "or_sswp": (ctypes.c_int, [_U32, _P, _P, _P, _U32, _P]),
            "or_cc": (ctypes.c_int, [_U32, _U64, _P, _P, _P]),
            "or_pagerank": (ctypes.c_int, [_U32, _P, _P, _U32, ctypes.c_double, ctypes.c_int, _P]),
            "or_udt": (_U64, [_U32, _P, _P, _P, _U64, _U32, _U32, _P, _P, _P, _P]),
            "or_push_virtual": (_I64, [_U32, _P, _P, _P, _P, _P, _U64, ctypes.c_int, _U64,
                                       ctypes.c_int, _U32, ctypes.c_int, ctypes.c_int, _P, _U64, _P]),
        }
        for name, (res, args) in sig.items():
            f = getattr(lib, name)
            f.restype = res
            f.argtypes = args
        _LIB = lib
    return _LIB


def _p(a):
    return None if a is None else a.ctypes.data


def _u32(a):
    return None if a is None else np.ascontiguousarray(a, dtype=np.uint32)


class CSR:
    """Oracle-side CSR (Fig. 10a): row_ptr int64[n+1], col uint32[m], wt uint32[m] or None."""

    def __init__(self, n, row_ptr, col, wt):
        self.n, self.row_ptr, self.col, self.wt = n, row_ptr, col, wt

    @property
    def m(self):
        return int(self.row_ptr[-1]) if self.n else 0

    def degrees(self):
        return np.diff(self.row_ptr)


def symmetrize(src, dst, w=None):
    """c2: append (dst, src, w) for every arc (weak connectivity for CC, L363-365)."""
    s2 = np.concatenate([_u32(src), _u32(dst)])
    d2 = np.concatenate([_u32(dst), _u32(src)])
    w2 = None if w is None else np.concatenate([_u32(w), _u32(w)])
    return s2, d2, w2


def csr_build(n, src, dst, w=None) -> CSR:
    src, dst, w = _u32(src), _u32(dst), _u32(w)
    m = len(src)
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    col = np.empty(m, dtype=np.uint32)
    wt = np.empty(m, dtype=np.uint32) if w is not None else None
    rc = _lib().or_csr_build(n, m, _p(src), _p(dst), _p(w), _p(row_ptr), _p(col), _p(wt))
    if rc:
        raise ValueError(f"or_csr_build failed ({rc})")
    return CSR(n, row_ptr, col, wt)


class Virtual:
    """Virtual node array (Fig. 10b): vnode_ptr uint64[n+1], vn_phys uint32[NV]."""

    def __init__(self, g: CSR, K: int):
        self.g, self.K = g, K
        self.vnode_ptr = np.zeros(g.n + 1, dtype=np.uint64)
        nv = _lib().or_virtual_count(g.n, _p(g.row_ptr), K, _p(self.vnode_ptr))
        self.nv = int(nv)
        self.vn_phys = np.empty(self.nv, dtype=np.uint32)
        _lib().or_virtual_emit(g.n, _p(self.vnode_ptr), _p(self.vn_phys))

    def edges(self, i: int, layout: int, chunk: int = 1) -> np.ndarray:
        """Absolute CSR edge indices owned by vnode i (layout 0 consecutive, 1 strided)."""
        v = int(self.vn_phys[i])
        d = int(self.g.row_ptr[v + 1] - self.g.row_ptr[v])
        out = np.empty(max(d, 1), dtype=np.int64)
        cnt = _lib().or_vnode_edges(_p(self.g.row_ptr), _p(self.vnode_ptr), _p(self.vn_phys),
                                    i, self.K, layout, chunk, _p(out))
        return out[:cnt]


def bfs(g: CSR, source: int) -> np.ndarray:
    out = np.empty(g.n, dtype=np.uint32)
    rc = _lib().or_bfs(g.n, _p(g.row_ptr), _p(g.col), source, _p(out))
    if rc:
        raise ValueError(f"or_bfs failed ({rc})")
    return out


def sssp(g: CSR, source: int) -> np.ndarray:
    out = np.empty(g.n, dtype=np.uint32)
    rc = _lib().or_sssp(g.n, _p(g.row_ptr), _p(g.col), _p(g.wt), source, _p(out))
    if rc:
        raise ValueError(f"or_sssp failed ({rc})")
    return out


def sswp(g: CSR, source: int) -> np.ndarray:
    out = np.empty(g.n, dtype=np.uint32)
    rc = _lib().or_sswp(g.n, _p(g.row_ptr), _p(g.col), _p(g.wt), source, _p(out))
    if rc:
        raise ValueError(f"or_sswp failed ({rc})")
    return out


def cc(n: int, src, dst) -> np.ndarray:
    src, dst = _u32(src), _u32(dst)
    out = np.empty(n, dtype=np.uint32)
    rc = _lib().or_cc(n, len(src), _p(src), _p(dst), _p(out))
    if rc:
        raise ValueError(f"or_cc failed ({rc})")
    return out


def pagerank(g: CSR, iters: int = 20, damping: float = 0.85, dangling: int = 0) -> np.ndarray:
    out = np.empty(g.n, dtype=np.float64)
    rc = _lib().or_pagerank(g.n, _p(g.row_ptr), _p(g.col), iters, damping, dangling, _p(out))
    if rc:
        raise ValueError(f"or_pagerank failed ({rc})")
    return out


def push_virtual(g: CSR, vg: Virtual, algo: int, source: int = 0, layout: int = 1, chunk: int = 1,
                 schedule: int = 1, worklist: int = 1, max_iters: int = 1 << 30):
    """Paper-literal Alg. 2/3 on the virtual graph, sequential.

    Returns (values, iterations, converged); stops after max_iters iterations."""
    out = np.empty(g.n, dtype=np.uint32)
    conv = ctypes.c_int(0)
    it = _lib().or_push_virtual(g.n, _p(g.row_ptr), _p(g.col), _p(g.wt), _p(vg.vnode_ptr),
                                _p(vg.vn_phys), vg.K, layout, chunk, algo, source, schedule,
                                worklist, _p(out), max_iters, ctypes.byref(conv))
    if it < 0:
        raise ValueError(f"or_push_virtual failed ({it})")
    return out, int(it), bool(conv.value)


def udt(g: CSR, K: int, dumb: int, unit_weight: int = 1):
    """Alg. 1 (UDT) on the oracle CSR: returns (n', src, dst, w) of the transformed graph.
    Arcs to original neighbours keep their weight (unit_weight when g is unweighted), arcs
    to new split nodes get `dumb` (0 for SSSP/BFS, 0xFFFFFFFF for SSWP; Cor. 2-3)."""
    m = ctypes.c_uint64(0)
    _lib().or_udt(g.n, _p(g.row_ptr), _p(g.col), _p(g.wt), K, dumb, unit_weight, None, None, None,
                  ctypes.byref(m))
    src = np.empty(m.value, np.uint32)
    dst = np.empty(m.value, np.uint32)
    w = np.empty(m.value, np.uint32)
    n2 = _lib().or_udt(g.n, _p(g.row_ptr), _p(g.col), _p(g.wt), K, dumb, unit_weight, _p(src), _p(dst),
                       _p(w), ctypes.byref(m))
    if n2 == 0 and g.n:
        raise ValueError("or_udt failed (K < 2?)")
    return int(n2), src, dst, w


def run(algo: str, n: int, src, dst, w=None, source: int = 0, pr_iters: int = 20,
        damping: float = 0.85, dangling: int = 0):
    """Oracle result for `algo` on the COO graph (CC symmetrises first, reading c6)."""
    a = ALGOS[algo]
    if a == CC:
        return cc(n, *symmetrize(src, dst)[:2])
    g = csr_build(n, src, dst, w)
    if a == BFS:
        return bfs(g, source)
    if a == SSSP:
        return sssp(g, source)
    if a == SSWP:
        return sswp(g, source)
    return pagerank(g, pr_iters, damping, dangling)
