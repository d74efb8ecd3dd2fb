"""B200-native Tigr hot path: Python binding of libtigr.so (include/tigr.h).

Argument marshalling only -- every step of the path (R-MAT generation, CSR build, virtual
split, layout, relax kernels, frontier, PageRank apply, multi-GPU exchange) runs in the CUDA
kernels of libtigr.so.  There is no CPU fallback: importing this package fails loudly if the
library is missing, and every call raises TigrError when the C ABI reports an error.

Function names mirror the C ABI.  Arrays may be numpy arrays (host) or torch tensors
(host or CUDA); 32-bit data is passed as uint32 (numpy) / int32 or uint32 (torch) bits.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("TIGR_LIB") or os.path.join(_HERE, "libtigr.so")  # TIGR_LIB: A/B builds (development)

if not os.path.exists(LIB_PATH):
    raise ImportError(
        f"{LIB_PATH} is missing: build it with `python -c 'import __graft_entry__ as g; g.build()'` "
        "(nvcc, sm_100a). There is no CPU fallback.")

_lib = ctypes.CDLL(LIB_PATH)

TIGR_OK, TIGR_EINVAL, TIGR_ENOMEM, TIGR_ECUDA, TIGR_ENCCL, TIGR_ERANGE, TIGR_ENOTCONV, TIGR_EUNSUPPORTED = \
    0, -1, -2, -3, -4, -5, -6, -7
TIGR_BFS, TIGR_SSSP, TIGR_CC, TIGR_SSWP, TIGR_PR = 0, 1, 2, 3, 4
TIGR_LAYOUT_CONSECUTIVE, TIGR_LAYOUT_STRIDED = 0, 1
TIGR_FRONTIER_AUTO, TIGR_FRONTIER_DENSE, TIGR_FRONTIER_NONE, TIGR_FRONTIER_QUEUE = 0, 1, 2, 3
TIGR_EXCHANGE_AUTO, TIGR_EXCHANGE_DENSE, TIGR_EXCHANGE_SPARSE, TIGR_EXCHANGE_FUSED = 0, 1, 2, 3
EXCHANGES = {"auto": TIGR_EXCHANGE_AUTO, "dense": TIGR_EXCHANGE_DENSE, "sparse": TIGR_EXCHANGE_SPARSE,
             "fused": TIGR_EXCHANGE_FUSED}
ALGOS = {"bfs": TIGR_BFS, "sssp": TIGR_SSSP, "cc": TIGR_CC, "sswp": TIGR_SSWP, "pr": TIGR_PR}
LAYOUTS = {"consecutive": TIGR_LAYOUT_CONSECUTIVE, "strided": TIGR_LAYOUT_STRIDED}
INF = 0xFFFFFFFF
K_NO_SPLIT = 0xFFFFFFFF


class TigrError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"tigr status {status}: {msg}")
        self.status = status


class tigr_run_opts(ctypes.Structure):
    _fields_ = [("max_iters", ctypes.c_uint32), ("pr_iters", ctypes.c_uint32), ("pr_damping", ctypes.c_double),
                ("pr_dangling", ctypes.c_int), ("schedule", ctypes.c_int), ("frontier", ctypes.c_int),
                ("use_graph", ctypes.c_int), ("collect_stats", ctypes.c_int), ("time_kernels", ctypes.c_int),
                ("comm", ctypes.c_void_p), ("stream", ctypes.c_void_p), ("exchange", ctypes.c_int),
                ("frontier_div", ctypes.c_uint32)]


class tigr_stats(ctypes.Structure):
    _fields_ = [("iterations", ctypes.c_uint32), ("relax_launches", ctypes.c_uint32),
                ("edges_processed", ctypes.c_uint64), ("updates", ctypes.c_uint64),
                ("active_vnodes", ctypes.c_uint64), ("ms_total", ctypes.c_double), ("ms_relax", ctypes.c_double),
                ("ms_exchange", ctypes.c_double), ("queue_iterations", ctypes.c_uint32), ("sparse_exchanges", ctypes.c_uint32),
                ("active_nodes", ctypes.c_uint64), ("ms_kernels", ctypes.c_double), ("bytes_alg", ctypes.c_uint64)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


_P, _U32, _U64, _I, _D = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int, ctypes.c_double
_SIGS = {
    "tigr_run_opts_default": (None, [ctypes.POINTER(tigr_run_opts)]),
    "tigr_graph_from_coo": (_I, [_U32, _U64, _P, _P, _P, _I, _I, _P, ctypes.POINTER(_P)]),
    "tigr_graph_from_csr": (_I, [_U32, _U64, _P, _P, _P, _I, _I, _P, ctypes.POINTER(_P)]),
    "tigr_graph_from_coo_part": (_I, [_U32, _U64, _P, _P, _P, _I, _I, _U32, _U32, _P, ctypes.POINTER(_P)]),
    "tigr_coo_source_cuts": (_I, [_U32, _U64, _P, _P, _I, _I, _I, _P, _P]),
    "tigr_rmat_coo": (_I, [_U32, _U64, _D, _D, _D, _U64, _U64, _U32, _U32, _P, _P, _P, _P]),
    "tigr_graph_rmat": (_I, [_U32, _U64, _D, _D, _D, _U64, _U64, _U32, _U32, _I, _I, _P, ctypes.POINTER(_P)]),
    "tigr_graph_info": (_I, [_P, ctypes.POINTER(_U32), ctypes.POINTER(_U64), ctypes.POINTER(_I),
                             ctypes.POINTER(_I), ctypes.POINTER(_I), ctypes.POINTER(_U64)]),
    "tigr_graph_transpose": (_I, [_P, _P, ctypes.POINTER(_P)]),
    "tigr_graph_udt": (_I, [_P, _U32, _U32, _U32, _P, ctypes.POINTER(_P)]),
    "tigr_graph_reorder": (_I, [_P, _P, ctypes.POINTER(_P)]),
    "tigr_graph_permutation": (_I, [_P, _P, _P, _I, _P]),
    "tigr_graph_export_csr": (_I, [_P, _P, _P, _P, _I, _P]),
    "tigr_graph_export_coo": (_I, [_P, _P, _P, _P, _I, _P]),
    "tigr_graph_free": (None, [_P]),
    "tigr_virtualize": (_I, [_P, _U32, _I, _P, ctypes.POINTER(_P)]),
    "tigr_vgraph_info": (_I, [_P, ctypes.POINTER(_U64), ctypes.POINTER(_U64), ctypes.POINTER(_D),
                              ctypes.POINTER(_U32), ctypes.POINTER(_U32)]),
    "tigr_vgraph_export": (_I, [_P, _P, _P, _I, _P]),
    "tigr_vgraph_pr_profile": (_I, [_P, _P, ctypes.POINTER(_U64), ctypes.POINTER(_U64), ctypes.POINTER(_U32),
                                    ctypes.POINTER(_U32)]),
    "tigr_vgraph_assignment": (_I, [_P, _P, _P, _P, _I, _P]),
    "tigr_vgraph_partition": (_I, [_P, _I, _I]),
    "tigr_partition_ranges": (_I, [_U32, _P, _P, _I, _P, _P]),
    "tigr_vgraph_free": (None, [_P]),
    "tigr_run": (_I, [_P, _I, _U32, ctypes.POINTER(tigr_run_opts), _P, _I, ctypes.POINTER(tigr_stats)]),
    "tigr_comm_unique_id": (_I, [_P]),
    "tigr_comm_init": (_I, [_I, _I, _P, _I, ctypes.POINTER(_P)]),
    "tigr_comm_free": (None, [_P]),
    "tigr_comm_group_create": (_I, [_I, ctypes.POINTER(_P)]),
    "tigr_comm_init_group": (_I, [_P, _I, ctypes.POINTER(_P)]),
    "tigr_comm_group_free": (None, [_P]),
    "tigr_comm_init_node": (_I, [ctypes.c_char_p, _I, _I, ctypes.POINTER(_P)]),
    "tigr_last_error": (ctypes.c_char_p, []),
    "tigr_launch_count": (_U64, []),
    "tigr_release_cached_memory": (None, []),
    "tigr_version": (ctypes.c_char_p, []),
}
for _name, (_res, _args) in _SIGS.items():
    _f = getattr(_lib, _name)
    _f.restype = _res
    _f.argtypes = _args

EXPORTED_SYMBOLS = tuple(_SIGS)


def _check(status: int):
    if status != TIGR_OK:
        raise TigrError(status, _lib.tigr_last_error().decode(errors="replace"))


def _arr(a, dtype=np.uint32):
    """(pointer, is_device, keepalive) for a numpy array / torch tensor / None."""
    if a is None:
        return None, 0, None
    mod = type(a).__module__
    if mod.startswith("torch"):
        if not a.is_contiguous():
            raise ValueError("tensor must be contiguous")
        return a.data_ptr(), int(a.is_cuda), a
    arr = np.ascontiguousarray(a, dtype=dtype)
    return arr.ctypes.data, 0, arr


def _stream_ptr(stream):
    if stream is None:
        return None
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream  # torch.cuda.Stream


def _len(a):
    return 0 if a is None else (a.numel() if type(a).__module__.startswith("torch") else len(a))


# ------------------------------------------------------------------------------ handles
class Graph:
    """Owning wrapper of a tigr_graph* (device CSR)."""

    def __init__(self, ptr):
        self._ptr = ctypes.c_void_p(ptr)

    @property
    def ptr(self):
        return self._ptr

    def info(self):
        n, m, wt, sym, tr, b = _U32(), _U64(), _I(), _I(), _I(), _U64()
        _check(_lib.tigr_graph_info(self._ptr, n, m, wt, sym, tr, b))
        return {"n": n.value, "m": m.value, "weighted": bool(wt.value), "symmetric": bool(sym.value),
                "transposed": bool(tr.value), "device_bytes": b.value}

    def free(self):
        if self._ptr:
            _lib.tigr_graph_free(self._ptr)
            self._ptr = ctypes.c_void_p(None)

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


class VGraph:
    """Owning wrapper of a tigr_vgraph* (keeps its Graph alive)."""

    def __init__(self, ptr, graph: Graph):
        self._ptr = ctypes.c_void_p(ptr)
        self.graph = graph

    @property
    def ptr(self):
        return self._ptr

    def info(self):
        nv, b, ms, lo, hi = _U64(), _U64(), _D(), _U32(), _U32()
        _check(_lib.tigr_vgraph_info(self._ptr, nv, b, ms, lo, hi))
        return {"nv": nv.value, "bytes": b.value, "ms_build": ms.value, "lo": lo.value, "hi": hi.value}

    def free(self):
        if self._ptr:
            _lib.tigr_vgraph_free(self._ptr)
            self._ptr = ctypes.c_void_p(None)

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


class Comm:
    def __init__(self, ptr, nranks, rank):
        self._ptr = ctypes.c_void_p(ptr)
        self.nranks, self.rank = nranks, rank

    @property
    def ptr(self):
        return self._ptr

    def free(self):
        if self._ptr:
            _lib.tigr_comm_free(self._ptr)
            self._ptr = ctypes.c_void_p(None)

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


class CommGroup:
    """Owning wrapper of a tigr_comm_group* (ranks that are threads of this process)."""

    def __init__(self, ptr, nranks):
        self._ptr = ctypes.c_void_p(ptr)
        self.nranks = nranks

    @property
    def ptr(self):
        return self._ptr

    def free(self):
        if self._ptr:
            _lib.tigr_comm_group_free(self._ptr)
            self._ptr = ctypes.c_void_p(None)

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


# ------------------------------------------------------------------------------ C ABI, same names
def tigr_run_opts_default() -> tigr_run_opts:
    o = tigr_run_opts()
    _lib.tigr_run_opts_default(ctypes.byref(o))
    return o


def tigr_graph_from_coo(n, src, dst, w=None, symmetrize=False, stream=None) -> Graph:
    m = _len(src)
    ps, ds, ks = _arr(src)
    pd, dd, kd = _arr(dst)
    pw, dw, kw = _arr(w)
    if _len(dst) != m or (w is not None and _len(w) != m):
        raise ValueError("src/dst/w lengths differ")
    if len({x for x in (ds, dd, dw if w is not None else ds)}) != 1:
        raise ValueError("src/dst/w must all be host or all device")
    out = _P()
    _check(_lib.tigr_graph_from_coo(n, m, ps, pd, pw, ds, int(symmetrize), _stream_ptr(stream), ctypes.byref(out)))
    return Graph(out.value)


def tigr_graph_from_coo_part(n, src, dst, w=None, symmetrize=False, src_lo=0, src_hi=0xFFFFFFFF,
                             stream=None) -> Graph:
    """Partitioned build: keep only arcs with source in [src_lo, src_hi) (multi-GPU ranks)."""
    m = _len(src)
    ps, ds, ks = _arr(src)
    pd, dd, kd = _arr(dst)
    pw, dw, kw = _arr(w)
    out = _P()
    _check(_lib.tigr_graph_from_coo_part(n, m, ps, pd, pw, ds, int(symmetrize), src_lo, src_hi,
                                         _stream_ptr(stream), ctypes.byref(out)))
    return Graph(out.value)


def tigr_coo_source_cuts(n, src, dst, nranks, symmetrize=False, stream=None):
    """Source-node cuts (nranks+1 entries) balancing arc counts across ranks."""
    ps, ds, ks = _arr(src)
    pd, dd, kd = _arr(dst)
    cuts = np.empty(nranks + 1, dtype=np.uint32)
    _check(_lib.tigr_coo_source_cuts(n, _len(src), ps, pd, ds, int(symmetrize), nranks, _stream_ptr(stream),
                                     cuts.ctypes.data))
    return cuts


def tigr_graph_from_csr(n, row_ptr, col, w=None, symmetric_hint=False, stream=None) -> Graph:
    m = _len(col)
    pr, dr, kr = _arr(row_ptr, np.int64)
    pc, dc, kc = _arr(col)
    pw, dw, kw = _arr(w)
    out = _P()
    _check(_lib.tigr_graph_from_csr(n, m, pr, pc, pw, dr, int(symmetric_hint), _stream_ptr(stream),
                                    ctypes.byref(out)))
    return Graph(out.value)


def tigr_rmat_coo(n, m, a, b, c, seed, wseed, wmin, wmax, src, dst, w=None, stream=None):
    """Device R-MAT into caller-owned CUDA tensors src/dst[/w] (length m)."""
    ps, ds, _ = _arr(src)
    pd, dd, _ = _arr(dst)
    pw, dw, _ = _arr(w)
    if not ds or not dd or (w is not None and not dw):
        raise ValueError("tigr_rmat_coo writes device buffers: pass CUDA tensors")
    _check(_lib.tigr_rmat_coo(n, m, a, b, c, seed, wseed, wmin, wmax, ps, pd, pw, _stream_ptr(stream)))


def tigr_graph_rmat(n, m, a, b, c, seed, wseed=0, wmin=1, wmax=64, weighted=True, symmetrize=False,
                    stream=None) -> Graph:
    out = _P()
    _check(_lib.tigr_graph_rmat(n, m, a, b, c, seed, wseed, wmin, wmax, int(weighted), int(symmetrize),
                                _stream_ptr(stream), ctypes.byref(out)))
    return Graph(out.value)


def tigr_graph_transpose(g: Graph, stream=None) -> Graph:
    """In-CSR of g (arcs reversed; carries g's out-degrees: TIGR_PR on it is pull-based)."""
    out = _P()
    _check(_lib.tigr_graph_transpose(g.ptr, _stream_ptr(stream), ctypes.byref(out)))
    return Graph(out.value)


def tigr_graph_reorder(g: Graph, stream=None) -> Graph:
    """Same graph, nodes relabelled by decreasing in-degree; runs on it take and return original ids."""
    out = _P()
    _check(_lib.tigr_graph_reorder(g.ptr, _stream_ptr(stream), ctypes.byref(out)))
    return Graph(out.value)


def tigr_graph_permutation(g: Graph, stream=None):
    """Host copies (cid uint32[n]: original -> new id, order uint32[n]: new -> original id)."""
    n = g.info()["n"]
    cid = np.empty(max(n, 1), dtype=np.uint32)
    order = np.empty(max(n, 1), dtype=np.uint32)
    _check(_lib.tigr_graph_permutation(g.ptr, cid.ctypes.data, order.ctypes.data, 0, _stream_ptr(stream)))
    return cid[:n], order[:n]


def tigr_graph_udt(g: Graph, K: int, dumb_weight: int = 0, unit_weight: int = 1, stream=None) -> Graph:
    """Physical UDT transformation (Alg. 1): n + T nodes; originals keep ids 0..n-1."""
    out = _P()
    _check(_lib.tigr_graph_udt(g.ptr, K, dumb_weight, unit_weight, _stream_ptr(stream), ctypes.byref(out)))
    return Graph(out.value)


def tigr_graph_export_csr(g: Graph, stream=None):
    """Host copies (row_ptr int64[n+1], col uint32[m], w uint32[m] or None)."""
    info = g.info()
    rp = np.empty(info["n"] + 1, dtype=np.int64)
    col = np.empty(info["m"], dtype=np.uint32)
    w = np.empty(info["m"], dtype=np.uint32) if info["weighted"] else None
    _check(_lib.tigr_graph_export_csr(g.ptr, rp.ctypes.data, col.ctypes.data,
                                      None if w is None else w.ctypes.data, 0, _stream_ptr(stream)))
    return rp, col, w


def tigr_graph_export_coo(g: Graph, stream=None):
    """Host copies (src uint32[m], dst uint32[m], w uint32[m] or None) in canonical CSR order."""
    info = g.info()
    m = info["m"]
    src = np.empty(max(m, 1), dtype=np.uint32)
    dst = np.empty(max(m, 1), dtype=np.uint32)
    w = np.empty(max(m, 1), dtype=np.uint32) if info["weighted"] else None
    _check(_lib.tigr_graph_export_coo(g.ptr, src.ctypes.data, dst.ctypes.data,
                                      None if w is None else w.ctypes.data, 0, _stream_ptr(stream)))
    return src[:m], dst[:m], (None if w is None else w[:m])


def tigr_virtualize(g: Graph, K: int = 8, layout="strided", stream=None) -> VGraph:
    lay = LAYOUTS[layout] if isinstance(layout, str) else int(layout)
    out = _P()
    _check(_lib.tigr_virtualize(g.ptr, K, lay, _stream_ptr(stream), ctypes.byref(out)))
    return VGraph(out.value, g)


def tigr_vgraph_export(vg: VGraph, stream=None):
    """Host copies (vnode_ptr uint32[n+1], vn_phys uint32[NV])."""
    n = vg.graph.info()["n"]
    nv = vg.info()["nv"]
    vp = np.empty(n + 1, dtype=np.uint32)
    ph = np.empty(max(nv, 1), dtype=np.uint32)
    _check(_lib.tigr_vgraph_export(vg.ptr, vp.ctypes.data, ph.ctypes.data, 0, _stream_ptr(stream)))
    return vp, ph[:nv]


def tigr_vgraph_pr_profile(vg: VGraph, stream=None) -> dict:
    """Push PageRank's split of this rank's arcs: shared-memory hot slots vs global float64 REDs."""
    a, r, h, ni = _U64(), _U64(), _U32(), _U32()
    _check(_lib.tigr_vgraph_pr_profile(vg.ptr, _stream_ptr(stream), ctypes.byref(a), ctypes.byref(r),
                                       ctypes.byref(h), ctypes.byref(ni)))
    return {"arcs": a.value, "global_reds": r.value, "hot_slots": h.value, "n_in": ni.value}


def tigr_vgraph_assignment(vg: VGraph, stream=None):
    """Host copies (counts uint32[NV], nbr uint32[m], w uint32[m] or None) as walked by the kernels."""
    gi = vg.graph.info()
    nv = vg.info()["nv"]
    counts = np.empty(max(nv, 1), dtype=np.uint32)
    nbr = np.empty(max(gi["m"], 1), dtype=np.uint32)
    w = np.empty(max(gi["m"], 1), dtype=np.uint32) if gi["weighted"] else None
    _check(_lib.tigr_vgraph_assignment(vg.ptr, counts.ctypes.data, nbr.ctypes.data,
                                       None if w is None else w.ctypes.data, 0, _stream_ptr(stream)))
    return counts[:nv], nbr[:gi["m"]], (None if w is None else w[:gi["m"]])


def tigr_vgraph_partition(vg: VGraph, nranks: int, rank: int):
    _check(_lib.tigr_vgraph_partition(vg.ptr, nranks, rank))


def tigr_partition_ranges(row_ptr, vnode_ptr, nranks: int):
    """Host-only: (lo[nranks], hi[nranks]) vnode ranges from host row_ptr / vnode_ptr arrays."""
    rp = np.ascontiguousarray(row_ptr, dtype=np.int64)
    vp = np.ascontiguousarray(vnode_ptr, dtype=np.uint32)
    lo = np.empty(nranks, dtype=np.uint32)
    hi = np.empty(nranks, dtype=np.uint32)
    _check(_lib.tigr_partition_ranges(len(rp) - 1, rp.ctypes.data, vp.ctypes.data, nranks, lo.ctypes.data,
                                      hi.ctypes.data))
    return lo, hi


def tigr_run(vg: VGraph, algo, source=0, opts: tigr_run_opts | None = None, out=None, stream=None,
             return_stats=False, **kw):
    """Run `algo` ('bfs'|'sssp'|'cc'|'sswp'|'pr' or TIGR_*) and return per-vertex values.

    out: optional preallocated numpy array / torch tensor (host or CUDA) of n elements
    (uint32 / int32 bits, float64 for PR).  Keyword options override fields of `opts`."""
    a = ALGOS[algo] if isinstance(algo, str) else int(algo)
    o = opts if opts is not None else tigr_run_opts_default()
    for k, v in kw.items():
        if k == "comm":
            v = v.ptr if isinstance(v, Comm) else v
        elif k == "exchange" and isinstance(v, str):
            v = EXCHANGES[v]
        setattr(o, k, v)
    if stream is not None:
        o.stream = _stream_ptr(stream)
    n = vg.graph.info()["n"]
    if out is None:
        out = np.empty(n, dtype=np.float64 if a == TIGR_PR else np.uint32)
    po, do, keep = _arr(out, np.float64 if a == TIGR_PR else np.uint32)
    st = tigr_stats()
    _check(_lib.tigr_run(vg.ptr, a, source, ctypes.byref(o), po, do, ctypes.byref(st)))
    return (keep, st.as_dict()) if return_stats else keep


def tigr_comm_unique_id() -> bytes:
    buf = (ctypes.c_uint8 * 128)()
    _check(_lib.tigr_comm_unique_id(buf))
    return bytes(buf)


def tigr_comm_init(nranks: int, rank: int, uid: bytes, device: int = -1) -> Comm:
    """NCCL communicator of `rank` on CUDA device `device` (-1: the current device)."""
    buf = (ctypes.c_uint8 * 128).from_buffer_copy(uid)
    out = _P()
    _check(_lib.tigr_comm_init(nranks, rank, buf, device, ctypes.byref(out)))
    return Comm(out.value, nranks, rank)


def tigr_comm_group_create(nranks: int) -> CommGroup:
    """A group of `nranks` ranks that are threads of this process (one tigr_comm each)."""
    out = _P()
    _check(_lib.tigr_comm_group_create(nranks, ctypes.byref(out)))
    return CommGroup(out.value, nranks)


def tigr_comm_init_group(group: CommGroup, rank: int) -> Comm:
    """Join `group` as `rank` on the calling thread's current CUDA device; returns once every
    rank has joined (call it from each rank's thread)."""
    out = _P()
    _check(_lib.tigr_comm_init_group(group.ptr, rank, ctypes.byref(out)))
    return Comm(out.value, group.nranks, rank)


def tigr_comm_init_node(name: str, nranks: int, rank: int) -> Comm:
    """Join the node communicator `name` (ranks = processes of this node, CUDA IPC + shared
    memory, no NCCL) as `rank` on the current CUDA device; returns once all ranks joined."""
    out = _P()
    _check(_lib.tigr_comm_init_node(name.encode(), nranks, rank, ctypes.byref(out)))
    return Comm(out.value, nranks, rank)


def tigr_last_error() -> str:
    return _lib.tigr_last_error().decode(errors="replace")


def tigr_launch_count() -> int:
    return int(_lib.tigr_launch_count())


def tigr_release_cached_memory() -> None:
    _lib.tigr_release_cached_memory()


def tigr_version() -> str:
    return _lib.tigr_version().decode()
