"""Pins for the CPU oracle (oracle/), independent of the oracle itself and of
the CUDA path: the paper's worked examples (tests/golden/), brute force on tiny
graphs (tests/brute.py), library routines (scipy.sparse.csgraph), closed forms
and invariants.  Each test names what a plausible oracle bug would break.
"""
import numpy as np
import pytest
import scipy.sparse as sp
from scipy.sparse import csgraph

import graphgen
import oracle
from tests import brute

INF = oracle.INF


def _coo_small(seed, n=24, m=70, wmax=9):
    return graphgen.random_small(n, m, seed, wmax=wmax)


# --------------------------------------------------------------------------------------------
# worked examples from the paper
# --------------------------------------------------------------------------------------------

def _inf(row):
    return [INF if x == "inf" else x for x in row]


def test_fig2_sssp_trace(golden):
    """Fig. 2 (L242-309): BSP value rows of the SSSP example, iteration by iteration."""
    g0 = golden("fig2_sssp_trace.json")
    g = oracle.csr_build(g0["n"], g0["src"], g0["dst"], g0["w"])
    rows = [_inf(r) for _, r in g0["rows"]]
    for K in (1, 2, 8, 1 << 40):
        vg = oracle.Virtual(g, K)
        for it, want in enumerate(rows[1:], start=1):
            vals, n_it, _ = oracle.push_virtual(g, vg, oracle.SSSP, g0["source"], schedule=1,
                                                worklist=0, max_iters=it)
            assert n_it == it and list(vals) == want, (K, it)
        vals, n_it, conv = oracle.push_virtual(g, vg, oracle.SSSP, g0["source"], schedule=1,
                                               worklist=0)
        assert conv and n_it == 3 and list(vals) == rows[-1]
    # the fixed point is the textbook result
    assert list(oracle.sssp(g, 0)) == rows[-1]


def _fig10_graph(fx):
    src, dst = [], []
    for v, nbrs in sorted(fx["adjacency"].items(), key=lambda kv: int(kv[0])):
        src += [int(v)] * len(nbrs)
        dst += nbrs
    return oracle.csr_build(fx["n"], src, dst, None)


def test_fig10_virtual_node_array(golden):
    fx = golden("fig10_virtual_array.json")
    g = _fig10_graph(fx)
    assert list(g.row_ptr[1:4]) == fx["node_array_v1_v3"]
    vg = oracle.Virtual(g, fx["K"])
    assert list(vg.vn_phys) == fx["virtual_physical_ids"]
    # edge pointers of the vnodes, consecutive assignment (Alg. 2 start = edgePointer)
    starts = [int(vg.edges(i, 0)[0]) for i in range(vg.nv)] + [g.m]
    assert starts == fx["virtual_edge_pointers"] + [12][: len(starts) - 4]
    nbrs = [list(g.col[vg.edges(i, 0)]) for i in range(vg.nv)]
    assert nbrs == fx["consecutive_vnode_nbrs"]


def test_fig12_strided_assignment(golden):
    fx10 = golden("fig10_virtual_array.json")
    fx = golden("fig12_strided.json")
    g = _fig10_graph(fx10)
    vg = oracle.Virtual(g, fx10["K"])
    v = fx["vertex"]
    fam = range(int(vg.vnode_ptr[v]), int(vg.vnode_ptr[v + 1]))
    assert len(fam) == fx["family_size"]
    base = int(g.row_ptr[v])
    assert list(g.col[base:base + len(fx["segment"])]) == fx["segment"]
    for j, i in enumerate(fam):
        e = vg.edges(i, 1)
        assert list(e - base) == fx["positions"][j]
        assert list(g.col[e]) == fx["nbrs"][j]


def test_table6_space_shape(golden):
    """Table 6 (L1428-1438) space cost, shape check on R-MAT s20 (reading R9): within 5 points
    of both the LiveJournal and the twitter column (SURVEY.md §8(c) c3 gate)."""
    fx = golden("table6_space_cost.json")
    rec = graphgen.recipe("cfg2")
    src, dst, _ = graphgen.generate(rec, weighted=False)
    g = oracle.csr_build(rec.n, src, dst)
    csr_bytes = 4 * (rec.n + 1) + 4 * rec.m
    for K, lj, tw in zip(fx["K"], fx["LiveJournal"], fx["twitter"]):
        nv = oracle.Virtual(g, K).nv
        pct = 100.0 * (csr_bytes + 8 * nv) / csr_bytes
        assert abs(pct - lj) < 5.0 and abs(pct - tw) < 5.0, (K, pct)


# --------------------------------------------------------------------------------------------
# CSR (c2)
# --------------------------------------------------------------------------------------------

def test_csr_matches_stable_sort():
    src, dst, w = graphgen.rmat(300, 5000, 0.57, 0.19, 0.19, seed=21, wseed=22)
    g = oracle.csr_build(300, src, dst, w)
    order = np.argsort(src, kind="stable")
    assert np.array_equal(g.col, dst[order]) and np.array_equal(g.wt, w[order])
    assert np.array_equal(g.row_ptr, np.concatenate([[0], np.cumsum(np.bincount(src, minlength=300))]))
    with pytest.raises(ValueError):
        oracle.csr_build(10, [1, 10], [0, 0])


# --------------------------------------------------------------------------------------------
# virtual split (c3) -- invariants; Thm. 2; Table 8 iteration equality
# --------------------------------------------------------------------------------------------

@pytest.mark.parametrize("K", [1, 2, 3, 8, 33, 1 << 40])
def test_virtual_split_invariants(K):
    src, dst, _ = graphgen.rmat(512, 9000, 0.57, 0.19, 0.19, seed=31, weighted=False)
    g = oracle.csr_build(512, src, dst)
    vg = oracle.Virtual(g, K)
    deg = g.degrees()
    # family sizes: smallest number of <=K-edge pieces, zero for zero degree (Def. 2(iii))
    fam = np.diff(vg.vnode_ptr.astype(np.int64))
    assert ((fam == 0) == (deg == 0)).all()
    assert ((fam * K >= deg) & ((fam - 1) * K < deg) | (deg == 0)).all()
    if K == 1:
        assert vg.nv == g.m
    if K >= deg.max():
        assert vg.nv == int((deg > 0).sum())
    for layout, chunk in [(0, 1), (1, 1), (1, 2), (1, 4), (1, 8)]:
        seen = np.zeros(g.m, dtype=np.int64)
        for v in np.flatnonzero(deg):
            counts = []
            for i in range(int(vg.vnode_ptr[v]), int(vg.vnode_ptr[v + 1])):
                e = vg.edges(i, layout, chunk)
                assert ((e >= g.row_ptr[v]) & (e < g.row_ptr[v + 1])).all()
                seen[e] += 1
                counts.append(len(e))
            assert max(counts) <= K or K % chunk  # chunked layout keeps <=K when chunk | K
            if layout == 0:
                assert all(c == K for c in counts[:-1])
            if layout == 1 and chunk == 1:
                assert max(counts) - min(counts) <= 1
        assert (seen == 1).all(), (layout, chunk)


@pytest.mark.parametrize("K", [1, 2, 4, 8, 12, 32])
@pytest.mark.parametrize("chunk", [1, 2, 4, 8])
def test_strided_chunk_closed_form(K, chunk):
    """Strided layout with c-arc units (Fig. 12 L1141-1159 with c = 1):
    vnode j of a family of m_v owns units j, j + m_v, j + 2 m_v, ... of its segment, i.e. its
    t-th unit starts at row_ptr[v] + c (t m_v + j) and covers c consecutive arcs, cut at the
    segment end.  Written out per (v, j, t) -- no modular arithmetic -- and compared with the
    oracle's assignment arc by arc, in order."""
    src, dst, _ = graphgen.rmat(256, 6000, 0.57, 0.19, 0.19, seed=41, weighted=False)
    g = oracle.csr_build(256, src, dst)
    vg = oracle.Virtual(g, K)
    deg = g.degrees()
    for v in np.flatnonzero(deg):
        d, base = int(deg[v]), int(g.row_ptr[v])
        mv = int(vg.vnode_ptr[v + 1] - vg.vnode_ptr[v])
        for j in range(mv):
            want, t = [], 0
            while chunk * (t * mv + j) < d:
                start = chunk * (t * mv + j)
                want.extend(base + start + u for u in range(chunk) if start + u < d)
                t += 1
            got = vg.edges(int(vg.vnode_ptr[v]) + j, 1, chunk)
            assert list(got) == want, (v, j, K, chunk)


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_thm2_virtual_push_equals_textbook(seed):
    """Thm. 2 (L1030-1045): push on the virtual graph reaches the original-graph result,
    for every K, layout, schedule; BSP iteration counts are K-invariant (Table 8)."""
    n = 400
    src, dst, w = graphgen.rmat(n, 6000, 0.57, 0.19, 0.19, seed=40 + seed, wseed=50 + seed)
    g = oracle.csr_build(n, src, dst, w)
    sym = oracle.symmetrize(src, dst, w)
    gs = oracle.csr_build(n, *sym)
    want = {oracle.BFS: oracle.bfs(g, 0), oracle.SSSP: oracle.sssp(g, 0),
            oracle.SSWP: oracle.sswp(g, 0), oracle.CC: oracle.cc(n, src, dst)}
    for algo, ref in want.items():
        gg = gs if algo == oracle.CC else g
        iters = set()
        for K in (1, 3, 8, 1 << 40):
            vg = oracle.Virtual(gg, K)
            for layout, chunk in [(0, 1), (1, 1), (1, 4), (1, 8)]:
                for schedule in (0, 1):
                    vals, it, conv = oracle.push_virtual(gg, vg, algo, 0, layout, chunk, schedule, 1)
                    assert conv and np.array_equal(vals, ref), (algo, K, layout, schedule)
                    if schedule == 1:
                        iters.add(it)
        assert len(iters) == 1, (algo, iters)


# --------------------------------------------------------------------------------------------
# algorithms vs brute force (tiny) and library routines (cfg1)
# --------------------------------------------------------------------------------------------

@pytest.mark.parametrize("seed", range(6))
def test_algorithms_vs_brute_force(seed):
    n = 20 + seed
    src, dst, w = _coo_small(seed, n=n, m=3 * n)
    g = oracle.csr_build(n, src, dst, w)
    for s in (0, n // 2):
        assert np.array_equal(oracle.bfs(g, s), brute.bfs(n, src, dst, s))
        assert np.array_equal(oracle.sssp(g, s), brute.sssp(n, src, dst, w, s))
        assert np.array_equal(oracle.sswp(g, s), brute.sswp(n, src, dst, w, s))
    assert np.array_equal(oracle.cc(n, src, dst), brute.cc(n, src, dst))
    for dangling in (0, 1):
        x = oracle.pagerank(g, 20, 0.85, dangling)
        assert np.abs(x - brute.pagerank_dense(n, src, dst, 20, 0.85, dangling)).max() < 1e-15


def _scipy_graph(n, src, dst, w):
    # csgraph sums duplicate entries; keep the minimum weight per (src, dst) pair first
    key = src.astype(np.int64) * n + dst
    order = np.lexsort((w, key))
    key, w = key[order], w[order]
    first = np.ones(len(key), dtype=bool)
    first[1:] = key[1:] != key[:-1]
    k = key[first]
    return sp.csr_matrix((w[first].astype(np.float64), (k // n, k % n)), shape=(n, n))


def test_cfg1_against_scipy_csgraph():
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    g = oracle.csr_build(rec.n, src, dst, w)
    A = _scipy_graph(rec.n, src, dst, w)
    d = csgraph.dijkstra(A, directed=True, indices=0)
    want = np.where(np.isinf(d), INF, d).astype(np.uint32)
    assert np.array_equal(oracle.sssp(g, 0), want)
    h = csgraph.shortest_path(A, directed=True, indices=0, unweighted=True)
    assert np.array_equal(oracle.bfs(g, 0), np.where(np.isinf(h), INF, h).astype(np.uint32))
    ncomp, lab = csgraph.connected_components(A, directed=True, connection="weak")
    first = np.full(ncomp, rec.n)
    np.minimum.at(first, lab, np.arange(rec.n))
    assert np.array_equal(oracle.cc(rec.n, src, dst), first[lab].astype(np.uint32))


def test_cfg1_sswp_and_sssp_vs_floyd_warshall():
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    g = oracle.csr_build(rec.n, src, dst, w)
    assert np.array_equal(oracle.sssp(g, 0), brute.sssp(rec.n, src, dst, w, 0))
    assert np.array_equal(oracle.sswp(g, 0), brute.sswp(rec.n, src, dst, w, 0))


# --------------------------------------------------------------------------------------------
# special cases and closed forms
# --------------------------------------------------------------------------------------------

def test_special_cases():
    # single vertex, no edges
    g = oracle.csr_build(1, [], [], [])
    assert list(oracle.bfs(g, 0)) == [0] and list(oracle.sswp(g, 0)) == [INF]
    assert list(oracle.cc(1, [], [])) == [0]
    assert oracle.pagerank(g, 20)[0] == pytest.approx(0.15)  # dangling mass dropped
    # source with out-degree 0: only the source is reached
    g = oracle.csr_build(3, [1], [2], [5])
    assert list(oracle.sssp(g, 0)) == [0, INF, INF]
    assert list(oracle.sswp(g, 0)) == [INF, 0, 0]
    # SSSP with all-unit weights == BFS (L718-720)
    src, dst, _ = _coo_small(7, n=50, m=200)
    g = oracle.csr_build(50, src, dst, np.ones(len(src), np.uint32))
    assert np.array_equal(oracle.sssp(g, 3), oracle.bfs(g, 3))
    # SSWP with constant weight c: every reachable non-source vertex has width c
    g = oracle.csr_build(50, src, dst, np.full(len(src), 7, np.uint32))
    b = oracle.bfs(g, 3)
    s = oracle.sswp(g, 3)
    assert (s[(b != INF) & (np.arange(50) != 3)] == 7).all() and (s[b == INF] == 0).all()
    # CC: isolated vertices keep their id; two disjoint cliques -> their min ids
    lab = oracle.cc(7, [1, 2, 3, 5, 6], [2, 3, 1, 6, 5])
    assert list(lab) == [0, 1, 1, 1, 4, 5, 5]


def test_pagerank_closed_forms():
    n = 37
    cyc = np.arange(n, dtype=np.uint32)
    g = oracle.csr_build(n, cyc, (cyc + 1) % n)
    for T in (1, 5, 20):
        assert (oracle.pagerank(g, T) == 1.0 / n).all()
    # no dangling vertices -> mass conserved
    src, dst, _ = _coo_small(3, n=60, m=600)
    src = np.concatenate([src, np.arange(60, dtype=np.uint32)])
    dst = np.concatenate([dst, (np.arange(60, dtype=np.uint32) * 7) % 60])
    g = oracle.csr_build(60, src, dst)
    assert abs(oracle.pagerank(g, 20).sum() - 1.0) < 1e-13
    # T -> infinity converges to the linear solve at rate 0.85^T
    A = np.zeros((60, 60))
    np.add.at(A, (src.astype(np.int64), dst.astype(np.int64)), 1.0)
    P = A / A.sum(axis=1, keepdims=True)
    xs = np.linalg.solve(np.eye(60) - 0.85 * P.T, np.full(60, 0.15 / 60))
    assert np.abs(oracle.pagerank(g, 200) - xs).max() < 1e-14


def test_fixed_point_invariants_cfg2():
    """Fixed point + tightness on a config-size graph (properties that hold at any size)."""
    rec = graphgen.recipe("cfg2")
    src, dst, w = graphgen.rmat(rec.n, rec.m // 4, rec.a, rec.b, rec.c, rec.seed, rec.wseed)
    n = rec.n
    g = oracle.csr_build(n, src, dst, w)
    s64, d64, w64 = src.astype(np.int64), dst.astype(np.int64), w.astype(np.int64)
    lvl = oracle.bfs(g, 0).astype(np.int64)
    fin = lvl[s64] != INF
    assert (lvl[d64][fin] <= lvl[s64][fin] + 1).all()
    tight = np.zeros(n, bool)
    tight[d64[fin & (lvl[d64] == lvl[s64] + 1)]] = True
    reached = lvl != INF
    reached[0] = False
    assert tight[reached].all()
    dist = oracle.sssp(g, 0).astype(np.int64)
    fin = dist[s64] != INF
    assert (dist[d64][fin] <= dist[s64][fin] + w64[fin]).all()
    tight[:] = False
    tight[d64[fin & (dist[d64] == dist[s64] + w64)]] = True
    assert tight[(dist != INF) & (np.arange(n) != 0)].all()
    assert ((dist == INF) == (lvl == INF)).all()
    wid = oracle.sswp(g, 0).astype(np.int64)
    pos = wid[s64] > 0
    assert (wid[d64][pos] >= np.minimum(wid[s64][pos], w64[pos])).all()
    lab = oracle.cc(n, src, dst)
    assert (lab[src] == lab[dst]).all() and (lab <= np.arange(n)).all()
    assert (lab[lab] == lab).all()


# --------------------------------------------------------------------------------------------
# UDT (Alg. 1) -- pinned by Thm. 1 / Cor. 1-3 against the textbook results on the original
# --------------------------------------------------------------------------------------------

@pytest.mark.parametrize("K", [2, 3, 8])
def test_udt_preserves_results(K):
    n = 300
    src, dst, w = graphgen.rmat(n, 5000, 0.57, 0.19, 0.19, seed=61, wseed=62)
    g = oracle.csr_build(n, src, dst, w)
    deg = g.degrees()
    # SSSP with dumb weight 0 (Cor. 2): distances of original nodes unchanged
    n2, us, ud, uw = oracle.udt(g, K, 0)
    gu = oracle.csr_build(n2, us, ud, uw)
    assert np.array_equal(oracle.sssp(gu, 0)[:n], oracle.sssp(g, 0))
    # structure: every node has out-degree <= K; new nodes exactly K (L567-569); arcs = m + #new
    du = gu.degrees()
    assert du.max() <= K and (du[n:] == K).all() and gu.m == g.m + (n2 - n)
    # #new nodes per high-degree node d: ceil((d-K)/(K-1)) (queue shrinks by K-1 per new node)
    hi_deg = deg[deg > K]
    assert n2 - n == int(sum(-(-(d - K) // (K - 1)) for d in hi_deg))
    # BFS = SSSP with unit weights on original arcs and dumb 0 (L718-720)
    g1 = oracle.csr_build(n, src, dst)
    n2, us, ud, uw = oracle.udt(g1, K, 0, unit_weight=1)
    assert np.array_equal(oracle.sssp(oracle.csr_build(n2, us, ud, uw), 0)[:n], oracle.bfs(g1, 0))
    # SSWP with dumb weight +inf (Cor. 3)
    n2, us, ud, uw = oracle.udt(g, K, 0xFFFFFFFF)
    assert np.array_equal(oracle.sswp(oracle.csr_build(n2, us, ud, uw), 0)[:n], oracle.sswp(g, 0))
    # connectivity (Cor. 1): weak components restricted to original nodes unchanged
    assert np.array_equal(oracle.cc(n2, us, ud)[:n], oracle.cc(n, src, dst))


def test_udt_example_degree_five():
    """Fig. 6-(b) (L566): a node of degree five with K = 2 -> 3 new nodes, root keeps 2."""
    g = oracle.csr_build(6, [0] * 5, [1, 2, 3, 4, 5], [1, 1, 1, 1, 1])
    n2, us, ud, uw = oracle.udt(g, 2, 0)
    assert n2 == 6 + 3
    gu = oracle.csr_build(n2, us, ud, uw)
    assert list(gu.degrees()) == [2, 0, 0, 0, 0, 0, 2, 2, 2]
