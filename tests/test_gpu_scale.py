"""GPU parity at BASELINE.json's full sizes, in the launch configuration bench.py times
(K = 8, strided layout, default kernels: hot-destination PR, 4-vnodes-per-thread frontier
kernels, CUDA-graph loop).  The oracle computes the full results on the host copy of the
same seeded graph (graphgen/, bit-identical to the device generator), so the comparison is
element by element: bit-exact for BFS/SSSP/CC/SSWP, max |diff| <= 1e-6 for PageRank."""
import numpy as np
import pytest

import graphgen
import oracle

torch = pytest.importorskip("torch")
pytestmark = [pytest.mark.gpu, pytest.mark.slow]


@pytest.fixture(scope="module")
def tigr():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_asplos_sabetq018_b200 as t
    return t


@pytest.fixture(scope="module")
def cfg4():
    rec = graphgen.recipe("cfg4")
    src, dst, w = graphgen.generate(rec)
    return rec, src, dst, w


def test_cfg4_pagerank_full(tigr, cfg4):
    """The bench workload itself: R-MAT scale 24, PageRank 20 iterations, K=8 strided."""
    rec, src, dst, _ = cfg4
    g = tigr.tigr_graph_rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, weighted=False)
    vg = tigr.tigr_virtualize(g, 8, "strided")
    got = tigr.tigr_run(vg, "pr")
    want = oracle.pagerank(oracle.csr_build(rec.n, src, dst), 20)
    err = np.abs(got - want).max()
    assert err <= 1e-6, err
    # normalised error too (values are ~6e-8, so also demand relative agreement)
    assert np.abs(rec.n * got - rec.n * want).max() <= 1e-6


def test_cfg4_host_input_e2e_path(tigr, cfg4):
    """bench.py's e2e path at full size: the pinned host arc list through tigr_graph_from_coo
    (16 copy chunks sorted as they land, merged by k_place_runs) gives the oracle's CSR element
    by element, and PageRank with the ranks written to a pinned host array matches the oracle."""
    rec, src, dst, _ = cfg4
    hs = torch.from_numpy(src.view(np.int32)).pin_memory()
    hd = torch.from_numpy(dst.view(np.int32)).pin_memory()
    g = tigr.tigr_graph_from_coo(rec.n, hs, hd, None)
    rp, col, _ = tigr.tigr_graph_export_csr(g)
    o = oracle.csr_build(rec.n, src, dst)
    assert np.array_equal(rp, o.row_ptr) and np.array_equal(col, o.col)
    vg = tigr.tigr_virtualize(g, 8, "strided")
    hout = torch.empty(rec.n, dtype=torch.float64).pin_memory()
    tigr.tigr_run(vg, "pr", out=hout)
    assert float(np.abs(hout.numpy() - oracle.pagerank(o, 20)).max()) <= 1e-6


def test_cfg4_frontier_algorithms_full(tigr, cfg4):
    rec, src, dst, w = cfg4
    g = tigr.tigr_graph_rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, rec.wmin, rec.wmax,
                             weighted=True)
    vg = tigr.tigr_virtualize(g, 8, "strided")
    o = oracle.csr_build(rec.n, src, dst, w)
    assert np.array_equal(tigr.tigr_run(vg, "bfs", 0), oracle.bfs(o, 0))
    assert np.array_equal(tigr.tigr_run(vg, "sssp", 0), oracle.sssp(o, 0))
    assert np.array_equal(tigr.tigr_run(vg, "sswp", 0), oracle.sswp(o, 0))
    del vg, g, o
    gs = tigr.tigr_graph_rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, weighted=False,
                              symmetrize=True)
    vgs = tigr.tigr_virtualize(gs, 8, "strided")
    assert np.array_equal(tigr.tigr_run(vgs, "cc"), oracle.cc(rec.n, src, dst))


@pytest.mark.parametrize("K", [4, 8, 16, 32])
def test_cfg3_sssp_sswp_k_sweep(tigr, K, cfg3_oracle):
    rec, want_sssp, want_sswp = cfg3_oracle
    g = tigr.tigr_graph_rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, rec.wmin, rec.wmax,
                             weighted=True)
    vg = tigr.tigr_virtualize(g, K, "strided")
    assert np.array_equal(tigr.tigr_run(vg, "sssp", rec.source), want_sssp)
    assert np.array_equal(tigr.tigr_run(vg, "sswp", rec.source), want_sswp)


@pytest.fixture(scope="module")
def cfg3_oracle():
    rec = graphgen.recipe("cfg3")
    src, dst, w = graphgen.generate(rec)
    o = oracle.csr_build(rec.n, src, dst, w)
    return rec, oracle.sssp(o, rec.source), oracle.sswp(o, rec.source)


def test_cfg4_pagerank_k_and_layout_invariance(tigr, cfg4):
    """Thm. 2: the virtual split does not change the result (PR up to summation order)."""
    rec = cfg4[0]
    g = tigr.tigr_graph_rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, weighted=False)
    ref = tigr.tigr_run(tigr.tigr_virtualize(g, 8, "strided"), "pr")
    for K, lay in ((4, "strided"), (32, "consecutive"), (0xFFFFFFFF, "strided")):
        got = tigr.tigr_run(tigr.tigr_virtualize(g, K, lay), "pr")
        assert np.abs(got - ref).max() <= 1e-12, (K, lay)


def test_cfg5_twitter_shaped_full(tigr):
    """Config 5 (41.7M vertices, 1.47B arcs, 2.94B symmetrised) on ONE B200: BFS, SSSP and CC
    element by element against the oracle on the host copy of the same graph (~2.5 min, of
    which ~2.2 min are host-side generation + oracle)."""
    rec = graphgen.recipe("cfg5")
    g = tigr.tigr_graph_rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, rec.wmin, rec.wmax,
                             weighted=True)
    vg = tigr.tigr_virtualize(g, 8, "strided")
    got_bfs = tigr.tigr_run(vg, "bfs", rec.source)
    got_sssp = tigr.tigr_run(vg, "sssp", rec.source)
    del vg, g
    gs = tigr.tigr_graph_rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, weighted=False,
                              symmetrize=True)
    vgs = tigr.tigr_virtualize(gs, 8, "strided")
    got_cc = tigr.tigr_run(vgs, "cc")
    del vgs, gs
    src, dst, w = graphgen.generate(rec)
    o = oracle.csr_build(rec.n, src, dst, w)
    assert np.array_equal(got_bfs, oracle.bfs(o, rec.source))
    assert np.array_equal(got_sssp, oracle.sssp(o, rec.source))
    del o
    assert np.array_equal(got_cc, oracle.cc(rec.n, src, dst))


def test_cfg4_pull_pagerank_full(tigr, cfg4):
    """NEXT-1 at the bench's size: pull PageRank on the in-CSR of R-MAT scale 24, K=8 strided."""
    rec, src, dst, _ = cfg4
    g = tigr.tigr_graph_rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, weighted=False)
    gt = tigr.tigr_graph_transpose(g)
    del g
    got = tigr.tigr_run(tigr.tigr_virtualize(gt, 8, "strided"), "pr")
    want = oracle.pagerank(oracle.csr_build(rec.n, src, dst), 20)
    assert np.abs(got - want).max() <= 1e-6
    assert np.abs(rec.n * got - rec.n * want).max() <= 1e-6


def _export_csr_device(tigr, g):
    """row_ptr / col / w of a graph as CUDA tensors (tigr_graph_export_csr to device buffers)."""
    info = g.info()
    rp = torch.empty(info["n"] + 1, dtype=torch.int64, device="cuda")
    col = torch.empty(max(info["m"], 1), dtype=torch.int32, device="cuda")
    w = torch.empty_like(col) if info["weighted"] else None
    tigr._check(tigr._lib.tigr_graph_export_csr(g.ptr, rp.data_ptr(), col.data_ptr(),
                                                None if w is None else w.data_ptr(), 1, None))
    torch.cuda.synchronize()
    return rp, col, w


def test_cfg5_host_input_sorted_runs(tigr):
    """Config 5's 1.47 B weighted arcs from pinned host memory: 64 copy chunks of 23 M arcs, each
    radix-sorted as it lands, merged into the rows by row-space windows (sort.cu
    build_sorted_runs) -- row_ptr, targets and weights equal element by element to the
    device-input build (whose BFS, SSSP and CC are oracle-exact at this size, test_cfg5_twitter_shaped_full)."""
    rec = graphgen.recipe("cfg5")
    src = torch.empty(rec.m, dtype=torch.int32, device="cuda")
    dst, w = torch.empty_like(src), torch.empty_like(src)
    tigr.tigr_rmat_coo(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, rec.wmin, rec.wmax, src, dst, w)
    gd = tigr.tigr_graph_from_coo(rec.n, src, dst, w)
    want = _export_csr_device(tigr, gd)
    gd.free()
    hs, hd, hw = src.cpu().pin_memory(), dst.cpu().pin_memory(), w.cpu().pin_memory()
    del src, dst, w
    torch.cuda.empty_cache()
    gh = tigr.tigr_graph_from_coo(rec.n, hs, hd, hw)
    got = _export_csr_device(tigr, gh)
    gh.free()
    for a, b in zip(got, want):
        assert torch.equal(a, b)
