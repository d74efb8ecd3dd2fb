"""The multi-core CPU baseline bench.py reports (tools/cpu_baseline/omp_pagerank.c, OpenMP pull
PageRank) computes the oracle's PageRank: same iteration, only the summation order differs."""
import os

import numpy as np
import pytest

import graphgen
import oracle
from tests.conftest import ROOT


@pytest.fixture(scope="module")
def omp():
    from tools.native_build import build_c_shared
    build_c_shared([os.path.join(ROOT, "tools", "cpu_baseline", "omp_pagerank.c")],
                   os.path.join(ROOT, "tools", "cpu_baseline", "libomp_pr.so"), extra=["-fopenmp"])
    from tools import cpu_baseline
    return cpu_baseline


@pytest.mark.parametrize("cfg", ["cfg1"])
def test_omp_pagerank_matches_oracle(omp, cfg):
    rec = graphgen.recipe(cfg)
    src, dst, w = graphgen.generate(rec)
    want = oracle.pagerank(oracle.csr_build(rec.n, src, dst, w), 20)
    for threads in (1, 4):
        got, _, _ = omp.omp_pagerank(rec.n, src, dst, 20, 0.85, threads)
        assert np.abs(got - want).max() <= 1e-15


def test_omp_pagerank_edge_graphs(omp):
    """No arcs (every rank (1-d)/n after the first iteration), a 3-cycle (uniform 1/3)."""
    got, _, _ = omp.omp_pagerank(5, np.zeros(0, np.uint32), np.zeros(0, np.uint32), 3, 0.85, 2)
    assert np.allclose(got, (1 - 0.85) / 5, rtol=0, atol=1e-17)
    got, _, _ = omp.omp_pagerank(3, np.array([0, 1, 2], np.uint32), np.array([1, 2, 0], np.uint32), 20, 0.85, 2)
    assert np.allclose(got, 1.0 / 3, rtol=0, atol=1e-15)


@pytest.mark.parametrize("cfg", ["cfg1", "cfg2"])
def test_omp_bfs_matches_oracle(omp, cfg):
    rec = graphgen.recipe(cfg)
    src, dst, w = graphgen.generate(rec, weighted=(cfg == "cfg1"))
    want = oracle.bfs(oracle.csr_build(rec.n, src, dst, w), 0)
    for threads in (1, 4):
        got, _, _ = omp.omp_bfs(rec.n, src, dst, 0, threads)
        assert np.array_equal(got, want)
