"""Host input generator (graphgen/): Philox KAT, determinism, R-MAT shape.

The generator is an input recipe, not the paper's method; these tests pin it so
that the oracle's inputs are what DESIGN.md says they are.
"""
import numpy as np
import pytest

import graphgen


def test_philox_known_answers(golden):
    for vec in golden("philox_kat.json")["vectors"]:
        ctr = [int(x, 16) for x in vec["ctr"]]
        key = [int(x, 16) for x in vec["key"]]
        assert graphgen.philox4x32_10(ctr, key) == tuple(int(x, 16) for x in vec["out"])


def test_rmat_deterministic_and_thread_invariant():
    a = graphgen.rmat(1000, 20000, 0.57, 0.19, 0.19, seed=11, wseed=12, threads=1)
    b = graphgen.rmat(1000, 20000, 0.57, 0.19, 0.19, seed=11, wseed=12, threads=7)
    for x, y in zip(a, b):
        assert np.array_equal(x, y)
    # a prefix of a longer draw is the shorter draw (counter-based: edge e depends on e only)
    c = graphgen.rmat(1000, 5000, 0.57, 0.19, 0.19, seed=11, wseed=12)
    for x, y in zip(a, c):
        assert np.array_equal(x[:5000], y)


def test_rmat_ranges_and_rejection():
    n = 1000  # not a power of two: rejection from s = 10
    src, dst, w = graphgen.rmat(n, 50000, 0.48, 0.21, 0.21, seed=3, wseed=4, wmin=1, wmax=64)
    assert src.max() < n and dst.max() < n
    assert w.min() >= 1 and w.max() <= 64
    assert len(np.unique(w)) == 64
    s2, d2, w2 = graphgen.rmat(n, 100, 0.48, 0.21, 0.21, seed=3, wseed=4, weighted=False)
    assert w2 is None and np.array_equal(s2, src[:100])


def test_rmat_quadrant_rule_single_level():
    # n = 2: one level; with a=1 every edge is (0,0); with b=1 (0,1); c=1 (1,0); d=1 (1,1)
    for (a, b, c), want in [((1, 0, 0), (0, 0)), ((0, 1, 0), (0, 1)), ((0, 0, 1), (1, 0)),
                            ((0, 0, 0), (1, 1))]:
        s, d, _ = graphgen.rmat(2, 64, a, b, c, seed=5, weighted=False)
        assert (s == want[0]).all() and (d == want[1]).all()


def test_rmat_quadrant_frequencies():
    # n = 2: P(src=1) = c + d, P(dst=1) = b + d
    s, d, _ = graphgen.rmat(2, 200000, 0.57, 0.19, 0.19, seed=9, weighted=False)
    assert abs(s.mean() - 0.24) < 0.005
    assert abs(d.mean() - 0.24) < 0.005
    assert abs(((s == 1) & (d == 1)).mean() - 0.05) < 0.003


def test_cfg1_shape():
    # SURVEY.md Appendix A [sim]: deg(0) ~ 1,030, ~21% zero out-degree, ~26% duplicate arcs
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    assert len(src) == 16384
    deg = np.bincount(src, minlength=rec.n)
    assert deg.argmax() == 0 and 900 < deg[0] < 1200
    assert 0.17 < (deg == 0).mean() < 0.26
    dup = 1 - len(np.unique(src.astype(np.int64) * rec.n + dst)) / len(src)
    assert 0.2 < dup < 0.32
    # expected top out-degree ~ m (a+b)^s = 16384 * 0.76^10
    assert abs(deg[0] / (16384 * 0.76 ** 10) - 1) < 0.1
