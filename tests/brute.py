"""Brute-force checkers (tests only; numpy).  Independent of oracle/ and of the
CUDA path: they recompute each result from its mathematical definition on tiny
graphs (SURVEY.md §4 item 1, §8(c) pins)."""
import numpy as np

INF = 0xFFFFFFFF


def minplus_closure(n, src, dst, w):
    """Floyd-Warshall over (min, +): all-pairs shortest path sums (int64, inf = big)."""
    BIG = np.int64(1) << 60
    D = np.full((n, n), BIG, dtype=np.int64)
    np.fill_diagonal(D, 0)
    for s, d, x in zip(src, dst, w):
        D[s, d] = min(D[s, d], int(x))
    for k in range(n):
        D = np.minimum(D, D[:, k:k + 1] + D[k:k + 1, :])
    return D, BIG


def sssp(n, src, dst, w, source):
    D, BIG = minplus_closure(n, src, dst, w)
    row = D[source]
    return np.where(row >= BIG, INF, row).astype(np.uint32)


def bfs(n, src, dst, source):
    return sssp(n, src, dst, np.ones(len(src), dtype=np.int64), source)


def maxmin_closure(n, src, dst, w):
    """Floyd-Warshall over (max, min): widest-path widths; diagonal = +inf (empty path)."""
    W = np.zeros((n, n), dtype=np.int64)
    for s, d, x in zip(src, dst, w):
        W[s, d] = max(W[s, d], int(x))
    np.fill_diagonal(W, INF)
    for k in range(n):
        W = np.maximum(W, np.minimum(W[:, k:k + 1], W[k:k + 1, :]))
    return W


def sswp(n, src, dst, w, source):
    return maxmin_closure(n, src, dst, w)[source].astype(np.uint32)


def reach_closure(n, src, dst):
    """Boolean transitive-reflexive closure by repeated squaring."""
    R = np.eye(n, dtype=bool)
    R[np.asarray(src, dtype=np.int64), np.asarray(dst, dtype=np.int64)] = True
    while True:
        R2 = (R.astype(np.int32) @ R.astype(np.int32)) > 0
        if (R2 == R).all():
            return R
        R = R2


def cc(n, src, dst):
    """Weak CC: closure of the symmetrised graph; label = min id reachable."""
    s = np.concatenate([src, dst])
    d = np.concatenate([dst, src])
    R = reach_closure(n, s, d)
    return np.array([int(np.flatnonzero(R[v])[0]) for v in range(n)], dtype=np.uint32)


def pagerank_dense(n, src, dst, iters=20, damping=0.85, dangling=0):
    """x <- (1-d)/n + d * A^T D^+ x with a dense matrix (arcs with multiplicity)."""
    A = np.zeros((n, n))
    np.add.at(A, (np.asarray(src, np.int64), np.asarray(dst, np.int64)), 1.0)
    deg = A.sum(axis=1)
    P = np.divide(A, deg[:, None], out=np.zeros_like(A), where=deg[:, None] > 0)
    x = np.full(n, 1.0 / n)
    for _ in range(iters):
        extra = damping * x[deg == 0].sum() / n if dangling else 0.0
        x = (1 - damping) / n + damping * (P.T @ x) + extra
    return x
