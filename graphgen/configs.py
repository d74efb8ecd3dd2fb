"""Input recipes for BASELINE.json's five configs (SURVEY.md §8(d) "Synthetic inputs").

Shapes only: vertex/edge counts, R-MAT quadrant probabilities, seeds, weight
range, degree bound K and which algorithms run.  No method arithmetic.
"""
from __future__ import annotations

from dataclasses import dataclass, field

GRAPH500 = (0.57, 0.19, 0.19)


@dataclass(frozen=True)
class GraphRecipe:
    name: str
    n: int
    m: int
    a: float
    b: float
    c: float
    seed: int
    wseed: int
    wmin: int = 1
    wmax: int = 64
    weighted: bool = True
    K: tuple = (8,)
    algos: tuple = ()
    source: int = 0
    gpus: tuple = (1,)
    note: str = ""
    extra: dict = field(default_factory=dict)


CONFIGS = {
    # BASELINE.json configs[0]: "R-MAT scale 10 (1,024 vertices, 16K edges, int weights 1-64)
    # SSSP from vertex 0, K=8, 1 GPU"
    "cfg1": GraphRecipe("rmat-s10", 1 << 10, 16 << 10, *GRAPH500, seed=1, wseed=2,
                        K=(8,), algos=("sssp",)),
    # configs[1]: "R-MAT scale 20 (1M vertices, 16M edges) BFS + CC, K=8, 1 GPU"
    "cfg2": GraphRecipe("rmat-s20", 1 << 20, 16 << 20, *GRAPH500, seed=1, wseed=2,
                        K=(8,), algos=("bfs", "cc")),
    # configs[2]: "LiveJournal-shaped power-law graph (4.8M vertices, 69M edges) SSSP + SSWP,
    # K sweep 4-32" -- exact SNAP soc-LiveJournal1 counts, rejection sampling from s=23.
    "cfg3": GraphRecipe("lj-shaped", 4_847_571, 68_993_773, 0.48, 0.21, 0.21, seed=3, wseed=4,
                        K=(4, 8, 16, 32), algos=("sssp", "sswp")),
    # configs[3]: "R-MAT scale 24 (16M vertices, 268M edges) PageRank 20 iterations, 1/2/4/8 GPUs"
    "cfg4": GraphRecipe("rmat-s24", 1 << 24, 16 << 24, *GRAPH500, seed=5, wseed=6,
                        K=(8,), algos=("pr",), gpus=(1, 2, 4, 8)),
    # configs[4]: "Twitter-shaped power-law graph (41.7M vertices, 1.47B edges) BFS/SSSP/CC
    # across 8xB200" -- exact Kwak-2010 counts, rejection sampling from s=26.
    "cfg5": GraphRecipe("twitter-shaped", 41_652_230, 1_468_365_182, 0.55, 0.20, 0.20,
                        seed=7, wseed=8, K=(8,), algos=("bfs", "sssp", "cc"), gpus=(8,)),
}


def recipe(name: str) -> GraphRecipe:
    return CONFIGS[name]
