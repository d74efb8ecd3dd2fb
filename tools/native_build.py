"""Build helpers for the host-side C libraries (graphgen/, oracle/) and the CUDA
product library.  Plain subprocess calls to gcc / nvcc; no torch extension
machinery, so the built .so files live in-tree and travel with gpurun.
"""
from __future__ import annotations

import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _stale(target: str, sources: list[str]) -> bool:
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(s) > t for s in sources)


def build_c_shared(sources: list[str], target: str, extra: list[str] | None = None,
                   force: bool = False) -> str:
    """gcc -O2 -shared -fPIC sources -o target (only when stale)."""
    if not force and not _stale(target, sources):
        return target
    cmd = ["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-Wall", "-Wextra",
           "-Wno-unused-parameter", *sources, "-o", target + ".tmp", "-lm"]
    if extra:
        cmd[1:1] = extra
    subprocess.run(cmd, check=True)
    os.replace(target + ".tmp", target)
    return target


if __name__ == "__main__":
    sys.path.insert(0, ROOT)
    import __graft_entry__  # noqa: E402

    __graft_entry__.build()
