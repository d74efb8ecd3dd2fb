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


NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _nccl_include() -> list[str]:
    cands = ["/opt/prime-rl/.venv/lib/python3.12/site-packages/nvidia/nccl/include", "/usr/include"]
    for c in cands:
        if os.path.exists(os.path.join(c, "nccl.h")):
            return ["-I", c]
    return []


def build_tigr(force: bool = False, verbose: bool = False, dev: bool = False) -> str:
    """nvcc -gencode arch=compute_100a,code=sm_100a every csrc/*.cu -> libtigr.so (in-tree).

    dev=True builds build/libtigr_dev.so with -DTIGR_DEV_KNOBS (the TIGR_* development knobs of
    DESIGN.md §10c read from the environment; load it with TIGR_LIB for A/B sweeps)."""
    from concurrent.futures import ThreadPoolExecutor

    pkg = os.path.join(ROOT, "paper_conf_asplos_sabetq018_b200")
    csrc = os.path.join(pkg, "csrc")
    target = os.path.join(ROOT, "build", "libtigr_dev.so") if dev else os.path.join(pkg, "libtigr.so")
    objdir = os.path.join(ROOT, "build", "obj_dev" if dev else "obj")
    os.makedirs(objdir, exist_ok=True)
    sources = sorted(os.path.join(csrc, f) for f in os.listdir(csrc) if f.endswith(".cu"))
    headers = sorted(os.path.join(csrc, f) for f in os.listdir(csrc) if f.endswith((".cuh", ".h")))
    headers.append(os.path.join(ROOT, "include", "tigr.h"))
    flags = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xcompiler", "-Wall",
             "--expt-relaxed-constexpr", "--extended-lambda", *ARCH, "-I", os.path.join(ROOT, "include"),
             *_nccl_include()]
    if dev:
        flags += ["-DTIGR_DEV_KNOBS"]
    if os.environ.get("TIGR_PTXAS_VERBOSE"):
        flags += ["-Xptxas", "-v"]

    def compile_one(src):
        obj = os.path.join(objdir, os.path.basename(src)[:-3] + ".o")
        if force or _stale(obj, [src, *headers]):
            cmd = [NVCC, *flags, "-c", src, "-o", obj]
            if verbose:
                print(" ".join(cmd), flush=True)
            subprocess.run(cmd, check=True)
        return obj

    with ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 1)) as ex:
        objs = list(ex.map(compile_one, sources))
    if force or _stale(target, objs):
        cmd = [NVCC, *ARCH, "-shared", "-o", target + ".tmp", *objs, "-ldl"]
        subprocess.run(cmd, check=True)
        os.replace(target + ".tmp", target)
    return target


def build_micro(force: bool = False) -> str:
    """tools/micro/gather_ceiling.cu -> build/libmicro.so (measurement helper bench.py loads;
    not part of the product library)."""
    src = os.path.join(ROOT, "tools", "micro", "gather_ceiling.cu")
    target = os.path.join(ROOT, "build", "libmicro.so")
    os.makedirs(os.path.dirname(target), exist_ok=True)
    if force or _stale(target, [src]):
        subprocess.run([NVCC, "-O3", "-lineinfo", *ARCH, "-Xcompiler", "-fPIC", "-shared", src, "-o", target + ".tmp"],
                       check=True)
        os.replace(target + ".tmp", target)
    return target


if __name__ == "__main__":
    sys.path.insert(0, ROOT)
    import __graft_entry__  # noqa: E402

    __graft_entry__.build()
    if "--dev" in sys.argv:
        build_tigr(dev=True)
