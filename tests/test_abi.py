"""C-ABI checks that need no GPU: the library loads, exports every symbol include/tigr.h
declares, and fails loudly (TIGR_ECUDA, no CPU fallback) when no device is present."""
import ctypes
import os
import re
import subprocess

import pytest

from tests.conftest import ROOT

HEADER = os.path.join(ROOT, "include", "tigr.h")


def _declared():
    txt = open(HEADER).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(tigr_[a-z_]+)\s*\(", txt)))


def test_header_declares_the_boundary():
    names = _declared()
    for must in ("tigr_graph_from_csr", "tigr_graph_from_coo", "tigr_virtualize", "tigr_run",
                 "tigr_comm_init", "tigr_last_error"):
        assert must in names


def test_library_exports_every_declared_symbol():
    import paper_conf_asplos_sabetq018_b200 as tigr
    out = subprocess.run(["nm", "-D", "--defined-only", tigr.LIB_PATH], capture_output=True, text=True,
                         check=True).stdout
    exported = set(re.findall(r" T (tigr_\w+)", out))
    missing = [s for s in _declared() if s not in exported]
    assert not missing, missing
    assert set(tigr.EXPORTED_SYMBOLS) <= exported


def test_library_built_for_sm100a():
    import paper_conf_asplos_sabetq018_b200 as tigr
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", tigr.LIB_PATH],
                         capture_output=True, text=True, check=True).stdout
    assert "sm_100a" in out


def test_product_does_not_import_oracle():
    """The product path never imports, links or loads oracle/ (or the host generator)."""
    pkg = os.path.join(ROOT, "paper_conf_asplos_sabetq018_b200")
    bad = re.compile(r"^\s*(import\s+(oracle|graphgen)\b|from\s+(oracle|graphgen)\b)|"
                     r"#\s*include\s*[<\"][^>\"]*(oracle|graphgen)|liboracle|libgraphgen", re.M)
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dirpath, f)).read()
                assert not bad.search(txt), f


def test_no_device_fails_loudly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    import paper_conf_asplos_sabetq018_b200 as tigr
    with pytest.raises(tigr.TigrError) as ei:
        tigr.tigr_graph_from_coo(4, [0, 1], [1, 2])
    assert ei.value.status == tigr.TIGR_ECUDA
    with pytest.raises(tigr.TigrError):
        tigr.tigr_graph_rmat(1024, 100, 0.57, 0.19, 0.19, 1)


def test_opts_default_and_version():
    import paper_conf_asplos_sabetq018_b200 as tigr
    o = tigr.tigr_run_opts_default()
    assert o.pr_iters == 20 and abs(o.pr_damping - 0.85) < 1e-15 and o.use_graph == 1
    assert o.exchange == tigr.TIGR_EXCHANGE_AUTO
    assert "sm_100a" in tigr.tigr_version()
    # the ctypes mirrors of the option / stats structs match the C layout of include/tigr.h
    os.makedirs(os.path.join(ROOT, "build"), exist_ok=True)
    src = os.path.join(ROOT, "build", "abi_sizes.c")
    exe = os.path.join(ROOT, "build", "abi_sizes")
    with open(src, "w") as f:
        f.write('#include <stdio.h>\n#include <stddef.h>\n#include "tigr.h"\n'
                'int main(void){printf("%zu %zu %zu %zu %zu %zu\\n", sizeof(tigr_run_opts), sizeof(tigr_stats),'
                ' offsetof(tigr_run_opts, exchange), offsetof(tigr_stats, sparse_exchanges),'
                ' offsetof(tigr_run_opts, frontier_div), offsetof(tigr_stats, bytes_alg));return 0;}\n')
    subprocess.run(["gcc", "-std=c11", "-I", os.path.join(ROOT, "include"), src, "-o", exe], check=True)
    sizes = [int(x) for x in subprocess.run([exe], check=True, capture_output=True, text=True).stdout.split()]
    assert sizes == [ctypes.sizeof(tigr.tigr_run_opts), ctypes.sizeof(tigr.tigr_stats),
                     tigr.tigr_run_opts.exchange.offset, tigr.tigr_stats.sparse_exchanges.offset,
                     tigr.tigr_run_opts.frontier_div.offset, tigr.tigr_stats.bytes_alg.offset]


def _build_c_example():
    import paper_conf_asplos_sabetq018_b200 as tigr
    os.makedirs(os.path.join(ROOT, "build"), exist_ok=True)
    exe = os.path.join(ROOT, "build", "c_abi_bfs")
    libdir = os.path.dirname(tigr.LIB_PATH)
    subprocess.run(["gcc", "-std=c11", "-Wall", "-Werror", "-I", os.path.join(ROOT, "include"),
                    os.path.join(ROOT, "examples", "c_abi_bfs.c"), "-L", libdir, "-ltigr",
                    f"-Wl,-rpath,{libdir}", "-o", exe], check=True)
    return exe


def test_c_program_against_header_host_only():
    """A plain C program compiled against include/tigr.h links libtigr.so and runs the
    host-only entry points; compute calls report TIGR_ECUDA without a GPU."""
    import torch
    exe = _build_c_example()
    if torch.cuda.is_available():
        pytest.skip("GPU present: covered by the GPU variant")
    r = subprocess.run([exe], capture_output=True, text=True)
    assert r.returncode == 0, r.stdout + r.stderr


@pytest.mark.gpu
def test_c_program_against_header_gpu():
    exe = _build_c_example()
    r = subprocess.run([exe, "--gpu"], capture_output=True, text=True)
    assert r.returncode == 0, r.stdout + r.stderr
    assert "GPU checks ok" in r.stdout
