"""CPU-side checks of the C ABI: the library builds for sm_100a, loads, exports every symbol
include/buffalo.h declares, its pure-host memory model (buffalo_estimate_mem, R15) equals the
oracle's restatement, and the CUDA Philox (csrc/philox.cuh, compiled for the host) matches the
Random123 known-answer vectors.  No compute call needs a GPU here."""
import os
import re
import subprocess

import numpy as np
import pytest

from conftest import ROOT, read_golden
import oracle as O


@pytest.fixture(scope="module")
def blib():
    from paper_conf_hpca_yangzl25_b200 import build_lib
    build_lib.build()
    from paper_conf_hpca_yangzl25_b200 import buffalo as B
    return B


def _declared():
    txt = open(os.path.join(ROOT, "include", "buffalo.h")).read()
    return sorted(set(re.findall(r"BUFFALO_API\s+[\w\s\*]+?\b(buffalo_\w+)\s*\(", txt)))


def test_exports_every_declared_symbol(blib):
    names = _declared()
    assert len(names) >= 15
    L = blib.lib(require_gpu=False)
    for n in names:
        assert hasattr(L, n), n
    assert set(names) == set(blib.EXPORTS)
    nm = subprocess.run(["nm", "-D", "--defined-only", blib.LIB_PATH], capture_output=True, text=True).stdout
    for n in names:
        assert re.search(rf"\sT\s{n}$", nm, re.M), n


def test_library_is_sm100a_only(blib):
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", blib.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out and "sm_90" not in out


@pytest.mark.parametrize("gemm,agg", [(0, 0), (1, 0), (0, 1), (0, 2), (0, 3)])
def test_estimate_mem_equals_oracle(blib, gemm, agg):
    rng = np.random.default_rng(gemm + 7 * agg)
    for _ in range(200):
        L = int(rng.integers(1, 4))
        dims = [int(x) for x in rng.integers(1, 600 if not gemm else 257, L + 1)]
        dims[0] = int(rng.integers(1, 2000))
        n = [int(x) for x in rng.integers(0, 300000, L + 1)]
        e = [int(x) for x in rng.integers(0, 3000000, L)]
        m = blib.make_model(dims, gemm_mode=gemm, aggregator=agg)
        assert blib.estimate_mem(n, e, m) == O.mem_model(n, e, dims, O.BF16 if gemm else O.FP32,
                                                         ("mean", "pool", "lstm", "gat")[agg])


def test_estimate_mem_sharded_equals_oracle(blib):
    """The sharded-feature-table model (bf16, SAGE-mean) adds block 1's self-row copy."""
    rng = np.random.default_rng(99)
    sh = blib.make_shards([1 << 20, 2 << 20, 3 << 20], 1000)        # pointers are not dereferenced here
    for _ in range(100):
        L = int(rng.integers(1, 4))
        dims = [int(x) for x in rng.integers(1, 257, L + 1)]
        dims[0] = int(rng.integers(1, 2000))
        n = [int(x) for x in rng.integers(0, 300000, L + 1)]
        e = [int(x) for x in rng.integers(0, 3000000, L)]
        m = blib.make_model(dims, feat_dtype=1, gemm_mode=1, shards=sh)
        assert blib.estimate_mem(n, e, m) == O.mem_model(n, e, dims, O.BF16, sharded=True)
        assert blib.estimate_mem(n, e, m)[0] > O.mem_model(n, e, dims, O.BF16)[0] or n[1] == 0


def test_cuda_philox_known_answers(tmp_path):
    src = tmp_path / "kat.cu"
    src.write_text('#include <cstdio>\n#include "philox.cuh"\nint main(){unsigned v[6];\n'
                   'while(scanf("%x %x %x %x %x %x",&v[0],&v[1],&v[2],&v[3],&v[4],&v[5])==6){\n'
                   'auto o=buffalo::philox4x32_10({v[0],v[1],v[2],v[3]},v[4],v[5]);\n'
                   'printf("%08x %08x %08x %08x\\n",o.x,o.y,o.z,o.w);}}\n')
    exe = tmp_path / "kat"
    inc = os.path.join(ROOT, "paper_conf_hpca_yangzl25_b200", "csrc")
    subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-std=c++17", "-I", inc, str(src), "-o", str(exe)])
    rows = [ln.split() for ln in read_golden("philox_kat.txt")]
    inp = "\n".join(" ".join(r[:6]) for r in rows) + "\n"
    out = subprocess.run([str(exe)], input=inp, capture_output=True, text=True).stdout.split("\n")
    for r, o in zip(rows, out):
        assert o.split() == r[6:10]
