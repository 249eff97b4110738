"""the D&C sum (Alg 4/5) and the generic O(1)-combine template.

* dc_run_sum (Alg 4 through include/dc_reduce.cuh) and dc_run_sum_alg5 (the
  paper's Alg 5 GPU code: one launch per level, a[id] += a[id+m]) against the
  oracle's recursive Alg 4 sum, exactly.
* User code instantiating dc_reduce.cuh with two NON-commutative monoids
  (max-subarray tuples, a polynomial hash), compiled here with nvcc, against
  the CPU oracle / an exact Python fold.
"""
import ctypes
import os
import subprocess

import numpy as np
import pytest
import torch

import dcgen

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def dc():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ipps_lopez_ortizss13_b200 as m
    return m


SUM_SIZES = [1, 2, 3, 7, 1000, 8191, 8192, 8193, 17407, 17408, 17409, 100_003, 1 << 20,
             (1 << 24) + 17]


@pytest.mark.parametrize("n", SUM_SIZES)
@pytest.mark.parametrize("dist", ["uniform", "negative"])
def test_dc_sum_matches_alg4_oracle(dc, oracle_mod, n, dist):
    x = dcgen.maxsub_input(n, dist, seed=3, device="cuda")
    expect = oracle_mod.dc_sum(x.cpu().numpy())
    plan = dc.Plan(n)
    assert plan.sum(x) == expect
    assert plan.sum(x) == expect                      # re-armed ticket
    work = x.to(torch.int64)
    assert plan.sum_alg5(work) == expect             # the paper's per-level kernels


@pytest.fixture(scope="module")
def demo():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    out = "/tmp/dc_generic_demo.so"
    src = os.path.join(ROOT, "tests", "cuda", "generic_reduce_demo.cu")
    subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3",
                           "-std=c++17", "-shared", "-Xcompiler", "-fPIC", "-I",
                           os.path.join(ROOT, "include"), "-o", out, src])
    lib = ctypes.CDLL(out)
    for f in (lib.demo_maxsub, lib.demo_hash, lib.demo_maxsub_tma, lib.demo_hash_tma):
        f.argtypes = [ctypes.c_void_p, ctypes.c_longlong, ctypes.c_void_p, ctypes.c_void_p,
                      ctypes.c_void_p]
        f.restype = ctypes.c_int
    return lib


def _bufs(words_per_t):
    parts = torch.zeros(300 * words_per_t, dtype=torch.int64, device="cuda")
    ticket = torch.zeros(2, dtype=torch.int64, device="cuda")
    out = torch.zeros(words_per_t, dtype=torch.int64, device="cuda")
    return parts, ticket, out


@pytest.mark.parametrize("kernel", ["plain", "tma"])
@pytest.mark.parametrize("n", [1, 5, 2047, 2048, 2049, 4607, 4608, 4609, 100_003, 1 << 20])
def test_generic_template_maxsub_monoid(oracle_mod, demo, n, kernel):
    x = dcgen.maxsub_input(n, "small", seed=9, device="cuda")
    parts, ticket, out = _bufs(8)
    f = demo.demo_maxsub if kernel == "plain" else demo.demo_maxsub_tma
    assert f(x.data_ptr(), n, parts.data_ptr(), ticket.data_ptr(), out.data_ptr()) == 0
    t = out.cpu().tolist()
    assert (t[3], t[6], t[7]) == oracle_mod.maxsub(x.cpu().numpy())


@pytest.mark.parametrize("kernel", ["plain", "tma"])
@pytest.mark.parametrize("n", [1, 33, 4096, 77_777, 1 << 20])
def test_generic_template_hash_monoid(demo, n, kernel):
    x = dcgen.maxsub_input(n, "uniform", seed=10, device="cuda")
    parts, ticket, out = _bufs(2)
    f = demo.demo_hash if kernel == "plain" else demo.demo_hash_tma
    assert f(x.data_ptr(), n, parts.data_ptr(), ticket.data_ptr(), out.data_ptr()) == 0
    got = int(out.cpu()[0]) & ((1 << 64) - 1)
    m = (1 << 64) - 1
    h = 0
    for v in x.cpu().numpy().view(np.uint32).tolist():   # exact left-to-right fold
        h = (h * 1000003 + v) & m
    assert got == h
