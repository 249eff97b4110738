"""GPU parity of tile-shape variants the default build does not exercise.

The one-level merge pass cuts every pair of runs (width 2w) into
ceil(2w / tout) output tiles, the last one short (PairGeom.tile_of).  With the
default shapes tout divides 2w; this builds the library with 160-thread merge
CTAs (tout = 160 x 51 = 8160, 2 x 25088 / 8160 = 6.1) and checks the one-level
schedule bit-exactly against the oracle in a subprocess bound to that build.
"""
import os
import subprocess
import sys

import pytest
import torch

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SCRIPT = r"""
import sys
import numpy as np
import torch
sys.path.insert(0, {root!r})
import dcgen, oracle
import paper_conf_ipps_lopez_ortizss13_b200 as dc
oracle.build()
p0 = dc.Plan(1 << 23)
p0.set_tile_class(2)
sch = p0.schedule("u32")
assert sch["tile"] == 25088, sch
for n, dist, kt, vals in [((1 << 23) + 12345, "uniform", "u32", False),
                          (2 * 25088 * 5 + 7, "few", "u32", False),
                          ((1 << 23) + 99, "uniform", "i32", False),
                          ((1 << 23) + 5, "few", "u32", True)]:
    keys = dcgen.sort_keys(n, dist, seed=41, key_type=kt, device="cuda")
    v = dcgen.sort_vals(n, device="cuda") if vals else None
    ka = keys.cpu().numpy()
    ka = ka.view(np.uint32) if kt == "u32" else ka.view(np.int32)
    if vals:
        ek, ev = oracle.mergesort(ka, v.cpu().numpy().view(np.uint32), key_type=kt)
    else:
        ek = oracle.mergesort(ka, key_type=kt)
    plan = dc.Plan(n)
    plan.set_tile_class(2)
    plan.set_two_level(False)
    plan.sort_(keys, v, key_type=kt)
    torch.cuda.synchronize()
    got = keys.cpu().numpy().view(ek.dtype)
    assert np.array_equal(got, ek), (n, dist, kt)
    if vals:
        assert np.array_equal(v.cpu().numpy().view(np.uint32), ev), (n, dist, kt)
print("variant ok")
"""


def test_one_level_tiles_not_dividing_pairs(tmp_path):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_lopez_ortizss13_b200 import build

    lib = build.build(out=str(tmp_path / "libdc_nt160.so"),
                      defines=["DC_FAST_NT3=160", "DC_STABLE_NT3=160"])
    env = dict(os.environ, DC_LIB=lib)
    r = subprocess.run([sys.executable, "-c", SCRIPT.format(root=ROOT)], env=env,
                       capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-4000:]
    assert "variant ok" in r.stdout


VONLY_SCRIPT = r"""
import sys
import numpy as np
import torch
sys.path.insert(0, {root!r})
import dcgen, oracle
import paper_conf_ipps_lopez_ortizss13_b200 as dc
oracle.build()
cases = []
for n in [1, 67, 68, 69, 2176, 2177, 70_001, 1 << 20, (1 << 24) + 3]:
    for lo in (-1, -2):
        g = torch.Generator().manual_seed(n * 7 + lo)
        cases.append(torch.randint(lo, 2, (n,), generator=g, dtype=torch.int32))
for n, dist in [(1 << 24, "uniform"), ((1 << 20) + 5, "small"), (777, "negative"),
                (1 << 16, "zero"), (100_003, "positive")]:
    cases.append(dcgen.maxsub_input(n, dist, seed=2))
for x in cases:
    n = x.numel()
    assert dc.Plan(n).max_subarray(x.cuda()) == oracle.maxsub(x.numpy()), n
    tup = torch.empty(8, dtype=torch.int64, device="cuda")
    dc.Plan(n).max_subarray_tuple_async(x.cuda(), tup, index_offset=5)
    t = tup.cpu().tolist()
    a = x.numpy().astype(np.int64)
    pre = np.cumsum(a)
    suf = np.cumsum(a[::-1])[::-1]
    s, b, e = oracle.maxsub(x.numpy())
    assert t == [int(a.sum()), int(pre.max()), int(suf.max()), s,
                 int(np.argmax(pre)) + 5, int(np.argmax(suf)) + 5, b + 5, e + 5], (n, t)
print("variant ok")
"""


def test_maxsub_values_only_fold(tmp_path):
    """NK4 with the indexed element fold (-DDC_MS_VONLY=0, L = 68: the r02
    default; the default build now folds values only and recovers indices from
    chunk labels, R21): bit-exact (sum, start, end) and summary
    tuple on tie-heavy and degenerate inputs."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_lopez_ortizss13_b200 import build

    lib = build.build(out=str(tmp_path / "libdc_indexed.so"), defines=["DC_MS_VONLY=0", "DC_MS_P=68"])
    env = dict(os.environ, DC_LIB=lib)
    r = subprocess.run([sys.executable, "-c", VONLY_SCRIPT.format(root=ROOT)], env=env,
                       capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-4000:]
    assert "variant ok" in r.stdout


def test_maxsub_rows_kernel(tmp_path):
    """NK4 with one contiguous row per lane fed by 2-D TMA tensor copies
    (-DDC_MS_ROWS=1, maxsub_rows.cuh): bit-exact (sum, start, end) and summary
    tuple on tie-heavy, degenerate and ragged-tail inputs."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_lopez_ortizss13_b200 import build

    lib = build.build(out=str(tmp_path / "libdc_rows.so"), defines=["DC_MS_ROWS=1"])
    env = dict(os.environ, DC_LIB=lib)
    r = subprocess.run([sys.executable, "-c", VONLY_SCRIPT.format(root=ROOT)], env=env,
                       capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-4000:]
    assert "variant ok" in r.stdout

