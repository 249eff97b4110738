"""the paper's Sec. 5.2 work-division model (host-only, no GPU).

Pinned by the numbers the paper prints for its worked example (P:L709-718,
tests/golden/paper_numbers.json): mergesort, p = 4, g = 2^12, gamma = 1/160,
n = 2^24 -> alpha* ~ 0.16, the GPU does ~52 % of the work, level ~ 10.  The
library's C implementation (dc_model_*) is checked against that example and
against the oracle's literal Python transcription (oracle/planner.py) over a
range of alphas and both platforms of Table 2.
"""
import json
import math
import os

import pytest

import paper_conf_ipps_lopez_ortizss13_b200 as dc
from oracle import planner

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLD = json.load(open(os.path.join(ROOT, "tests", "golden", "paper_numbers.json")))


def _example():
    e = GOLD["model_example"]
    return e["a"], e["b"], e["p"], float(e["g"]), 1.0 / e["gamma_inv"], float(e["n"]), e


def test_oracle_reproduces_paper_example():
    a, b, p, g, gamma, n, e = _example()
    r = planner.optimise(a, b, p, g, gamma, n)
    assert abs(r["alpha"] - e["alpha_star"]) < 0.01
    assert abs(r["gpu_work_fraction"] - e["gpu_work_fraction"]) < 0.01
    assert abs(r["level_y"] - e["level_y"]) < 1.0          # "approximately 10"
    # "the gpu is both saturated and non-saturated during its execution"
    assert r["case"] == 3 and r["level_y"] < math.log2(g)


def test_library_reproduces_paper_example():
    a, b, p, g, gamma, n, e = _example()
    r = dc.model_optimise(a, b, p, g, gamma, n)
    assert abs(r["alpha"] - e["alpha_star"]) < 0.01
    assert abs(r["gpu_work_fraction"] - e["gpu_work_fraction"]) < 0.01
    assert abs(r["level_y"] - e["level_y"]) < 1.0
    assert r["case"] == 3


@pytest.mark.parametrize("platform", ["HPU1", "HPU2"])
@pytest.mark.parametrize("alpha", [0.02, 0.05, 0.1, 0.16, 0.25, 0.5, 0.9])
@pytest.mark.parametrize("n", [2 ** 20, 2 ** 24, 10 ** 7])
def test_library_matches_oracle(platform, alpha, n):
    pl = GOLD["platforms"][platform]
    args = (2, 2, pl["p"], float(pl["g"]), 1.0 / pl["gamma_inv"], float(n))
    f, y, c = planner.gpu_work_fraction(*args, alpha)
    r = dc.model_gpu_work(*args, alpha)
    assert r["case"] == c
    assert math.isclose(r["gpu_work_fraction"], f, rel_tol=1e-9, abs_tol=1e-12)
    assert math.isclose(r["level_y"], y, rel_tol=1e-9, abs_tol=1e-9)


def test_model_properties():
    # more GPU cores or a faster GPU never lowers the optimal GPU share
    base = dc.model_optimise(2, 2, 4, 4096.0, 1 / 160, 2.0 ** 24)["gpu_work_fraction"]
    assert dc.model_optimise(2, 2, 4, 8192.0, 1 / 160, 2.0 ** 24)["gpu_work_fraction"] >= base
    assert dc.model_optimise(2, 2, 4, 4096.0, 1 / 80, 2.0 ** 24)["gpu_work_fraction"] >= base
    for alpha in (0.01, 0.3, 0.7):
        r = dc.model_gpu_work(2, 2, 4, 4096.0, 1 / 160, 2.0 ** 24, alpha)
        assert 0.0 <= r["gpu_work_fraction"] <= 1.0 - alpha + 1e-12


@pytest.mark.parametrize("args", [(1, 2, 4, 4096.0, 0.01, 2.0 ** 20, 0.1),
                                  (2, 2, 0, 4096.0, 0.01, 2.0 ** 20, 0.1),
                                  (2, 2, 4, 4096.0, 1.5, 2.0 ** 20, 0.1),
                                  (2, 2, 4, 4096.0, 0.01, 2.0 ** 20, 1.0)])
def test_model_validation(args):
    with pytest.raises(dc.DcError):
        dc.model_gpu_work(*args)
