"""The paper's advanced hybrid work-division model (Sec. 5.2) -- TEST ORACLE.

Test infrastructure only (see oracle/__init__.py).  Literal transcription of
the closed forms of Sec. 5.2.2 for D&C algorithms whose divide +
combine at size m costs f(m) = m^{log_b a} (mergesort: a = b = 2, f(m) = m),
on an HPU with p CPU cores, g GPU "cores" and CPU/GPU speed ratio gamma
(Sec. 3.2).  Notation: N = n^{log_b a}, L = log_b n.

  Tc(alpha)    = alpha N / p * (L - log_a(p/alpha) + 1)
  Tmaxg(alpha) = (1-alpha) N / (gamma g) * (L - log_a(g/(1-alpha)) + 1)
  Tg(alpha, y) =
    (i)   (1/gamma) (N a/(a-1) a^-y - 1/(a-1))           if (1-alpha) N < g
    (ii)  (1-alpha) N / (gamma g) (L - y + 1)            if (1-alpha) N >= g, Tmaxg >= Tc
    (iii) Tmaxg + N a / (gamma (a-1)) (a^-y - (1-alpha)/g)  otherwise
  y(alpha): solve Tg(alpha, y) = Tc(alpha)
  Wg(alpha) = (1-alpha) N (L - y(alpha) + 1);  total work N (L + 1)

Reading (R20): in case (iii) the garbled "(a^-y - 1-alpha / g)" is
read as a^-y - (1-alpha)/g, the value at which the saturated and unsaturated
GPU phases meet; with it the printed example (alpha* ~ 0.16, GPU ~ 52 % of the
work, transfer level ~ 10) is reproduced.
"""
from __future__ import annotations

import math


def _log(x, base):
    return math.log(x) / math.log(base)


def terms(a, b, p, g, gamma, n, alpha):
    N = n ** _log(a, b)
    L = _log(n, b)
    Tc = alpha * N / p * (L - _log(p / alpha, a) + 1)
    Tmaxg = (1 - alpha) * N / (gamma * g) * (L - _log(g / (1 - alpha), a) + 1)
    return N, L, Tc, Tmaxg


def level_y(a, b, p, g, gamma, n, alpha):
    """y(alpha) and the case (1, 2 or 3) that applies."""
    N, L, Tc, Tmaxg = terms(a, b, p, g, gamma, n, alpha)
    if (1 - alpha) * N < g:                                          # case (i)
        ay = (gamma * Tc + 1 / (a - 1)) * (a - 1) / (N * a)           # a^-y
        return -_log(ay, a), 1
    if Tmaxg >= Tc:                                                  # case (ii)
        return L + 1 - Tc * gamma * g / ((1 - alpha) * N), 2
    ay = (Tc - Tmaxg) * gamma * (a - 1) / (N * a) + (1 - alpha) / g  # case (iii)
    return -_log(ay, a), 3


def gpu_work_fraction(a, b, p, g, gamma, n, alpha):
    N, L, _, _ = terms(a, b, p, g, gamma, n, alpha)
    y, case = level_y(a, b, p, g, gamma, n, alpha)
    return (1 - alpha) * N * (L - y + 1) / (N * (L + 1)), y, case


def optimise(a, b, p, g, gamma, n, steps=20000):
    """alpha* maximising the GPU work (grid search over alpha in [p/N, 1))."""
    N = n ** _log(a, b)
    lo, hi = p / N, 1.0
    best = None
    for k in range(1, steps):
        alpha = lo + (hi - lo) * k / steps
        frac, y, case = gpu_work_fraction(a, b, p, g, gamma, n, alpha)
        if best is None or frac > best[1]:
            best = (alpha, frac, y, case)
    return {"alpha": best[0], "gpu_work_fraction": best[1], "level_y": best[2],
            "case": best[3]}
