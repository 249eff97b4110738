"""CPU oracle for the hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
and ``--impl reference`` legs may import this package.  The product package
(``paper_conf_ipps_lopez_ortizss13_b200``) never imports it and shares no code
with it.

The arithmetic lives in ``oracle.c`` (plain C, built with gcc into
``liboracle.so``); this module only marshals numpy arrays.  Each function cites
the PAPER.md passage it follows (``P:Lx-y`` = /root/reference/PAPER.md lines).

* :func:`mergesort`     -- Alg 6 recursive mergesort, stable.
* :func:`mergesort_bf`  -- Alg 7 breadth-first mergesort, n = 2^k.
* :func:`maxsub`        -- textbook recursive D&C maximum subarray (north star).
* :func:`dc_sum`        -- Alg 4 recursive D&C sum.
* :mod:`oracle.planner` -- the Sec. 5.2 work-division model.

Parity status: every function here is pinned by tests/test_oracle.py against
brute force, closed forms, library routines or the paper's printed numbers.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
MAX_DEPTH = 64
KEY_TYPES = {"u32": 0, "i32": 1, "f32": 2}
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (plain -O2, no vectorisation tricks)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-fPIC", "-shared", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        i64p = ctypes.POINTER(ctypes.c_int64)
        lib.oracle_mergesort.argtypes = [ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p,
                                         ctypes.c_int64, ctypes.c_void_p, ctypes.c_void_p]
        lib.oracle_mergesort_bf.argtypes = [ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p,
                                            ctypes.c_int64]
        lib.oracle_maxsub.argtypes = [ctypes.c_void_p, ctypes.c_int64, i64p, i64p, i64p,
                                      ctypes.c_void_p]
        lib.oracle_sum.argtypes = [ctypes.c_void_p, ctypes.c_int64]
        for f in (lib.oracle_mergesort, lib.oracle_mergesort_bf, lib.oracle_maxsub,
                  lib.oracle_sum):
            f.restype = ctypes.c_int
        _lib = lib
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data


def _as_u32_bits(keys: np.ndarray, key_type: str) -> np.ndarray:
    dt = {"u32": np.uint32, "i32": np.int32, "f32": np.float32}[key_type]
    k = np.ascontiguousarray(keys, dtype=dt).copy()
    return k.view(np.uint32)


def mergesort(keys: np.ndarray, vals: np.ndarray | None = None, key_type: str = "u32",
              counters: bool = False):
    """Alg 6: returns sorted copies (keys[, vals]) -- stable.

    With ``counters=True`` also returns (level_combines, level_elems): per
    recursion depth d (0 = root) the number of combine (merge)
    calls and the number of elements merged.
    """
    kt = KEY_TYPES[key_type]
    k = _as_u32_bits(keys, key_type)
    v = None if vals is None else np.ascontiguousarray(vals, dtype=np.uint32).copy()
    if v is not None and v.shape != k.shape:
        raise ValueError("keys/vals length mismatch")
    lc = np.zeros(MAX_DEPTH, np.int64) if counters else None
    le = np.zeros(MAX_DEPTH, np.int64) if counters else None
    rc = _load().oracle_mergesort(kt, _ptr(k), _ptr(v), k.size, _ptr(lc), _ptr(le))
    if rc != 0:
        raise RuntimeError("oracle_mergesort failed")
    out_k = k.view({"u32": np.uint32, "i32": np.int32, "f32": np.float32}[key_type])
    res = (out_k,) if v is None else (out_k, v)
    if counters:
        res = res + (lc, le)
    return res[0] if len(res) == 1 else res


def mergesort_bf(keys: np.ndarray, vals: np.ndarray | None = None, key_type: str = "u32"):
    """Alg 7 breadth-first mergesort; n must be a power of two."""
    kt = KEY_TYPES[key_type]
    k = _as_u32_bits(keys, key_type)
    v = None if vals is None else np.ascontiguousarray(vals, dtype=np.uint32).copy()
    rc = _load().oracle_mergesort_bf(kt, _ptr(k), _ptr(v), k.size)
    if rc != 0:
        raise ValueError("oracle_mergesort_bf: n must be a power of two")
    out_k = k.view({"u32": np.uint32, "i32": np.int32, "f32": np.float32}[key_type])
    return out_k if v is None else (out_k, v)


def maxsub(x: np.ndarray, counters: bool = False):
    """Recursive D&C maximum subarray (north star instance 2).

    Returns (sum, start, end), end inclusive, non-empty subarray, int64 sums,
    lexicographically smallest (start, end) among the maxima.
    """
    a = np.ascontiguousarray(x, dtype=np.int32)
    s, b, e = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
    lc = np.zeros(MAX_DEPTH, np.int64) if counters else None
    rc = _load().oracle_maxsub(_ptr(a), a.size, ctypes.byref(s), ctypes.byref(b),
                               ctypes.byref(e), _ptr(lc))
    if rc != 0:
        raise ValueError("oracle_maxsub: n must be >= 1")
    res = (s.value, b.value, e.value)
    return (res, lc) if counters else res


def dc_sum(x: np.ndarray) -> int:
    """Alg 4 recursive D&C sum in int64."""
    a = np.ascontiguousarray(x, dtype=np.int64).copy()
    if _load().oracle_sum(_ptr(a), a.size) != 0:
        raise ValueError("oracle_sum: n must be >= 1")
    return int(a[0])
