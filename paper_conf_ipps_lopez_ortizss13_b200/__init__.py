"""B200-native breadth-first divide-and-conquer (Lopez-Ortiz, Salinger, Suderman).

Thin Python binding over the C ABI in ``include/dc.h`` (``libdcb200.so``,
built by :mod:`.build`).  This module only marshals arguments: every step of
the hot path runs in the library's sm_100a kernels.  There is no CPU fallback:
if the library is missing or no CUDA device is present, calls raise.

    import paper_conf_ipps_lopez_ortizss13_b200 as dc
    dc.sort_(keys, vals=None)            # in-place stable sort on the GPU
    dc.max_subarray(x) -> (sum, start, end)
    dc.Plan(n)                            # explicit plan: level table, schedule, runs

Multi-GPU (one process per GPU): ``plan = dc.init_dist(n)`` binds a plan of
global size n to a library-owned NCCL communicator; ``plan.sort_(shard)`` then
runs the whole distributed sort in the library.  :mod:`.dist` drives it for
bench.py and verifies the global result.
"""
from __future__ import annotations

import atexit
import ctypes
import os
import subprocess
import weakref

import torch

from . import build as _build

__all__ = [
    "DcError", "Plan", "sort_", "max_subarray", "lib", "KEY_U32", "KEY_I32", "KEY_F32",
    "MaxsubResult", "MaxsubTuple", "get_unique_id", "init_dist", "LoopbackGroup",
    "broadcast_unique_id", "mg_exchange_sizes",
]

KEY_U32, KEY_I32, KEY_F32 = 0, 1, 2
_KEY_NAMES = {"u32": KEY_U32, "i32": KEY_I32, "f32": KEY_F32}
_STATUS = {0: "DC_OK", 1: "DC_ERR_INVALID_ARG", 2: "DC_ERR_UNSUPPORTED",
           3: "DC_ERR_OUT_OF_MEMORY", 4: "DC_ERR_CUDA", 5: "DC_ERR_NCCL",
           6: "DC_ERR_BAD_STATE"}


class DcError(RuntimeError):
    def __init__(self, status: int, detail: str):
        super().__init__(f"{_STATUS.get(status, status)}: {detail}")
        self.status = status


class MaxsubResult(ctypes.Structure):
    _fields_ = [("sum", ctypes.c_int64), ("start", ctypes.c_int64), ("end", ctypes.c_int64)]


class MaxsubTuple(ctypes.Structure):
    _fields_ = [(f, ctypes.c_int64) for f in ("tot", "pre", "suf", "best", "pe", "ss", "bs", "be")]


_lib = None
_P = ctypes.c_void_p
_I64 = ctypes.c_int64
_I32 = ctypes.c_int32
_SIGS = {
    "dc_plan": ([_I64, _I32, _I32, _I64, ctypes.POINTER(_P)], ctypes.c_int),
    "dc_plan_levels": ([_P, ctypes.POINTER(_I32), _P, _P, _I32], ctypes.c_int),
    "dc_plan_schedule": ([_P, ctypes.c_int, _I32, ctypes.POINTER(_I32), ctypes.POINTER(_I32),
                          ctypes.POINTER(_I32), ctypes.POINTER(_I32)], ctypes.c_int),
    "dc_plan_set_two_level": ([_P, _I32], ctypes.c_int),
    "dc_plan_set_tile_class": ([_P, _I32], ctypes.c_int),
    "dc_plan_set_nk1_cluster": ([_P, _I32], ctypes.c_int),
    "dc_plan_set_fused_partition": ([_P, _I32], ctypes.c_int),
    "dc_plan_set_graphs": ([_P, _I32], ctypes.c_int),
    "dc_plan_set_pipeline": ([_P, _I32], ctypes.c_int),
    "dc_sort_host_submit": ([_P, ctypes.c_int, _P, _P, _P, _P], ctypes.c_int),
    "dc_sort_host_wait": ([_P], ctypes.c_int),
    "dc_plan_set_stream": ([_P, _P], ctypes.c_int),
    "dc_plan_scratch_bytes": ([_P, _I32, ctypes.POINTER(ctypes.c_size_t)], ctypes.c_int),
    "dc_plan_set_scratch": ([_P, _P, ctypes.c_size_t], ctypes.c_int),
    "dc_free": ([_P], ctypes.c_int),
    "dc_run_mergesort": ([_P, ctypes.c_int, _P, _P], ctypes.c_int),
    "dc_run_mergesort_host": ([_P, ctypes.c_int, _P, _P], ctypes.c_int),
    "dc_run_maxsubarray": ([_P, _P, ctypes.POINTER(MaxsubResult)], ctypes.c_int),
    "dc_run_maxsubarray_async": ([_P, _P, _I64, _P], ctypes.c_int),
    "dc_run_maxsubarray_tuple_async": ([_P, _P, _I64, _P], ctypes.c_int),
    "dc_maxsub_combine_async": ([_P, _P, _I32, _P], ctypes.c_int),
    "dc_run_maxsubarray_host": ([_P, _P, ctypes.POINTER(MaxsubResult)], ctypes.c_int),
    "dc_status_string": ([ctypes.c_int], ctypes.c_char_p),
    "dc_last_error": ([], ctypes.c_char_p),
    "dc_plan_launch_count": ([_P], _I64),
    "dc_version": ([], ctypes.c_char_p),
    "dc_plan_enable_timing": ([_P, _I32], ctypes.c_int),
    "dc_plan_kernel_time": ([_P, _I32, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(_I64)],
                            ctypes.c_int),
}

_SIGS.update({
    "dc_mg_sendbuf_words": ([_I32, _I64], _I64),
    "dc_mg_sample": ([_P, _P, _I64, _I64, _P], ctypes.c_int),
    "dc_mg_count": ([_P, ctypes.c_int, _P, _I64, _I32, _P, _I64, _I64, _I64, _P], ctypes.c_int),
    "dc_mg_windows": ([_P, _P, _I64, _I32, _I32, _P, _P, _I64, _I64, _I64, _P], ctypes.c_int),
    "dc_mg_split_matrix": ([_P, ctypes.c_int, _P, _I32, _I64, _I64, _P], ctypes.c_int),
    "dc_mg_error": ([_P, ctypes.POINTER(_I32)], ctypes.c_int),
    "dc_mg_merge_runs": ([_P, ctypes.c_int, _P, _P, _P, _P, _P, _I32], ctypes.c_int),
    "dc_mg_exchange_sizes": ([_P, _I32, _I32, _I64, _P, _P, _P, _P], ctypes.c_int),
})

_SIGS.update({
    "dc_get_unique_id": ([_P], ctypes.c_int),
    "dc_plan_set_comm": ([_P, _P, _I32, _I32], ctypes.c_int),
    "dc_loopback_create": ([_I32, ctypes.POINTER(_P)], ctypes.c_int),
    "dc_loopback_free": ([_P], ctypes.c_int),
    "dc_plan_set_loopback": ([_P, _P, _I32], ctypes.c_int),
    "dc_plan_comm_info": ([_P, ctypes.POINTER(_I32), ctypes.POINTER(_I32), ctypes.POINTER(_I64)],
                          ctypes.c_int),
    "dc_plan_set_mg_stride": ([_P, _I64], ctypes.c_int),
    "dc_plan_last_splits": ([_P, _P], ctypes.c_int),
    "dc_plan_set_mg_p2p": ([_P, _I32], ctypes.c_int),
    "dc_plan_mg_phase_times": ([_P, _P, ctypes.POINTER(_I64), ctypes.POINTER(_I64)], ctypes.c_int),
    "dc_plan_mg_reset_phases": ([_P], ctypes.c_int),
    "dc_plan_mg_exchange_mode": ([_P, ctypes.POINTER(_I32)], ctypes.c_int),
    "dc_mg_merge_peers": ([_P, ctypes.c_int, _P, _P, _P, _P, _P, _I32, _P, _P, _P, _P],
                          ctypes.c_int),
})

class SortSchedule(ctypes.Structure):
    _fields_ = [("tile_class", _I32), ("two_level", _I32), ("tile", _I32),
                ("fused_levels", _I32), ("global_levels", _I32), ("hbm_passes", _I32),
                ("predicted_ms", ctypes.c_double), ("candidates_ms", ctypes.c_double * 4)]


_SIGS.update({
    "dc_model_sort_schedule": ([_I64, ctypes.c_int, _I32, _I32, _I32, ctypes.POINTER(SortSchedule)],
                               ctypes.c_int),
    "dc_run_sum": ([_P, _P, ctypes.POINTER(_I64)], ctypes.c_int),
    "dc_run_sum_async": ([_P, _P, _P], ctypes.c_int),
    "dc_run_sum_alg5": ([_P, _P, ctypes.POINTER(_I64)], ctypes.c_int),
})

_D = ctypes.c_double
_SIGS.update({
    "dc_model_gpu_work": ([_I32, _I32, _I32, _D, _D, _D, _D, ctypes.POINTER(_D), ctypes.POINTER(_D),
                           ctypes.POINTER(_I32)], ctypes.c_int),
    "dc_model_optimise": ([_I32, _I32, _I32, _D, _D, _D, ctypes.POINTER(_D), ctypes.POINTER(_D),
                           ctypes.POINTER(_D), ctypes.POINTER(_I32)], ctypes.c_int),
})


def model_gpu_work(a: int, b: int, p: int, g: float, gamma: float, n: float,
                   alpha: float) -> dict:
    """Paper Sec. 5.2 model: GPU work share, level y and case for a given alpha."""
    f, y, c = ctypes.c_double(), ctypes.c_double(), _I32()
    st = lib().dc_model_gpu_work(a, b, p, g, gamma, n, alpha, ctypes.byref(f), ctypes.byref(y),
                                 ctypes.byref(c))
    if st != 0:
        raise DcError(st, "invalid model parameters")
    return {"gpu_work_fraction": f.value, "level_y": y.value, "case": c.value}


def model_sort_schedule(n: int, key_type: str = "u32", with_vals: bool = False,
                        tile_class: int = 0, two_level: int = -1) -> dict:
    """The B200 schedule planner (dc_model_sort_schedule): the
    schedule of least predicted time and every candidate's prediction."""
    s = SortSchedule()
    _check(lib().dc_model_sort_schedule(n, _KEY_NAMES[key_type], int(with_vals), tile_class,
                                        two_level, ctypes.byref(s)))
    return {"tile_class": s.tile_class, "two_level": bool(s.two_level), "tile": s.tile,
            "fused_levels": s.fused_levels, "global_levels": s.global_levels,
            "hbm_passes": s.hbm_passes, "predicted_ms": s.predicted_ms,
            "candidates_ms": {"quarter_one": s.candidates_ms[0], "quarter_two": s.candidates_ms[1],
                              "full_one": s.candidates_ms[2], "full_two": s.candidates_ms[3]}}


def model_optimise(a: int, b: int, p: int, g: float, gamma: float, n: float) -> dict:
    """Paper Sec. 5.2 model: alpha* maximising the GPU work."""
    al, f, y, c = ctypes.c_double(), ctypes.c_double(), ctypes.c_double(), _I32()
    st = lib().dc_model_optimise(a, b, p, g, gamma, n, ctypes.byref(al), ctypes.byref(f),
                                 ctypes.byref(y), ctypes.byref(c))
    if st != 0:
        raise DcError(st, "invalid model parameters")
    return {"alpha": al.value, "gpu_work_fraction": f.value, "level_y": y.value, "case": c.value}


#: kernel classes of dc_plan_kernel_time
KERNELS = {"nk1_blocksort": 0, "nk2_partition": 1, "nk3_merge": 2, "nk4_maxsub": 3}


def lib() -> ctypes.CDLL:
    """Load (building first if stale and nvcc is available) libdcb200.so."""
    global _lib
    if _lib is None:
        path = _build.LIB
        if os.environ.get("DC_LIB"):          # a tuning variant built by build.py --out
            path = os.environ["DC_LIB"]
        else:
            try:
                path = _build.build()
            except (OSError, FileNotFoundError, subprocess.CalledProcessError):
                if not os.path.exists(path):
                    raise
        handle = ctypes.CDLL(path)
        for name, (args, res) in _SIGS.items():
            fn = getattr(handle, name)
            fn.argtypes = args
            fn.restype = res
        _lib = handle
    return _lib


def _check(status: int) -> None:
    if status != 0:
        raise DcError(status, lib().dc_last_error().decode())


def _key_type(t: torch.Tensor, key_type: str | None) -> int:
    if key_type is not None:
        return _KEY_NAMES[key_type]
    if t.dtype == torch.uint32:
        return KEY_U32
    if t.dtype == torch.int32:
        return KEY_I32
    if t.dtype == torch.float32:
        return KEY_F32
    raise TypeError(f"unsupported key dtype {t.dtype}")


def _require_cuda(t: torch.Tensor, what: str, numel: int | None = None) -> None:
    if not t.is_cuda:
        raise ValueError(f"{what} must be a CUDA tensor (no CPU fallback)")
    if not t.is_contiguous():
        raise ValueError(f"{what} must be contiguous")
    if t.element_size() != 4:
        raise ValueError(f"{what} must have 4-byte elements")
    if numel is not None and t.numel() != numel:
        raise ValueError(f"{what} must have {numel} elements, not {t.numel()}")


def _require_host(t: torch.Tensor, what: str, numel: int) -> None:
    """Host buffers the C side copies n*4 bytes into / out of."""
    if t.is_cuda:
        raise ValueError(f"{what} must be a host tensor")
    if not t.is_contiguous():
        raise ValueError(f"{what} must be contiguous")
    if t.element_size() != 4:
        raise ValueError(f"{what} must have 4-byte elements")
    if t.numel() != numel:
        raise ValueError(f"{what} must have {numel} elements, not {t.numel()}")


def _require_out(t: torch.Tensor, what: str, min_numel: int) -> None:
    """Device int64 result buffers written by the library."""
    if not t.is_cuda or t.dtype != torch.int64 or not t.is_contiguous():
        raise ValueError(f"{what} must be a contiguous CUDA int64 tensor")
    if t.numel() < min_numel:
        raise ValueError(f"{what} needs at least {min_numel} elements")


class Plan:
    """A ``dc_plan`` handle: T(n) = aT(n/b) + f(n) recursion for n elements."""

    def __init__(self, n: int, a: int = 2, b: int = 2, base_size: int = 1):
        h = _P()
        _check(lib().dc_plan(n, a, b, base_size, ctypes.byref(h)))
        self._h = h
        self.n, self.a, self.b, self.base_size = n, a, b, base_size
        _live_plans.add(self)

    def close(self) -> None:
        """Free the plan's device state now (idempotent; also done by GC / at exit)."""
        h = getattr(self, "_h", None)
        if h is not None and _lib is not None:
            _lib.dc_free(h)
        self._h = None

    def __del__(self):
        self.close()

    def levels(self) -> list[tuple[int, int]]:
        """[(nodes a^i, size ceil(n/b^i)) for each level i]."""
        cnt = _I32()
        _check(lib().dc_plan_levels(self._h, ctypes.byref(cnt), None, None, 0))
        nodes = (_I64 * cnt.value)()
        sizes = (_I64 * cnt.value)()
        _check(lib().dc_plan_levels(self._h, ctypes.byref(cnt), nodes, sizes, cnt.value))
        return list(zip(nodes, sizes))

    def schedule(self, key_type: str = "u32", with_vals: bool = False) -> dict:
        t, f, p, h = _I32(), _I32(), _I32(), _I32()
        _check(lib().dc_plan_schedule(self._h, _KEY_NAMES[key_type], int(with_vals),
                                      ctypes.byref(t), ctypes.byref(f), ctypes.byref(p),
                                      ctypes.byref(h)))
        return {"tile": t.value, "fused_levels": f.value, "global_passes": p.value,
                "hbm_passes": h.value}

    # ------------------------------------------------ library communicator
    def _attached(self) -> None:
        r, w, m = _I32(), _I32(), _I64()
        _check(lib().dc_plan_comm_info(self._h, ctypes.byref(r), ctypes.byref(w), ctypes.byref(m)))
        self.rank, self.world, self.n_global, self.n = r.value, w.value, self.n, m.value

    def set_comm(self, uid: bytes, rank: int, world: int) -> None:
        """Join the NCCL communicator ``uid`` (from :func:`get_unique_id`) as
        ``rank`` of ``world``; afterwards ``self.n`` is this rank's shard size
        and sort_ / max_subarray run the multi-GPU method (include/dc.h)."""
        if len(uid) != 128:
            raise ValueError("unique id must be 128 bytes")
        buf = ctypes.create_string_buffer(bytes(uid), 128)
        _check(lib().dc_plan_set_comm(self._h, buf, rank, world))
        self._attached()

    def set_loopback(self, group: "LoopbackGroup", rank: int) -> None:
        """Join an in-process loopback group (threads sharing one GPU; tests)."""
        _check(lib().dc_plan_set_loopback(self._h, group._h, rank))
        self._group = group            # the group outlives its member plans
        self._attached()

    def set_mg_stride(self, stride: int) -> None:
        _check(lib().dc_plan_set_mg_stride(self._h, stride))

    def set_mg_p2p(self, enable: bool) -> None:
        """Fused exchange (merge reads the peers' shards) vs NCCL all-to-all."""
        _check(lib().dc_plan_set_mg_p2p(self._h, int(enable)))

    def mg_phase_times(self) -> dict:
        """{'local_sort','splitters','exchange_merge'} ms summed over timed sorts,
        'sorts', 'keys_received' (dc_plan_mg_phase_times)."""
        ms = (ctypes.c_double * 3)()
        n, k = _I64(), _I64()
        _check(lib().dc_plan_mg_phase_times(self._h, ms, ctypes.byref(n), ctypes.byref(k)))
        return {"local_sort": ms[0], "splitters": ms[1], "exchange_merge": ms[2],
                "sorts": n.value, "keys_received": k.value}

    def mg_reset_phases(self) -> None:
        _check(lib().dc_plan_mg_reset_phases(self._h))

    def exchange_mode(self) -> str:
        m = _I32()
        _check(lib().dc_plan_mg_exchange_mode(self._h, ctypes.byref(m)))
        return {1: "fused", -1: "all_to_all", 0: "undecided"}[m.value]

    def last_splits(self) -> list[list[int]]:
        """Split matrix c[r][d] of the last multi-GPU sort (world x (world+1))."""
        w = getattr(self, "world", 1)
        buf = (_I64 * (w * (w + 1)))()
        _check(lib().dc_plan_last_splits(self._h, buf))
        return [list(buf[r * (w + 1):(r + 1) * (w + 1)]) for r in range(w)]

    def set_pipeline(self, chunks: int) -> None:
        """Chunked multi-stream pipeline of the one-level schedule (0/1 = off, the default)."""
        _check(lib().dc_plan_set_pipeline(self._h, chunks))

    def set_graphs(self, enable: bool) -> None:
        """CUDA-graph replay of the sort's launch sequence (default on)."""
        _check(lib().dc_plan_set_graphs(self._h, int(enable)))

    def set_fused_partition(self, enable: bool) -> None:
        """L2-resident sorts: merge CTAs find their own co-ranks (default on)."""
        _check(lib().dc_plan_set_fused_partition(self._h, int(enable)))

    def set_two_level(self, enable: bool | None) -> None:
        """Force (True) / forbid (False) two merge levels per HBM pass (SURVEY
        f1), or leave the choice to the planner (None, the default)."""
        _check(lib().dc_plan_set_two_level(self._h, -1 if enable is None else int(enable)))

    def set_tile_class(self, tile_class: int) -> None:
        """NK1 tile class: 1 quarter-size, 2 full, 0 planner (default)."""
        _check(lib().dc_plan_set_tile_class(self._h, tile_class))

    def set_nk1_cluster(self, cs: int) -> None:
        """NK1 cluster size for keys-only u32/i32 sorts: 2/4/8/16
        fuse log2(cs) more levels through distributed shared memory, 1 off,
        0 the planner's rule (default)."""
        _check(lib().dc_plan_set_nk1_cluster(self._h, int(cs)))

    def scratch_bytes(self, with_vals: bool = False) -> int:
        b = ctypes.c_size_t()
        _check(lib().dc_plan_scratch_bytes(self._h, int(with_vals), ctypes.byref(b)))
        return b.value

    def set_scratch(self, buf: torch.Tensor) -> None:
        _check(lib().dc_plan_set_scratch(self._h, buf.data_ptr(), buf.numel() * buf.element_size()))
        self._scratch_ref = buf

    def launch_count(self) -> int:
        return int(lib().dc_plan_launch_count(self._h))

    def enable_timing(self, on: bool = True) -> None:
        """Bracket every launch with CUDA events on the plan stream (resets totals)."""
        _check(lib().dc_plan_enable_timing(self._h, int(on)))

    def kernel_times(self) -> dict:
        """{kernel: (total_ms, launches)} since enable_timing (waits for the events)."""
        out = {}
        for name, k in KERNELS.items():
            ms, cnt = ctypes.c_double(), _I64()
            _check(lib().dc_plan_kernel_time(self._h, k, ctypes.byref(ms), ctypes.byref(cnt)))
            out[name] = (ms.value, cnt.value)
        return out

    def _bind_stream(self, t: torch.Tensor) -> None:
        _check(lib().dc_plan_set_stream(self._h, torch.cuda.current_stream(t.device).cuda_stream))

    def sort_(self, keys: torch.Tensor, vals: torch.Tensor | None = None,
              key_type: str | None = None) -> torch.Tensor:
        """In-place stable sort of keys (and vals alongside) on the GPU."""
        _require_cuda(keys, "keys")
        if keys.numel() != self.n:
            raise ValueError("keys length != plan n")
        if vals is not None:
            _require_cuda(vals, "vals")
            if vals.numel() != self.n:
                raise ValueError("vals length != plan n")
        kt = _key_type(keys, key_type)
        self._bind_stream(keys)
        _check(lib().dc_run_mergesort(self._h, kt, keys.data_ptr(),
                                      None if vals is None else vals.data_ptr()))
        return keys

    def sort_host_(self, keys: torch.Tensor, vals: torch.Tensor | None = None,
                   key_type: str | None = None) -> torch.Tensor:
        """End-to-end sort of HOST tensors (pinned for full speed): H2D, sort, D2H."""
        _require_host(keys, "keys", self.n)
        if vals is not None:
            _require_host(vals, "vals", self.n)
        kt = _key_type(keys, key_type)
        _check(lib().dc_plan_set_stream(self._h, torch.cuda.current_stream().cuda_stream))
        _check(lib().dc_run_mergesort_host(self._h, kt, keys.data_ptr(),
                                           None if vals is None else vals.data_ptr()))
        return keys

    def sort_host_submit(self, keys_in: torch.Tensor, keys_out: torch.Tensor,
                         vals_in: torch.Tensor | None = None,
                         vals_out: torch.Tensor | None = None, key_type: str | None = None):
        """Streaming end-to-end sort of pinned HOST tensors (input unmodified).

        Consecutive submissions overlap (upload / sort / download on separate
        streams); call :meth:`sort_host_wait` before reading the outputs."""
        if (vals_in is None) != (vals_out is None):
            raise ValueError("vals_in and vals_out: both or neither")
        for name, t in (("keys_in", keys_in), ("keys_out", keys_out), ("vals_in", vals_in),
                        ("vals_out", vals_out)):
            if t is not None:
                _require_host(t, name, self.n)
        _check(lib().dc_plan_set_stream(self._h, torch.cuda.current_stream().cuda_stream))
        _check(lib().dc_sort_host_submit(self._h, _key_type(keys_in, key_type),
                                         keys_in.data_ptr(),
                                         None if vals_in is None else vals_in.data_ptr(),
                                         keys_out.data_ptr(),
                                         None if vals_out is None else vals_out.data_ptr()))
        self._host_refs = getattr(self, "_host_refs", [])[-4:] + [
            (keys_in, keys_out, vals_in, vals_out)]

    def sort_host_wait(self) -> None:
        _check(lib().dc_plan_set_stream(self._h, torch.cuda.current_stream().cuda_stream))
        _check(lib().dc_sort_host_wait(self._h))
        self._host_refs = []

    def max_subarray(self, x: torch.Tensor) -> tuple[int, int, int]:
        _require_cuda(x, "x", self.n)
        self._bind_stream(x)
        r = MaxsubResult()
        _check(lib().dc_run_maxsubarray(self._h, x.data_ptr(), ctypes.byref(r)))
        return (r.sum, r.start, r.end)

    def max_subarray_async(self, x: torch.Tensor, out: torch.Tensor, index_offset: int = 0):
        """Enqueue only; ``out`` is a CUDA int64 tensor of 3 elements (sum, start, end)."""
        _require_cuda(x, "x", self.n)
        _require_out(out, "out", 3)
        self._bind_stream(x)
        _check(lib().dc_run_maxsubarray_async(self._h, x.data_ptr(), index_offset, out.data_ptr()))
        return out

    def max_subarray_tuple_async(self, x: torch.Tensor, out: torch.Tensor, index_offset: int = 0):
        """Enqueue only; ``out`` is a CUDA int64 tensor of 8 elements (segment summary)."""
        _require_cuda(x, "x", self.n)
        _require_out(out, "out", 8)
        self._bind_stream(x)
        _check(lib().dc_run_maxsubarray_tuple_async(self._h, x.data_ptr(), index_offset,
                                                    out.data_ptr()))
        return out

    def maxsub_combine_async(self, tuples: torch.Tensor, out: torch.Tensor):
        """Ordered combine of a (count, 8) int64 CUDA tensor of summaries into out[3]."""
        if tuples.dim() != 2 or tuples.shape[1] != 8 or tuples.shape[0] < 1:
            raise ValueError("tuples must have shape (count >= 1, 8)")
        _require_out(tuples, "tuples", 8)
        _require_out(out, "out", 3)
        self._bind_stream(tuples)
        _check(lib().dc_maxsub_combine_async(self._h, tuples.data_ptr(), tuples.shape[0],
                                             out.data_ptr()))
        return out

    def max_subarray_host(self, x: torch.Tensor) -> tuple[int, int, int]:
        """End-to-end max subarray of a HOST int32 tensor."""
        _require_host(x, "x", self.n)
        _check(lib().dc_plan_set_stream(self._h, torch.cuda.current_stream().cuda_stream))
        r = MaxsubResult()
        _check(lib().dc_run_maxsubarray_host(self._h, x.data_ptr(), ctypes.byref(r)))
        return (r.sum, r.start, r.end)


    # ---------------------------------------------------- D&C sum (f4)
    def sum(self, x: torch.Tensor) -> int:
        """Exact int64 sum of an int32 CUDA tensor (Alg 4 through dc_reduce.cuh)."""
        _require_cuda(x, "x", self.n)
        self._bind_stream(x)
        r = _I64()
        _check(lib().dc_run_sum(self._h, x.data_ptr(), ctypes.byref(r)))
        return r.value

    def sum_async(self, x: torch.Tensor, out: torch.Tensor) -> torch.Tensor:
        _require_cuda(x, "x", self.n)
        _require_out(out, "out", 1)
        self._bind_stream(x)
        _check(lib().dc_run_sum_async(self._h, x.data_ptr(), out.data_ptr()))
        return out

    def sum_alg5(self, work: torch.Tensor) -> int:
        """Alg 5 literally (one launch per level) on an int64 CUDA work tensor (clobbered)."""
        _require_out(work, "work", self.n)
        self._bind_stream(work)
        r = _I64()
        _check(lib().dc_run_sum_alg5(self._h, work.data_ptr(), ctypes.byref(r)))
        return r.value

    # ------------------------------------------ multi-GPU building blocks
    def mg_sample(self, keys: torch.Tensor, stride: int) -> torch.Tensor:
        """Every stride-th key of this rank's sorted shard (uint32 bits as int32)."""
        _require_cuda(keys, "keys")
        if stride < 1:
            raise ValueError("stride must be >= 1")
        out = torch.empty((keys.numel() + stride - 1) // stride, dtype=torch.int32,
                          device=keys.device)
        self._bind_stream(keys)
        _check(lib().dc_mg_sample(self._h, keys.data_ptr(), keys.numel(), stride, out.data_ptr()))
        return out

    def mg_count(self, keys: torch.Tensor, rank: int, cand: torch.Tensor, per_rank: int,
                 stride: int, key_type: str | None = None) -> torch.Tensor:
        """Composite counts of this rank's elements below every candidate (int64)."""
        _require_cuda(keys, "keys")
        _require_cuda(cand, "cand")
        if cand.numel() < 1 or cand.numel() % per_rank:
            raise ValueError("cand must hold world * per_rank candidates")
        out = torch.empty(cand.numel(), dtype=torch.int64, device=keys.device)
        self._bind_stream(keys)
        _check(lib().dc_mg_count(self._h, _key_type(keys, key_type), keys.data_ptr(),
                                 keys.numel(), rank, cand.data_ptr(), per_rank, stride,
                                 cand.numel(), out.data_ptr()))
        return out

    def mg_windows(self, keys: torch.Tensor, rank: int, world: int, counts: torch.Tensor,
                   ranks: torch.Tensor, per_rank: int, wcap: int) -> torch.Tensor:
        _require_cuda(keys, "keys")
        if counts.numel() != ranks.numel() or counts.dtype != torch.int64 or \
                ranks.dtype != torch.int64 or not counts.is_cuda or not ranks.is_cuda:
            raise ValueError("counts and ranks must be CUDA int64 tensors of equal length")
        words = int(lib().dc_mg_sendbuf_words(world, wcap))
        out = torch.zeros(words, dtype=torch.int32, device=keys.device)
        self._bind_stream(keys)
        _check(lib().dc_mg_windows(self._h, keys.data_ptr(), keys.numel(), rank, world,
                                   counts.data_ptr(), ranks.data_ptr(), per_rank, counts.numel(),
                                   wcap, out.data_ptr()))
        return out

    def mg_split_matrix(self, gathered: torch.Tensor, world: int, shard_n: int, wcap: int,
                        key_type: str) -> torch.Tensor:
        _require_cuda(gathered, "gathered", world * int(lib().dc_mg_sendbuf_words(world, wcap)))
        out = torch.empty((world, world + 1), dtype=torch.int64, device=gathered.device)
        self._bind_stream(gathered)
        _check(lib().dc_mg_split_matrix(self._h, _KEY_NAMES[key_type], gathered.data_ptr(),
                                        world, shard_n, wcap, out.data_ptr()))
        return out

    def mg_error(self) -> int:
        e = _I32()
        _check(lib().dc_mg_error(self._h, ctypes.byref(e)))
        return e.value

    def mg_merge_peers(self, runs: list, out_keys: torch.Tensor,
                       out_vals: torch.Tensor | None = None, tmp_keys: torch.Tensor | None = None,
                       tmp_vals: torch.Tensor | None = None, key_type: str | None = None):
        """Stable merge of runs stored in separate buffers: runs = [(keys_buf,
        vals_buf or None, offset, length), ...] (earlier runs win ties)."""
        r = len(runs)
        _require_cuda(out_keys, "out_keys")
        if out_vals is not None:
            _require_cuda(out_vals, "out_vals")
        for k, v, off, ln in runs:
            _require_cuda(k, "run keys")
            if off < 0 or ln < 0 or off + ln > k.numel():
                raise ValueError("run outside its buffer")
            if out_vals is not None and (v is None or v.numel() < off + ln):
                raise ValueError("run values missing or too short")
        kp = (_P * r)(*[t[0].data_ptr() for t in runs])
        vp = (_P * r)(*[t[1].data_ptr() for t in runs]) if out_vals is not None else None
        bound = (_I64 * r)(*[t[0].numel() for t in runs])
        off = (_I64 * r)(*[t[2] for t in runs])
        ln = (_I64 * r)(*[t[3] for t in runs])
        self._bind_stream(out_keys)
        _check(lib().dc_mg_merge_peers(
            self._h, _key_type(out_keys, key_type), kp, vp, bound, off, ln, r,
            None if tmp_keys is None else tmp_keys.data_ptr(),
            None if tmp_vals is None else tmp_vals.data_ptr(), out_keys.data_ptr(),
            None if out_vals is None else out_vals.data_ptr()))
        return out_keys

    def mg_merge_runs(self, in_keys: torch.Tensor, in_vals: torch.Tensor | None,
                      out_keys: torch.Tensor, out_vals: torch.Tensor | None, run_len: list[int],
                      key_type: str | None = None) -> torch.Tensor:
        """Stable merge of back-to-back sorted runs (earlier runs win ties)."""
        total = sum(run_len)
        for name, t in (("in_keys", in_keys), ("in_vals", in_vals), ("out_keys", out_keys),
                        ("out_vals", out_vals)):
            if t is not None:
                _require_cuda(t, name)
                if t.numel() < total:
                    raise ValueError(f"{name} holds fewer than sum(run_len) elements")
        lens = (_I64 * len(run_len))(*run_len)
        self._bind_stream(in_keys)
        _check(lib().dc_mg_merge_runs(self._h, _key_type(in_keys, key_type), in_keys.data_ptr(),
                                      None if in_vals is None else in_vals.data_ptr(),
                                      out_keys.data_ptr(),
                                      None if out_vals is None else out_vals.data_ptr(),
                                      lens, len(run_len)))
        return out_keys


# Plans (then groups) still alive at interpreter exit -- e.g. held by a
# traceback cycle -- are freed before the CUDA runtime is torn down.
_live_plans: "weakref.WeakSet[Plan]" = weakref.WeakSet()
_live_groups: "weakref.WeakSet[LoopbackGroup]" = weakref.WeakSet()


@atexit.register
def _free_at_exit() -> None:
    for p in list(_live_plans):
        p.close()
    for g in list(_live_groups):
        g.close()


def get_unique_id() -> bytes:
    """128-byte NCCL unique id for :meth:`Plan.set_comm` (create on one rank)."""
    buf = ctypes.create_string_buffer(128)
    _check(lib().dc_get_unique_id(buf))
    return buf.raw


class LoopbackGroup:
    """``world`` ranks as threads of this process sharing one GPU (dc_loopback_*)."""

    def __init__(self, world: int):
        h = _P()
        _check(lib().dc_loopback_create(world, ctypes.byref(h)))
        self._h, self.world = h, world
        _live_groups.add(self)

    def close(self) -> None:
        h = getattr(self, "_h", None)
        if h is not None and _lib is not None:
            _lib.dc_loopback_free(h)
        self._h = None

    def __del__(self):
        self.close()


def broadcast_unique_id(group=None) -> bytes:
    """The group's rank 0 creates a 128-byte NCCL id; torch.distributed
    broadcasts it to every member (any backend)."""
    import torch.distributed as tdist

    rank = tdist.get_rank(group)
    obj = [get_unique_id() if rank == 0 else None]
    tdist.broadcast_object_list(obj, src=tdist.get_global_rank(group, 0) if group else 0,
                                group=group)
    if not isinstance(obj[0], (bytes, bytearray)) or len(obj[0]) != 128:
        raise DcError(1, "bad unique id received")
    return bytes(obj[0])


def init_dist(n: int, group=None) -> Plan:
    """Plan of global size n bound to a library-owned NCCL communicator over
    the torch.distributed group (rank 0 creates the id, broadcast by torch).
    Set the CUDA device of this rank first."""
    import torch.distributed as tdist

    uid = broadcast_unique_id(group)
    plan = Plan(n)
    plan.set_comm(uid, tdist.get_rank(group), tdist.get_world_size(group))
    return plan


def mg_exchange_sizes(cmat, rank: int, shard_n: int) -> dict:
    """The runtime's host step (dc_mg_exchange_sizes): from a split matrix
    c[r][d] (world x (world+1)), what `rank` sends to / receives from every
    rank: {'send_cnt', 'send_off', 'recv_cnt', 'recv_off'} lists."""
    world = len(cmat)
    flat = (_I64 * (world * (world + 1)))(*[int(v) for row in cmat for v in row])
    arrs = [(_I64 * world)() for _ in range(4)]
    _check(lib().dc_mg_exchange_sizes(flat, world, rank, shard_n, *arrs))
    return dict(zip(("send_cnt", "send_off", "recv_cnt", "recv_off"),
                    [list(a) for a in arrs]))


_plans: dict = {}


def _plan_for(n: int, device) -> Plan:
    key = (n, str(device))
    p = _plans.get(key)
    if p is None:
        p = _plans[key] = Plan(n)
    return p


def sort_(keys: torch.Tensor, vals: torch.Tensor | None = None,
          key_type: str | None = None) -> torch.Tensor:
    """In-place stable GPU mergesort of ``keys`` (uint32/int32/float32 CUDA tensor).

    ``key_type`` overrides the dtype-derived key type ("u32", "i32", "f32"),
    e.g. to sort int32-stored bit patterns as unsigned.
    """
    return _plan_for(keys.numel(), keys.device).sort_(keys, vals, key_type)


def max_subarray(x: torch.Tensor) -> tuple[int, int, int]:
    """(sum, start, end) of the maximum non-empty subarray of an int32 CUDA tensor."""
    return _plan_for(x.numel(), x.device).max_subarray(x)
