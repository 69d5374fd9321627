"""Thin Python binding of the C-ABI library (include/smiless.h) -- argument marshalling only.

Every step of the hot path runs in libsmiless.so's CUDA kernels.  There is no CPU
fallback: if the library cannot be loaded or the GPU is missing, calls raise
SmilessError (the C side returns SMILESS_ECUDA / SMILESS_EJIT).
"""
from __future__ import annotations

import ctypes
import dataclasses
import os
from typing import Optional, Sequence, Tuple

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libsmiless.so")

OK, INFEASIBLE = 0, 1
EINVAL, ENOTTOPO, ERANGE, ESTATE, ECUDA, ENOMEM, EJIT = -1, -2, -3, -4, -5, -6, -7
FLAG_NO_PRUNE, FLAG_ARRIVALS_ON_DEVICE, FLAG_FORCE_INT64, FLAG_COST_CAP = 1, 2, 4, 8
PATH_NONE, PATH_PLAN, PATH_BNB, PATH_MEMO, PATH_MEMO_FUSED = 0, 1, 2, 3, 4   # smiless_plan_result.eval_path
_NAMES = {0: "OK", 1: "INFEASIBLE", -1: "EINVAL", -2: "ENOTTOPO", -3: "ERANGE", -4: "ESTATE",
          -5: "ECUDA", -6: "ENOMEM", -7: "EJIT"}

# every symbol include/smiless.h declares (checked by tests/test_abi.py)
EXPORTS = ("smiless_create", "smiless_set_stream", "smiless_destroy", "smiless_last_error",
           "smiless_load_dag", "smiless_load_profiles", "smiless_space_size", "smiless_plan", "smiless_plan_digits",
           "smiless_plan_sla_sweep", "smiless_derive_windows", "smiless_top1_search", "smiless_decompose_search", "smiless_decompose_plan",
           "smiless_decompose_plan_sharded",
           "smiless_autoscale", "smiless_autoscale_rows",
           "smiless_evaluate",
           "smiless_decode",
           "smiless_kernel_source", "smiless_jit_compile")


class SmilessError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"{_NAMES.get(code, code)}: {msg}")
        self.code = code


class PlanArgs(ctypes.Structure):
    _fields_ = [
        ("arrivals_us", ctypes.c_void_p),
        ("n_arrivals", ctypes.c_int64),
        ("sla_us", ctypes.c_int64),
        ("windows_us", ctypes.c_void_p),
        ("n_windows", ctypes.c_int32),
        ("n_fixed", ctypes.c_int32),
        ("fixed_digits", ctypes.c_void_p),
        ("begin", ctypes.c_uint64),
        ("end", ctypes.c_uint64),
        ("flags", ctypes.c_uint32),
        ("shard", ctypes.c_int32),
        ("n_shards", ctypes.c_int32),
        ("cost_out", ctypes.c_void_p),
        ("row_windows_us", ctypes.c_void_p),
        ("cost_cap", ctypes.c_double),
        ("instances", ctypes.c_void_p),
    ]


class PlanResultC(ctypes.Structure):
    _fields_ = [
        ("index", ctypes.c_uint64),
        ("cost", ctypes.c_double),
        ("max_latency_us", ctypes.c_int64),
        ("n_decided", ctypes.c_uint64),
        ("n_full_evals", ctypes.c_uint64),
        ("eval_kernel_ms", ctypes.c_double),
        ("total_device_ms", ctypes.c_double),
        ("int64_path", ctypes.c_int32),
        ("launches", ctypes.c_int32),
        ("h2d_bytes", ctypes.c_uint64),
        ("d2h_bytes", ctypes.c_uint64),
        ("eval_path", ctypes.c_int32),
        ("n_decided_hi", ctypes.c_uint32),
    ]


# int (*smiless_path_reduce_fn)(void *user, int32_t path, smiless_plan_result *res)
PATH_REDUCE_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_int32, ctypes.POINTER(PlanResultC))


@dataclasses.dataclass
class PlanResult:
    status: int                 # OK or INFEASIBLE
    index: Optional[int]
    cost: float
    max_latency_us: int
    config: np.ndarray
    window: np.ndarray
    n_decided: int
    n_full_evals: int
    eval_kernel_ms: float
    total_device_ms: float
    int64_path: bool
    launches: int
    h2d_bytes: int = 0          # host -> device bytes the call copied (counted by the library)
    d2h_bytes: int = 0          # device -> host bytes the call copied
    eval_path: int = 0          # PATH_* (which evaluator path decided the range)
    digit: Optional[int] = None  # plan_digits: the winner's value of the last pinned digit

    @property
    def feasible(self) -> bool:
        return self.status == OK


_lib = None


def load_library(build_if_missing: bool = True):
    """Load libsmiless.so (building it in-tree with nvcc when missing or stale)."""
    global _lib
    if _lib is not None:
        return _lib
    if build_if_missing:
        from . import build as _build
        if _build.stale():
            _build.build()
    lib = ctypes.CDLL(LIB_PATH)
    vp, i32, i64, u64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_uint64
    lib.smiless_create.argtypes = [ctypes.POINTER(vp), ctypes.c_int, vp]
    lib.smiless_set_stream.argtypes = [vp, vp]
    lib.smiless_destroy.argtypes = [vp]
    lib.smiless_destroy.restype = None
    lib.smiless_last_error.argtypes = [vp]
    lib.smiless_last_error.restype = ctypes.c_char_p
    lib.smiless_load_dag.argtypes = [vp, i32, vp, vp]
    lib.smiless_load_profiles.argtypes = [vp, vp, vp, vp, vp]
    lib.smiless_space_size.argtypes = [vp, i32, i32, ctypes.POINTER(u64)]
    lib.smiless_plan.argtypes = [vp, ctypes.POINTER(PlanArgs), ctypes.POINTER(PlanResultC), vp, vp]
    lib.smiless_plan_digits.argtypes = [vp, ctypes.POINTER(PlanArgs), i32, i32, ctypes.POINTER(PlanResultC),
                                        ctypes.POINTER(ctypes.c_int32), vp, vp]
    lib.smiless_plan_sla_sweep.argtypes = [vp, ctypes.POINTER(PlanArgs), vp, i32, ctypes.POINTER(PlanResultC),
                                           vp, vp]
    lib.smiless_derive_windows.argtypes = [vp, i64, vp]
    lib.smiless_autoscale.argtypes = [vp, vp, vp, vp, i64, vp, vp]
    lib.smiless_autoscale_rows.argtypes = [vp, vp, vp, vp, vp, vp, vp]
    lib.smiless_decompose_search.argtypes = [vp, ctypes.POINTER(PlanArgs), i64, ctypes.POINTER(PlanResultC), vp,
                                             vp, ctypes.POINTER(ctypes.c_int64)]
    lib.smiless_top1_search.argtypes = [vp, ctypes.POINTER(PlanArgs), i64, ctypes.POINTER(PlanResultC), vp, vp,
                                        ctypes.POINTER(ctypes.c_int64)]
    lib.smiless_decompose_plan.argtypes = [vp, ctypes.POINTER(PlanArgs), ctypes.POINTER(PlanResultC), vp, vp,
                                           ctypes.POINTER(ctypes.c_int64)]
    lib.smiless_decompose_plan_sharded.argtypes = [vp, ctypes.POINTER(PlanArgs), PATH_REDUCE_FN, vp,
                                                   ctypes.POINTER(PlanResultC), vp, vp, ctypes.POINTER(ctypes.c_int64)]
    lib.smiless_evaluate.argtypes = [vp, ctypes.POINTER(PlanArgs), vp, i64, vp, vp, vp]
    lib.smiless_decode.argtypes = [vp, i32, u64, ctypes.POINTER(PlanArgs), vp, vp]
    lib.smiless_kernel_source.argtypes = [vp, ctypes.POINTER(PlanArgs), ctypes.c_char_p, ctypes.c_size_t,
                                          ctypes.POINTER(ctypes.c_size_t)]
    lib.smiless_jit_compile.argtypes = [vp, ctypes.POINTER(PlanArgs), ctypes.c_char_p, ctypes.c_size_t,
                                        vp, ctypes.c_size_t, ctypes.POINTER(ctypes.c_size_t)]
    for name in EXPORTS:
        if name not in ("smiless_destroy", "smiless_last_error"):
            getattr(lib, name).restype = ctypes.c_int
    _lib = lib
    return lib


def _i32(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.int32))


def _is_device_tensor(x) -> bool:
    return hasattr(x, "is_cuda") and bool(getattr(x, "is_cuda"))


class Planner:
    """One smiless_ctx (one per host thread / GPU)."""

    def __init__(self, device: int = 0, stream: Optional[int] = None):
        self._lib = load_library()
        self._ctx = ctypes.c_void_p()
        rc = self._lib.smiless_create(ctypes.byref(self._ctx), int(device), ctypes.c_void_p(stream or 0))
        if rc != OK:
            raise SmilessError(rc, self._lib.smiless_last_error(None).decode())
        self._keep = []
        self.n_funcs = 0
        self.default_instances = None    # scale-out instances used when a call passes none

    def close(self):
        if self._ctx:
            self._lib.smiless_destroy(self._ctx)
            self._ctx = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def _check(self, rc: int, allow=(OK,)) -> int:
        if rc not in allow:
            raise SmilessError(rc, self._lib.smiless_last_error(self._ctx).decode())
        return rc

    def set_stream(self, stream: int):
        self._check(self._lib.smiless_set_stream(self._ctx, ctypes.c_void_p(stream)))

    # ---- loads ---------------------------------------------------------------------------
    def load_dag(self, pred_ptr: Sequence[int], pred_idx: Sequence[int]):
        ptr = _i32(pred_ptr)
        idx = _i32(pred_idx) if len(pred_idx) else np.zeros(1, np.int32)
        n = int(ptr.shape[0] - 1)
        self._check(self._lib.smiless_load_dag(self._ctx, n, ptr.ctypes.data,
                                               idx.ctypes.data if len(pred_idx) else None))
        self.n_funcs = n

    def load_profiles(self, n_configs, exec_us, init_us, price_per_us):
        m, e, t = _i32(n_configs), _i32(exec_us), _i32(init_us)
        self._n_rows = int(m.sum())
        u = np.ascontiguousarray(np.asarray(price_per_us, dtype=np.float64))
        self._check(self._lib.smiless_load_profiles(self._ctx, m.ctypes.data, e.ctypes.data, t.ctypes.data,
                                                    u.ctypes.data))

    # ---- args ----------------------------------------------------------------------------
    def _args(self, arrivals, sla_us, windows_us, n_fixed=0, fixed_digits=(), begin=0, end=0, flags=0,
              shard=0, n_shards=0, cost_out=None, row_windows=None, cost_cap=None, instances=None):
        if instances is None:
            instances = self.default_instances
        keep = []
        if _is_device_tensor(arrivals):
            import torch
            assert arrivals.dtype == torch.int64 and arrivals.is_contiguous()
            ptr = arrivals.data_ptr()
            n = int(arrivals.numel())
            flags |= FLAG_ARRIVALS_ON_DEVICE
            keep.append(arrivals)
        else:
            arr = np.ascontiguousarray(np.asarray(arrivals, dtype=np.int64))
            keep.append(arr)
            ptr, n = arr.ctypes.data, int(arr.shape[0])
        win = _i32(windows_us)
        fixed = _i32(list(fixed_digits) or [0])
        keep += [win, fixed]
        a = PlanArgs(arrivals_us=ptr, n_arrivals=n, sla_us=int(sla_us), windows_us=win.ctypes.data,
                     n_windows=int(win.shape[0]), n_fixed=int(n_fixed),
                     fixed_digits=fixed.ctypes.data if n_fixed else None, begin=int(begin), end=int(end),
                     flags=int(flags), shard=int(shard), n_shards=int(n_shards),
                     cost_out=cost_out.ctypes.data if cost_out is not None else None)
        if cost_cap is not None:
            a.flags |= FLAG_COST_CAP
            a.cost_cap = float(cost_cap)
        if row_windows is not None:
            rw = _i32(row_windows)
            keep.append(rw)
            a.row_windows_us = rw.ctypes.data
        if instances is not None:
            ins = _i32(instances)
            keep.append(ins)
            a.instances = ins.ctypes.data
        if cost_out is not None:
            assert cost_out.dtype == np.float64 and cost_out.flags.c_contiguous
            keep.append(cost_out)
        return a, keep

    # ---- API -----------------------------------------------------------------------------
    def derive_windows(self, it_us: int) -> np.ndarray:
        """The paper's adaptive pre-warm window per (function, config) row for a predicted
        inter-arrival time (smiless_derive_windows)."""
        n = int(self._n_rows)
        out = np.zeros(n, np.int32)
        self._check(self._lib.smiless_derive_windows(self._ctx, int(it_us), out.ctypes.data))
        return out

    def autoscale(self, slope_us, intercept_us, invocations, it_us, target_us):
        """The paper's auto-scaler (smiless_autoscale, Eq. (7)/(8)): per function
        (config, batch B, instances, cost)."""
        sl = np.ascontiguousarray(np.asarray(slope_us, dtype=np.float64))
        ic = np.ascontiguousarray(np.asarray(intercept_us, dtype=np.float64))
        G = np.ascontiguousarray(np.asarray(invocations, dtype=np.int64))
        tg = np.ascontiguousarray(np.asarray(target_us, dtype=np.int64))
        out = np.zeros(self.n_funcs, dtype=np.dtype([("config", np.int32), ("batch", np.int64),
                                                      ("instances", np.int64), ("cost", np.float64)], align=True))
        self._check(self._lib.smiless_autoscale(self._ctx, sl.ctypes.data, ic.ctypes.data, G.ctypes.data,
                                                int(it_us), tg.ctypes.data, out.ctypes.data))
        return out

    def autoscale_rows(self, slope_us, intercept_us, invocations, target_us):
        """Eq. (7)/(8) per (function, configuration) row (smiless_autoscale_rows): the largest
        batch B and the instances ceil(G/B) (0, 0 when infeasible)."""
        sl = np.ascontiguousarray(np.asarray(slope_us, dtype=np.float64))
        ic = np.ascontiguousarray(np.asarray(intercept_us, dtype=np.float64))
        G = np.ascontiguousarray(np.asarray(invocations, dtype=np.int64))
        tg = np.ascontiguousarray(np.asarray(target_us, dtype=np.int64))
        b = np.zeros(self._n_rows, np.int64)
        n = np.zeros(self._n_rows, np.int64)
        self._check(self._lib.smiless_autoscale_rows(self._ctx, sl.ctypes.data, ic.ctypes.data, G.ctypes.data,
                                                     tg.ctypes.data, b.ctypes.data, n.ctypes.data))
        return b, n

    def space_size(self, n_windows: int, n_fixed: int = 0) -> int:
        out = ctypes.c_uint64()
        self._check(self._lib.smiless_space_size(self._ctx, int(n_windows), int(n_fixed), ctypes.byref(out)))
        return int(out.value)

    def plan(self, arrivals, sla_us, windows_us, **kw) -> PlanResult:
        a, keep = self._args(arrivals, sla_us, windows_us, **kw)
        r = PlanResultC()
        cfg = np.zeros(max(self.n_funcs, 1), np.int32)
        win = np.zeros(max(self.n_funcs, 1), np.int32)
        rc = self._check(self._lib.smiless_plan(self._ctx, ctypes.byref(a), ctypes.byref(r), cfg.ctypes.data,
                                                win.ctypes.data), allow=(OK, INFEASIBLE))
        del keep
        return PlanResult(status=rc, index=None if rc == INFEASIBLE else int(r.index), cost=float(r.cost),
                          max_latency_us=int(r.max_latency_us), config=cfg[:self.n_funcs],
                          window=win[:self.n_funcs], n_decided=int(r.n_decided), n_full_evals=int(r.n_full_evals),
                          eval_kernel_ms=float(r.eval_kernel_ms), total_device_ms=float(r.total_device_ms),
                          int64_path=bool(r.int64_path), launches=int(r.launches),
                          h2d_bytes=int(r.h2d_bytes), d2h_bytes=int(r.d2h_bytes), eval_path=int(r.eval_path))

    def plan_digits(self, arrivals, sla_us, windows_us, d_begin: int, d_end: int, **kw) -> PlanResult:
        """Every value of the last pinned digit in [d_begin, d_end), one after the other in one
        call with the incumbent carried on the device (smiless_plan_digits).  kw as plan();
        n_fixed >= 1 and fixed_digits required (the last one is ignored).  n_decided sums all
        digits (it may exceed 2^64); .digit is the winner's digit."""
        a, keep = self._args(arrivals, sla_us, windows_us, **kw)
        r = PlanResultC()
        dg = ctypes.c_int32(-1)
        cfg = np.zeros(max(self.n_funcs, 1), np.int32)
        win = np.zeros(max(self.n_funcs, 1), np.int32)
        rc = self._check(self._lib.smiless_plan_digits(self._ctx, ctypes.byref(a), int(d_begin), int(d_end),
                                                       ctypes.byref(r), ctypes.byref(dg), cfg.ctypes.data,
                                                       win.ctypes.data), allow=(OK, INFEASIBLE))
        del keep
        return PlanResult(status=rc, index=None if rc == INFEASIBLE else int(r.index), cost=float(r.cost),
                          max_latency_us=int(r.max_latency_us), config=cfg[:self.n_funcs],
                          window=win[:self.n_funcs], n_decided=int(r.n_decided) + (int(r.n_decided_hi) << 64),
                          n_full_evals=int(r.n_full_evals), eval_kernel_ms=float(r.eval_kernel_ms),
                          total_device_ms=float(r.total_device_ms), int64_path=bool(r.int64_path),
                          launches=int(r.launches), h2d_bytes=int(r.h2d_bytes), d2h_bytes=int(r.d2h_bytes),
                          eval_path=int(r.eval_path), digit=None if rc == INFEASIBLE else int(dg.value))

    def plan_sla_sweep(self, arrivals, slas_us, windows_us, **kw):
        """One pass over the space, one winner per SLA (smiless_plan_sla_sweep)."""
        sl = np.ascontiguousarray(np.asarray(slas_us, dtype=np.int64))
        n = int(sl.shape[0])
        a, keep = self._args(arrivals, int(sl.max()), windows_us, **kw)
        rs = (PlanResultC * n)()
        cfg = np.zeros((n, max(self.n_funcs, 1)), np.int32)
        win = np.zeros((n, max(self.n_funcs, 1)), np.int32)
        self._check(self._lib.smiless_plan_sla_sweep(self._ctx, ctypes.byref(a), sl.ctypes.data, n, rs,
                                                     cfg.ctypes.data, win.ctypes.data))
        del keep
        out = []
        for i, r in enumerate(rs):
            feas = r.index != (1 << 64) - 1
            out.append(PlanResult(status=OK if feas else INFEASIBLE, index=int(r.index) if feas else None,
                                  cost=float(r.cost), max_latency_us=int(r.max_latency_us),
                                  config=cfg[i, :self.n_funcs], window=win[i, :self.n_funcs],
                                  n_decided=int(r.n_decided), n_full_evals=int(r.n_full_evals),
                                  eval_kernel_ms=float(r.eval_kernel_ms), total_device_ms=float(r.total_device_ms),
                                  int64_path=bool(r.int64_path), launches=int(r.launches)))
        return out

    def top1_search(self, arrivals, sla_us, it_us, row_windows, **kw):
        """SMIless's Top-1 path search (smiless_top1_search); returns (PlanResult, nodes)."""
        a, keep = self._args(arrivals, sla_us, [0], row_windows=row_windows, **kw)
        r = PlanResultC()
        cfg = np.zeros(max(self.n_funcs, 1), np.int32)
        win = np.zeros(max(self.n_funcs, 1), np.int32)
        nodes = ctypes.c_int64()
        rc = self._check(self._lib.smiless_top1_search(self._ctx, ctypes.byref(a), int(it_us), ctypes.byref(r),
                                                       cfg.ctypes.data, win.ctypes.data, ctypes.byref(nodes)),
                         allow=(OK, INFEASIBLE))
        del keep
        return PlanResult(status=rc, index=None if rc == INFEASIBLE else int(r.index), cost=float(r.cost),
                          max_latency_us=int(r.max_latency_us), config=cfg[:self.n_funcs],
                          window=win[:self.n_funcs], n_decided=int(r.n_decided), n_full_evals=int(r.n_full_evals),
                          eval_kernel_ms=0.0, total_device_ms=0.0, int64_path=False, launches=0), int(nodes.value)

    def decompose_search(self, arrivals, sla_us, it_us, row_windows, **kw):
        """SMIless's DAG decomposition + combine (smiless_decompose_search); (PlanResult, paths)."""
        a, keep = self._args(arrivals, sla_us, [0], row_windows=row_windows, **kw)
        r = PlanResultC()
        cfg = np.zeros(max(self.n_funcs, 1), np.int32)
        win = np.zeros(max(self.n_funcs, 1), np.int32)
        n = ctypes.c_int64()
        rc = self._check(self._lib.smiless_decompose_search(self._ctx, ctypes.byref(a), int(it_us), ctypes.byref(r),
                                                            cfg.ctypes.data, win.ctypes.data, ctypes.byref(n)),
                         allow=(OK, INFEASIBLE))
        del keep
        return PlanResult(status=rc, index=None if rc == INFEASIBLE else int(r.index), cost=float(r.cost),
                          max_latency_us=int(r.max_latency_us), config=cfg[:self.n_funcs],
                          window=win[:self.n_funcs], n_decided=1, n_full_evals=1, eval_kernel_ms=0.0,
                          total_device_ms=0.0, int64_path=False, launches=0), int(n.value)

    def decompose_plan(self, arrivals, sla_us, windows_us, reduce=None, **kw):
        """NEXT-3 with model M (smiless_decompose_plan): exhaustive GPU plan per source-to-sink
        path, the paper's combine; returns (PlanResult, number of paths).  With `reduce`
        (a callable (path, PlanResultC) -> None that replaces the result's index / cost /
        max_latency_us with the ranks' global winner) and shard / n_shards in kw, the path
        plans are sharded over ranks (smiless_decompose_plan_sharded)."""
        a, keep = self._args(arrivals, sla_us, windows_us, **kw)
        r = PlanResultC()
        cfg = np.zeros(max(self.n_funcs, 1), np.int32)
        win = np.zeros(max(self.n_funcs, 1), np.int32)
        npaths = ctypes.c_int64()
        if reduce is None:
            rc = self._check(self._lib.smiless_decompose_plan(self._ctx, ctypes.byref(a), ctypes.byref(r),
                                                              cfg.ctypes.data, win.ctypes.data, ctypes.byref(npaths)),
                             allow=(OK, INFEASIBLE))
        else:
            def _cb(user, path, res_p):
                try:
                    reduce(int(path), res_p.contents)
                    return 0
                except Exception:               # pragma: no cover  (reported as EINVAL by the library)
                    return 1
            cb = PATH_REDUCE_FN(_cb)
            rc = self._check(self._lib.smiless_decompose_plan_sharded(self._ctx, ctypes.byref(a), cb, None,
                                                                      ctypes.byref(r), cfg.ctypes.data,
                                                                      win.ctypes.data, ctypes.byref(npaths)),
                             allow=(OK, INFEASIBLE))
        del keep
        return PlanResult(status=rc, index=None if rc == INFEASIBLE else int(r.index), cost=float(r.cost),
                          max_latency_us=int(r.max_latency_us), config=cfg[:self.n_funcs],
                          window=win[:self.n_funcs], n_decided=int(r.n_decided), n_full_evals=int(r.n_full_evals),
                          eval_kernel_ms=0.0, total_device_ms=0.0, int64_path=False, launches=0), int(npaths.value)

    def evaluate(self, idx, arrivals, sla_us, windows_us, **kw) -> Tuple[np.ndarray, np.ndarray, np.ndarray]:
        a, keep = self._args(arrivals, sla_us, windows_us, **kw)
        ix = np.ascontiguousarray(np.asarray(idx, dtype=np.uint64).reshape(-1))
        n = int(ix.shape[0])
        cost = np.zeros(n, np.float64)
        lat = np.zeros(n, np.int64)
        feas = np.zeros(n, np.uint8)
        self._check(self._lib.smiless_evaluate(self._ctx, ctypes.byref(a), ix.ctypes.data, n, cost.ctypes.data,
                                               lat.ctypes.data, feas.ctypes.data))
        del keep
        return cost, lat, feas.astype(bool)

    def decode(self, index: int, n_windows: int, n_fixed: int = 0, fixed_digits=()):
        fixed = _i32(list(fixed_digits) or [0])
        a = PlanArgs(n_fixed=int(n_fixed), fixed_digits=fixed.ctypes.data if n_fixed else None)
        c = np.zeros(self.n_funcs, np.int32)
        w = np.zeros(self.n_funcs, np.int32)
        self._check(self._lib.smiless_decode(self._ctx, int(n_windows), int(index), ctypes.byref(a),
                                             c.ctypes.data, w.ctypes.data))
        return c, w

    def kernel_source(self, arrivals, sla_us, windows_us, **kw) -> str:
        a, keep = self._args(arrivals, sla_us, windows_us, **kw)
        n = ctypes.c_size_t()
        self._check(self._lib.smiless_kernel_source(self._ctx, ctypes.byref(a), None, 0, ctypes.byref(n)))
        buf = ctypes.create_string_buffer(n.value)
        self._check(self._lib.smiless_kernel_source(self._ctx, ctypes.byref(a), buf, n.value, ctypes.byref(n)))
        return buf.value.decode()

    def jit_compile(self, arrivals, sla_us, windows_us, want_cubin: bool = False, **kw):
        """NVRTC-compile the specialised evaluator (no GPU needed).

        Returns (ptxas log, cubin size) or, with want_cubin, (ptxas log, cubin bytes)."""
        a, keep = self._args(arrivals, sla_us, windows_us, **kw)
        log = ctypes.create_string_buffer(1 << 16)
        n = ctypes.c_size_t()
        cap = 8 << 20 if want_cubin else 0
        buf = ctypes.create_string_buffer(cap) if want_cubin else None
        self._check(self._lib.smiless_jit_compile(self._ctx, ctypes.byref(a), log, 1 << 16,
                                                  buf if want_cubin else None, cap, ctypes.byref(n)))
        if want_cubin:
            return log.value.decode(), buf.raw[:n.value]
        return log.value.decode(), int(n.value)


def planner_for(problem, device: int = 0, stream: Optional[int] = None) -> Planner:
    """Planner with a workloads.Problem-like object's DAG and profiles loaded; the problem's
    scale-out instance counts (if any) become the default `instances` of every call."""
    p = Planner(device, stream)
    p.default_instances = getattr(problem, "instances", None)
    p.load_dag(problem.pred_ptr, problem.pred_idx)
    p.load_profiles(problem.n_configs, problem.exec_us, problem.init_us, problem.price_per_us)
    return p
