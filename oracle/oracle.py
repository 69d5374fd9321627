"""ctypes front-end of the plain C oracle (oracle/smiless_oracle.c).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and
bench.py's cpu_baseline / --impl reference legs, never by the product path
(paper_conf_sc_luxl0y024_b200/).  It shares no code with the CUDA path; the
only thing both sides consume is the seeded input data from `workloads`.

What each function computes is documented (with PAPER.md citations) in
smiless_oracle.c.  Parity status of each part is listed in DESIGN.md
("Oracle pins").
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import Optional, Sequence, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "smiless_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")


def build(force: bool = False) -> str:
    """Compile the oracle with gcc: -O2, no intrinsics, no FMA contraction."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math",
                               "-fPIC", "-shared", "-pthread", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


class _Problem(ctypes.Structure):
    _fields_ = [
        ("n_funcs", ctypes.c_int32),
        ("pred_ptr", ctypes.c_void_p),
        ("pred_idx", ctypes.c_void_p),
        ("n_configs", ctypes.c_void_p),
        ("exec_us", ctypes.c_void_p),
        ("init_us", ctypes.c_void_p),
        ("price_per_us", ctypes.c_void_p),
        ("arrivals_us", ctypes.c_void_p),
        ("n_arrivals", ctypes.c_int64),
        ("sla_us", ctypes.c_int64),
        ("windows_us", ctypes.c_void_p),
        ("n_windows", ctypes.c_int32),
        ("n_fixed", ctypes.c_int32),
        ("fixed_digits", ctypes.c_void_p),
        ("row_windows", ctypes.c_void_p),
        ("instances", ctypes.c_void_p),
    ]


_lib = None


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        lib.oracle_space_size.restype = ctypes.c_uint64
        lib.oracle_space_size.argtypes = [ctypes.POINTER(_Problem)]
        lib.oracle_decode.restype = None
        lib.oracle_decode.argtypes = [ctypes.POINTER(_Problem), ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p]
        lib.oracle_simulate.restype = ctypes.c_int
        lib.oracle_simulate.argtypes = [ctypes.POINTER(_Problem), ctypes.c_void_p, ctypes.c_void_p,
                                        ctypes.c_void_p, ctypes.c_void_p]
        lib.oracle_evaluate.restype = ctypes.c_int
        lib.oracle_evaluate.argtypes = [ctypes.POINTER(_Problem), ctypes.c_void_p, ctypes.c_int64,
                                        ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]
        lib.oracle_plan.restype = ctypes.c_int
        lib.oracle_plan.argtypes = [ctypes.POINTER(_Problem), ctypes.c_uint64, ctypes.c_uint64, ctypes.c_int,
                                    ctypes.POINTER(ctypes.c_uint64), ctypes.POINTER(ctypes.c_double),
                                    ctypes.POINTER(ctypes.c_int64)]
        _lib = lib
    return _lib


class OracleProblem:
    """Holds contiguous copies of a workloads.Problem for the C oracle."""

    def __init__(self, prob, sla_us: Optional[int] = None, n_fixed: int = 0,
                 fixed_digits: Sequence[int] = (), row_windows: Optional[Sequence[int]] = None,
                 instances: Optional[Sequence[int]] = None):
        if instances is None:
            instances = getattr(prob, "instances", None)   # the workload's scale-out counts
        """row_windows (optional, [sum M]): the window of each (function, config) row, used
        instead of the grid (windows_us must then hold a single entry) -- the paper's
        derived pre-warm windows (NEXT-1).  instances (optional, [N]): n_k round-robin
        instances per function (NEXT-4 scale-out, reading G26); None = one each."""
        self.keep = dict(
            pred_ptr=np.ascontiguousarray(prob.pred_ptr, dtype=np.int32),
            pred_idx=np.ascontiguousarray(prob.pred_idx, dtype=np.int32) if len(prob.pred_idx) else np.zeros(1, np.int32),
            n_configs=np.ascontiguousarray(prob.n_configs, dtype=np.int32),
            exec_us=np.ascontiguousarray(prob.exec_us, dtype=np.int32),
            init_us=np.ascontiguousarray(prob.init_us, dtype=np.int32),
            price=np.ascontiguousarray(prob.price_per_us, dtype=np.float64),
            arrivals=np.ascontiguousarray(prob.arrivals_us, dtype=np.int64),
            windows=np.ascontiguousarray(prob.windows_us, dtype=np.int32),
            fixed=np.ascontiguousarray(np.asarray(list(fixed_digits) or [0], dtype=np.int32)),
            roww=None if row_windows is None else np.ascontiguousarray(np.asarray(row_windows, dtype=np.int32)),
            inst=None if instances is None else np.ascontiguousarray(np.asarray(instances, dtype=np.int32)),
        )
        if instances is not None:
            assert len(self.keep["inst"]) == int(prob.pred_ptr.shape[0] - 1)
        if row_windows is not None:
            assert len(prob.windows_us) == 1 and len(self.keep["roww"]) == int(np.sum(prob.n_configs))
        k = self.keep
        self.n_funcs = int(k["pred_ptr"].shape[0] - 1)
        self.n_arrivals = int(k["arrivals"].shape[0])
        self.s = _Problem(
            n_funcs=self.n_funcs,
            pred_ptr=k["pred_ptr"].ctypes.data, pred_idx=k["pred_idx"].ctypes.data,
            n_configs=k["n_configs"].ctypes.data, exec_us=k["exec_us"].ctypes.data,
            init_us=k["init_us"].ctypes.data, price_per_us=k["price"].ctypes.data,
            arrivals_us=k["arrivals"].ctypes.data, n_arrivals=self.n_arrivals,
            sla_us=int(prob.sla_us if sla_us is None else sla_us),
            windows_us=k["windows"].ctypes.data, n_windows=int(k["windows"].shape[0]),
            n_fixed=int(n_fixed), fixed_digits=k["fixed"].ctypes.data,
            row_windows=None if k["roww"] is None else k["roww"].ctypes.data,
            instances=None if k["inst"] is None else k["inst"].ctypes.data)

    # -- API ---------------------------------------------------------------
    def space_size(self) -> int:
        return int(_load().oracle_space_size(ctypes.byref(self.s)))

    def decode(self, index: int) -> Tuple[np.ndarray, np.ndarray]:
        c = np.zeros(self.n_funcs, np.int32)
        w = np.zeros(self.n_funcs, np.int32)
        _load().oracle_decode(ctypes.byref(self.s), int(index), c.ctypes.data, w.ctypes.data)
        return c, w

    def simulate(self, config: Sequence[int], window: Sequence[int]) -> Tuple[np.ndarray, np.ndarray]:
        """(billed[N] int64 us, latency[J] int64 us) for explicit config/window-index vectors."""
        c = np.ascontiguousarray(config, dtype=np.int32)
        w = np.ascontiguousarray(window, dtype=np.int32)
        billed = np.zeros(self.n_funcs, np.int64)
        lat = np.zeros(self.n_arrivals, np.int64)
        rc = _load().oracle_simulate(ctypes.byref(self.s), c.ctypes.data, w.ctypes.data,
                                     billed.ctypes.data, lat.ctypes.data)
        if rc != 0:
            raise ValueError("oracle_simulate: bad arguments")
        return billed, lat

    def evaluate(self, idx) -> Tuple[np.ndarray, np.ndarray, np.ndarray]:
        """(cost f64, max latency int64, feasible bool) per candidate index."""
        ix = np.ascontiguousarray(np.asarray(idx, dtype=np.uint64).reshape(-1))
        n = ix.shape[0]
        cost = np.zeros(n, np.float64)
        lat = np.zeros(n, np.int64)
        feas = np.zeros(n, np.uint8)
        rc = _load().oracle_evaluate(ctypes.byref(self.s), ix.ctypes.data, n, cost.ctypes.data,
                                     lat.ctypes.data, feas.ctypes.data)
        if rc != 0:
            raise ValueError("oracle_evaluate: bad arguments")
        return cost, lat, feas.astype(bool)

    def plan(self, begin: int = 0, end: int = 0, n_threads: Optional[int] = None):
        """Brute-force OPT over [begin, end): (index, cost, max latency) or None if infeasible."""
        if n_threads is None:
            n_threads = os.cpu_count() or 1
        bi = ctypes.c_uint64(0)
        bc = ctypes.c_double(0.0)
        bl = ctypes.c_int64(0)
        rc = _load().oracle_plan(ctypes.byref(self.s), int(begin), int(end), int(n_threads),
                                 ctypes.byref(bi), ctypes.byref(bc), ctypes.byref(bl))
        if rc < 0:
            raise ValueError("oracle_plan: bad arguments")
        if rc == 0:
            return None
        return int(bi.value), float(bc.value), int(bl.value)
