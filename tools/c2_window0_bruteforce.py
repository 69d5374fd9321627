#!/usr/bin/env python
"""Oracle brute force of C2's window-0 sub-space (every function keep-alive, P:188-194
Case II "window size zero"): 16^6 = 16,777,216 candidates at J = 10^4, every one
simulated with model M by the plain C oracle (oracle/smiless_oracle.c) -- no pruning,
no GPU, nothing from the CUDA path.

Writes tests/golden/C2_window0_bruteforce.json: the sub-space OPT, its index in the
sub-space (W = 1) and the same candidate's index in the full C2 space (W = 8, window
index 0 = grid value 0), which the GPU tests compare with the full-space plan.

Calls only oracle/ and workloads/ (the seeded inputs).  ~10 min on 8 host cores.
"""
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402
from oracle import OracleProblem  # noqa: E402


def main():
    p = W.make_config("C2")
    p0 = p.replace(windows_us=np.asarray([0], dtype=np.int32))
    o = OracleProblem(p0)
    space = o.space_size()
    assert space == 16 ** 6
    t0 = time.perf_counter()
    best = o.plan(0, 0, n_threads=os.cpu_count())
    dt = time.perf_counter() - t0
    assert best is not None
    idx0, cost, lat = best
    cfg, _ = o.decode(idx0)
    Wn = len(p.windows_us)
    full = 0
    for k in range(p.n_funcs):                      # digit = config * W + window(0)
        full = full * (int(p.n_configs[k]) * Wn) + int(cfg[k]) * Wn
    out = {
        "what": "OPT of C2's window-0 sub-space (all windows = grid value 0, keep-alive) by oracle brute force",
        "cite": "PAPER.md:305 (OPT determined through exhaustive search); P:188-194 (window 0 = keep alive); "
                "SURVEY.md 8(c) oracle definition",
        "workload": "workloads.make_config('C2') with windows_us = [0]",
        "space": space,
        "index_subspace": int(idx0),
        "index_full_space": int(full),
        "config": [int(c) for c in cfg],
        "cost": cost,
        "cost_hex": float(cost).hex(),
        "max_latency_us": int(lat),
        "oracle_seconds": dt,
        "oracle_threads": os.cpu_count(),
        "script": "tools/c2_window0_bruteforce.py (calls only oracle/ and workloads/)",
    }
    path = os.path.join(ROOT, "tests", "golden", "C2_window0_bruteforce.json")
    with open(path, "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
