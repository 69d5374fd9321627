"""NEXT-3 with model M: SMIless's DAG decomposition + combine where each
path is optimised exhaustively under model M -- TEST INFRASTRUCTURE ONLY (the oracle of
smiless_decompose_plan).

1. Decompose the DAG into its source-to-sink paths (DFS from each source).
2. Each path: the exhaustive optimum (oracle brute force, lowest index on ties) of the chain
   of the path's functions under model M with the same arrivals, SLA, window grid and
   instances ("executes the basic algorithm ... for each subgraph").
3. Combine (reading G25): a function on several paths takes the
   (configuration, window) with the shortest inference time among the paths' choices (the
   rule for F_s / F_e); then, paths in order and functions in path order, every function on
   one path only takes its cheapest (configuration, window) -- by the path chain's model-M
   cost with the other functions as they stand -- whose path latency stays at or below the
   path's latency before combining (ties: lowest digit).
4. The combined plan is evaluated with model M on the whole DAG.
"""
from __future__ import annotations

import dataclasses

import numpy as np


def _paths(prob):
    n = prob.n_funcs
    preds = [prob.preds(k) for k in range(n)]
    succ = [[] for _ in range(n)]
    for k in range(n):
        for q in preds[k]:
            succ[q].append(k)
    out = []

    def walk(k, cur):
        cur = cur + [k]
        if not succ[k]:
            out.append(cur)
        for s in succ[k]:
            walk(s, cur)

    for k in range(n):
        if not preds[k]:
            walk(k, [])
    return out


def _chain(prob, P, instances):
    off = np.concatenate([[0], np.cumsum(prob.n_configs)]).astype(int)
    rows = np.concatenate([np.arange(off[k], off[k + 1]) for k in P])
    L = len(P)
    ptr = np.asarray([0] + list(range(L)), dtype=np.int32)
    idx = np.asarray(list(range(L - 1)), dtype=np.int32)
    fields = dict(pred_ptr=ptr, pred_idx=idx, n_configs=np.asarray([prob.n_configs[k] for k in P], np.int32),
                  exec_us=np.asarray(prob.exec_us)[rows], init_us=np.asarray(prob.init_us)[rows],
                  price_per_us=np.asarray(prob.price_per_us)[rows],
                  instances=None if instances is None else np.asarray([instances[k] for k in P], np.int32))
    if hasattr(prob, "batch_slope_us"):
        fields.update(batch_slope_us=None, batch_intercept_us=None)
    return dataclasses.replace(prob, **fields)


def decompose_plan(prob, oracle_cls, trace=None):
    """Returns (configs, windows, cost, max latency, feasible, number of paths); `trace` (a
    dict) receives the paths, each path's optimum and latency, and the combined plan."""
    n = prob.n_funcs
    W = len(prob.windows_us)
    inst = getattr(prob, "instances", None)
    off = np.concatenate([[0], np.cumsum(prob.n_configs)]).astype(int)
    paths = _paths(prob)
    pc, pw, plat = [], [], []
    for P in paths:
        sub = _chain(prob, P, inst)
        o = oracle_cls(sub, instances=sub.instances)
        best = o.plan()
        if best is None:
            return [-1] * n, [-1] * n, float("inf"), -1, False, len(paths)
        c, w = o.decode(best[0])
        pc.append([int(v) for v in c])
        pw.append([int(v) for v in w])
        plat.append(best[2])
    cfg, win, n_on = [-1] * n, [-1] * n, [0] * n
    for P, c, w in zip(paths, pc, pw):
        for q, k in enumerate(P):
            n_on[k] += 1
            if cfg[k] < 0 or prob.exec_us[off[k] + c[q]] < prob.exec_us[off[k] + cfg[k]]:
                cfg[k], win[k] = c[q], w[q]
    for P, pl in zip(paths, plat):
        sub = _chain(prob, P, inst)
        o = oracle_cls(sub, instances=sub.instances)
        for q, k in enumerate(P):
            if n_on[k] != 1:
                continue
            R = int(prob.n_configs[k]) * W
            idx = []
            for d in range(R):
                v = 0
                for z, kz in enumerate(P):
                    dz = d if z == q else cfg[kz] * W + win[kz]
                    v = v * (int(prob.n_configs[kz]) * W) + dz
                idx.append(v)
            cost, lat, _ = o.evaluate(idx)
            best = None
            for d in range(R):
                if lat[d] <= pl and (best is None or cost[d] < cost[best]):
                    best = d
            if best is not None:
                cfg[k], win[k] = best // W, best % W
    if trace is not None:
        trace.update(paths=[list(P) for P in paths], path_configs=pc, path_windows=pw, path_latency=plat,
                     combined_configs=list(cfg), combined_windows=list(win))
    o = oracle_cls(prob, instances=inst)
    idx = 0
    for k in range(n):
        idx = idx * (int(prob.n_configs[k]) * W) + cfg[k] * W + win[k]
    c, l, f = o.evaluate([idx])
    return cfg, win, float(c[0]), int(l[0]), bool(f[0]), len(paths)
