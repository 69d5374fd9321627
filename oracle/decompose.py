"""SMIless's DAG decomposition + combine, step by step -- TEST
INFRASTRUCTURE ONLY (the oracle of smiless_decompose_search).

1. Decompose the DAG into its source-to-sink paths ("subgraphs that only contain
   sequential dependency"), in DFS order from each source.
2. Optimise each path with the Top-1 walk using the paper's O(1)
   closed form (Eq. (5)): path latency = sum of I, per-invocation cost
   U (T + I) in Case I / U IT in Case II; ties by lower config.
3. Combine (reading G25): a function on several paths takes the fastest of
   the paths' choices (the rule for F_s / F_e of a parallel substructure); each function
   on one path only moves to its cheapest config keeping that path's closed-form latency
   at or below its latency before combining (paths visited in order).
4. The combined plan is evaluated with model M (the C oracle).
"""
from __future__ import annotations

import numpy as np


def decompose_search(prob, it_us: int, row_windows, oracle_cls, trace=None):
    """Returns (configs, cost, max latency, feasible, number of paths).  If `trace` is a
    dict it receives the steps: "paths", "path_choices" (each path's Top-1 result, configs
    in path order), "path_latency" (closed form before combining), "combined"."""
    n = prob.n_funcs
    M = [int(m) for m in prob.n_configs]
    off = np.concatenate([[0], np.cumsum(prob.n_configs)]).astype(int)
    preds = [prob.preds(k) for k in range(n)]
    succ = [[] for _ in range(n)]
    for k in range(n):
        for q in preds[k]:
            succ[q].append(k)
    paths = []

    def walk(k, cur):
        cur = cur + [k]
        if not succ[k]:
            paths.append(cur)
        for s in succ[k]:
            walk(s, cur)

    for k in range(n):
        if not preds[k]:
            walk(k, [])

    def I(k, m):
        return int(prob.exec_us[off[k] + m])

    def cost(k, m):
        t, i = int(prob.init_us[off[k] + m]), I(k, m)
        return float(prob.price_per_us[off[k] + m]) * (float(t + i) if t + i < it_us else float(it_us))

    rank = [sorted(range(M[k]), key=lambda m, k=k: cost(k, m)) for k in range(n)]
    fastest = [min(range(M[k]), key=lambda m, k=k: (I(k, m), m)) for k in range(n)]
    sla = prob.sla_us
    choice = []
    for P in paths:
        c = [rank[k][0] for k in P]
        if sum(I(k, m) for k, m in zip(P, c)) > sla:
            chosen = []
            for q, k in enumerate(P):
                pick = fastest[k]
                for r in range(1 if q == 0 else 0, M[k]):
                    trial = chosen + [rank[k][r]] + [fastest[z] for z in P[q + 1:]]
                    if sum(I(z, m) for z, m in zip(P, trial)) <= sla:
                        pick = rank[k][r]
                        break
                chosen.append(pick)
            c = chosen
        choice.append(c)
    cfg = [-1] * n
    n_on = [0] * n
    path_lat = []
    for P, c in zip(paths, choice):
        path_lat.append(sum(I(k, m) for k, m in zip(P, c)))
        for k, m in zip(P, c):
            n_on[k] += 1
            if cfg[k] < 0 or I(k, m) < I(k, cfg[k]):
                cfg[k] = m
    for P, pl in zip(paths, path_lat):
        for q, k in enumerate(P):
            if n_on[k] != 1:
                continue
            others = sum(I(z, cfg[z]) for i, z in enumerate(P) if i != q)
            for r in range(M[k]):
                if others + I(k, rank[k][r]) <= pl:
                    cfg[k] = rank[k][r]
                    break
    if trace is not None:
        trace.update(paths=[list(P) for P in paths], path_choices=[list(c) for c in choice],
                     path_latency=list(path_lat), combined=list(cfg))
    o = oracle_cls(prob, row_windows=row_windows)
    idx = 0
    for k in range(n):
        idx = idx * M[k] + cfg[k]
    c, l, f = o.evaluate([idx])
    return cfg, float(c[0]), int(l[0]), bool(f[0]), len(paths)
