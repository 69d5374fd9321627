"""SMIless's Top-1 path search (Fig. 6, Eq. (6)), written step by step in
the paper's order -- TEST INFRASTRUCTURE ONLY (the oracle of smiless_top1_search).

Nodes are evaluated with the C oracle (model M) under per-row windows (the paper's
adaptive pre-warming).  Readings (G21-G23):
* per-function cost used for the ordering: U * (T + I) in Case I (T + I < IT), U * IT in
  Case II, ties by lower config index;
* root T^0 = every function on its cheapest config (Eq. 6); if it meets the SLA, stop;
* layer k (function order F_1..F_N): functions before k keep their chosen config, functions
  after k run on their fastest config ("the most advanced hardware", min I), F_k takes its
  configs in increasing cost order, the first node meeting the SLA fixes F_k; layer 1 starts
  at the second cheapest ("T^1_1 ... second smallest"); if no node of a layer
  meets the SLA, F_k stays on its fastest config; the leaf is the answer.
"""
from __future__ import annotations

import numpy as np


def top1_search(prob, it_us: int, row_windows, oracle_cls, trace=None):
    """Returns (leaf configs, cost, max latency, feasible, nodes evaluated).  If `trace` is a
    list, the nodes in the order the paper's walk visits them (each layer
    stops at its first SLA-meeting node) are appended as (layer, configs, meets SLA); layer 0
    is the root T^0."""
    n = prob.n_funcs
    M = [int(m) for m in prob.n_configs]
    off = np.concatenate([[0], np.cumsum(prob.n_configs)]).astype(int)
    rank, fastest = [], []
    for k in range(n):
        costs = []
        for m in range(M[k]):
            r = off[k] + m
            t, i = int(prob.init_us[r]), int(prob.exec_us[r])
            per_inv = float(t + i) if t + i < it_us else float(it_us)
            costs.append((float(prob.price_per_us[r]) * per_inv, m))
        rank.append([m for _, m in sorted(costs, key=lambda x: x[0])])      # stable: ties keep order
        fastest.append(int(np.argmin([int(prob.exec_us[off[k] + m]) for m in range(M[k])])))
    o = oracle_cls(prob, row_windows=row_windows)

    def index_of(cfg):
        idx = 0
        for k in range(n):
            idx = idx * M[k] + cfg[k]
        return idx

    nodes = 0

    def evaluate(cfgs):
        nonlocal nodes
        nodes += len(cfgs)
        return o.evaluate([index_of(c) for c in cfgs])

    root = [rank[k][0] for k in range(n)]
    cost, lat, feas = evaluate([root])
    if trace is not None:
        trace.append((0, list(root), bool(feas[0])))
    if feas[0]:
        return root, float(cost[0]), int(lat[0]), True, nodes
    chosen = []
    for k in range(n):
        layer = []
        for r in range(1 if k == 0 else 0, M[k]):
            layer.append(chosen + [rank[k][r]] + [fastest[q] for q in range(k + 1, n)])
        pick = None
        if layer:
            c, l, f = evaluate(layer)
            for i in range(len(layer)):
                if trace is not None:
                    trace.append((k + 1, list(layer[i]), bool(f[i])))
                if f[i]:
                    pick = layer[i][k]
                    break
        chosen.append(fastest[k] if pick is None else pick)
    cost, lat, feas = evaluate([chosen])
    return chosen, float(cost[0]), int(lat[0]), bool(feas[0]), nodes
