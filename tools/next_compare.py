"""NEXT-1 / NEXT-2 / NEXT-3 on the BASELINE configs: exhaustive OPT over configs x window grid vs
exhaustive OPT under the paper's derived windows (NEXT-1) vs SMIless's Top-1 path search
(NEXT-2, the paper's deployed heuristic) vs DAG decomposition (NEXT-3: closed-form Top-1 per
path, and exhaustive model-M plans per path on the GPU), all exact under model M on one GPU
(C3 / C5 with their scale-out instances, NEXT-4).  This is the
paper's Fig. 8 comparison "SMIless vs OPT (exhaustive search)" on synthetic inputs."""
import json, sys, time
sys.path.insert(0, '.')
import numpy as np
import torch
import workloads as W
from oracle import OracleProblem
from paper_conf_sc_luxl0y024_b200 import smiless as S


def run(name, p, check=True):
    stream = torch.cuda.current_stream().cuda_stream
    pl = S.planner_for(p, stream=stream)
    arr = torch.as_tensor(p.arrivals_us).cuda()
    it = int(np.diff(p.arrivals_us).mean())
    out = {"config": name, "J": len(p.arrivals_us), "IT_us": it}
    t0 = time.perf_counter()
    Wn = len(p.windows_us)
    try:
        full = pl.plan(arr, p.sla_us, p.windows_us)
        space = pl.space_size(Wn)
        fixed = {}
    except S.SmilessError:                       # > 2^63 (C5): pin function 0's digit, 128 sub-plans
        best, space = None, 0
        for d0 in range(int(p.n_configs[0]) * Wn):
            r = pl.plan(arr, p.sla_us, p.windows_us, n_fixed=1, fixed_digits=[d0])
            space += r.n_decided
            if r.feasible and (best is None or (r.cost, d0, r.index) < (best[0].cost, best[1], best[0].index)):
                best = (r, d0)
        full, fixed = best[0], dict(n_fixed=1, fixed_digits=[best[1]])
    out["opt_grid"] = {"cost": full.cost if full.feasible else None, "s": time.perf_counter() - t0,
                       "config": full.config.tolist(), "window": full.window.tolist(), "candidates": space}
    q = p.replace(windows_us=np.array([0], np.int32))
    plq = S.planner_for(q, stream=stream)
    rw = plq.derive_windows(it)
    t0 = time.perf_counter()
    der = plq.plan(arr, q.sla_us, [0], row_windows=rw)
    out["opt_derived_windows"] = {"cost": der.cost if der.feasible else None, "s": time.perf_counter() - t0,
                                  "config": der.config.tolist(), "candidates": plq.space_size(1)}
    t0 = time.perf_counter()
    h, nodes = plq.top1_search(p.arrivals_us, q.sla_us, it, rw)
    out["top1_search"] = {"cost": h.cost if h.feasible else None, "s": time.perf_counter() - t0, "nodes": nodes,
                          "config": h.config.tolist()}
    t0 = time.perf_counter()
    dc, n_paths = plq.decompose_search(p.arrivals_us, q.sla_us, it, rw)
    out["decompose_search"] = {"cost": dc.cost if dc.feasible else None, "s": time.perf_counter() - t0,
                               "paths": n_paths, "config": dc.config.tolist()}
    t0 = time.perf_counter()
    dm, n_paths_m = pl.decompose_plan(arr, p.sla_us, p.windows_us)    # NEXT-3 with model M (GPU per path)
    out["decompose_plan_model_m"] = {"cost": dm.cost if dm.feasible else None, "s": time.perf_counter() - t0,
                                     "paths": n_paths_m, "config": dm.config.tolist(), "window": dm.window.tolist()}
    if dm.feasible:
        pin = dict(n_fixed=1, fixed_digits=[int(dm.config[0]) * Wn + int(dm.window[0])]) if fixed else {}
        c, l, f = OracleProblem(p, **pin).evaluate([dm.index])
        out["decompose_plan_model_m"]["oracle_check"] = bool(f[0] and c[0] == dm.cost and l[0] == dm.max_latency_us)
    if full.feasible and dm.feasible:
        out["decompose_model_m_over_opt"] = dm.cost / full.cost
    if full.feasible and dc.feasible:
        out["decompose_over_opt"] = dc.cost / full.cost
    if full.feasible and h.feasible:
        out["top1_over_opt"] = h.cost / full.cost
    if full.feasible and der.feasible:
        out["derived_over_opt"] = der.cost / full.cost
    if check and full.feasible:
        c, l, f = OracleProblem(p, **fixed).evaluate([full.index])
        out["opt_grid"]["oracle_check"] = bool(f[0] and c[0] == full.cost and l[0] == full.max_latency_us)
    return out


res = []
for name in sys.argv[1:] or ["C1", "C2", "C3"]:
    if name.startswith("C4"):
        p = W.make_config("C4")
        for i, w in enumerate(W.c4_replans(int(name[3:] or 6))):
            for sla in (1_000_000, 2_000_000, 3_000_000):
                res.append(run(f"C4 window {i} SLA {sla}", p.replace(arrivals_us=w, sla_us=sla)))
    else:
        res.append(run(name, W.make_config(name)))
for r in res:
    print(json.dumps(r))
