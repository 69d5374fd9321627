"""Exhaustive SLA-constrained OPT of a BASELINE config on one GPU (pruned, exact), with the
winner cross-checked on the CPU oracle.
    python tools/time_to_optimal.py C2
    python tools/time_to_optimal.py C5 --fixed 7,0 7,0     # pin leading (config, window) digits
"""
import argparse, json, sys, time
sys.path.insert(0, '.')
import numpy as np
import torch
import workloads as W
from oracle import OracleProblem
from paper_conf_sc_luxl0y024_b200 import smiless as S

ap = argparse.ArgumentParser()
ap.add_argument("name", nargs="?", default="C2")
ap.add_argument("--fixed", nargs="*", default=[], help="config,window pairs pinning leading functions")
ap.add_argument("--sla", type=int, default=None)
a = ap.parse_args()
p = W.make_config(a.name)
if a.sla:
    p = p.replace(sla_us=a.sla)
Wn = len(p.windows_us)
fixed = [int(c) * Wn + int(w) for c, w in (f.split(",") for f in a.fixed)]
kw = dict(n_fixed=len(fixed), fixed_digits=fixed)
pl = S.planner_for(p, stream=torch.cuda.current_stream().cuda_stream)
arr = torch.as_tensor(p.arrivals_us).cuda()
space = pl.space_size(Wn, len(fixed))
pl.plan(arr, p.sla_us, p.windows_us, end=1 << 20, **kw)          # JIT + warm-up
torch.cuda.synchronize()
t0 = time.perf_counter()
r = pl.plan(arr, p.sla_us, p.windows_us, **kw)
torch.cuda.synchronize()
dt = time.perf_counter() - t0
out = {"config": a.name, "fixed": fixed, "sla_us": p.sla_us, "space": space, "time_to_optimal_s": dt,
       "device_ms": r.total_device_ms, "evaluator_ms": r.eval_kernel_ms, "launches": r.launches,
       "n_decided": r.n_decided, "n_full_evals": r.n_full_evals, "feasible": r.feasible, "index": r.index,
       "cost": r.cost, "max_latency_us": r.max_latency_us, "config_vec": r.config.tolist(),
       "window_vec": r.window.tolist(), "decided_per_s": r.n_decided / dt}
if r.feasible:
    oc, ol, of = OracleProblem(p, **kw).evaluate([r.index])
    out["oracle_check"] = {"feasible": bool(of[0]), "cost_bits_equal": bool(oc[0] == r.cost),
                           "latency_equal": int(ol[0]) == r.max_latency_us}
print(json.dumps(out))
