"""Exhaustive SLA-constrained OPT of a full BASELINE config on one GPU (pruned, exact), with
the winner cross-checked on the CPU oracle.  Usage: python tools/time_to_optimal.py C2"""
import json, sys, time
sys.path.insert(0, '.')
import numpy as np
import torch
import workloads as W
from oracle import OracleProblem
from paper_conf_sc_luxl0y024_b200 import smiless as S

name = sys.argv[1] if len(sys.argv) > 1 else 'C2'
p = W.make_config(name)
pl = S.planner_for(p, stream=torch.cuda.current_stream().cuda_stream)
arr = torch.as_tensor(p.arrivals_us).cuda()
Wn = len(p.windows_us)
space = pl.space_size(Wn)
pl.plan(arr, p.sla_us, p.windows_us, end=1 << 20)          # JIT + warm-up
torch.cuda.synchronize()
t0 = time.perf_counter()
r = pl.plan(arr, p.sla_us, p.windows_us)
torch.cuda.synchronize()
dt = time.perf_counter() - t0
out = {"config": name, "space": space, "time_to_optimal_s": dt, "device_ms": r.total_device_ms,
       "evaluator_ms": r.eval_kernel_ms, "launches": r.launches, "n_decided": r.n_decided,
       "n_full_evals": r.n_full_evals, "feasible": r.feasible, "index": r.index, "cost": r.cost,
       "max_latency_us": r.max_latency_us, "config_vec": r.config.tolist(), "window_vec": r.window.tolist(),
       "decided_per_s": r.n_decided / dt}
if r.feasible:
    oc, ol, of = OracleProblem(p).evaluate([r.index])
    out["oracle_check"] = {"feasible": bool(of[0]), "cost_bits_equal": bool(oc[0] == r.cost),
                           "latency_equal": int(ol[0]) == r.max_latency_us}
print(json.dumps(out))
