"""Estimate the exhaustive pruned time-to-optimal of the full C2 space (2^42) from a
random sample of its 2^28-candidate slices (functions 0, 1 pinned), on one GPU."""
import sys, time, json
import numpy as np
sys.path.insert(0, '.')
import torch
import workloads as W
from paper_conf_sc_luxl0y024_b200 import smiless as S

p = W.make_config('C2')
Wn = len(p.windows_us)
pl = S.planner_for(p, stream=torch.cuda.current_stream().cuda_stream)
arr = torch.as_tensor(p.arrivals_us).cuda()
rng = np.random.default_rng(int(sys.argv[1]) if len(sys.argv) > 1 else 0)
n = int(sys.argv[2]) if len(sys.argv) > 2 else 64
digits = [(int(a), int(b)) for a, b in rng.integers(0, 16 * Wn, size=(n, 2))]
pl.plan(arr, p.sla_us, p.windows_us, n_fixed=2, fixed_digits=list(digits[0]))   # warm-up + JIT
times, fulls, feas = [], [], 0
best = None
for d in digits:
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    r = pl.plan(arr, p.sla_us, p.windows_us, n_fixed=2, fixed_digits=list(d))
    times.append(time.perf_counter() - t0)
    fulls.append(r.n_full_evals / r.n_decided)
    feas += r.feasible
    if r.feasible and (best is None or r.cost < best[0]):
        best = (r.cost, d, r.index)
t = np.array(times)
print(json.dumps({"slices": n, "mean_ms": t.mean() * 1e3, "median_ms": float(np.median(t)) * 1e3,
                  "max_ms": t.max() * 1e3, "full_eval_frac_mean": float(np.mean(fulls)),
                  "feasible_slices": feas, "extrapolated_full_space_s": t.mean() * (16 * Wn) ** 2,
                  "best_in_sample": best}))
