#!/bin/bash
# compute-sanitizer over small plans exercising every kernel path (run under gpurun):
# prep/evaluator/reduce/exact, B&B bound kernel + list mode, compaction passes, int64 path.
cat > /tmp/san.py <<'PY'
import os, sys, numpy as np
sys.path.insert(0, '.')
import workloads as W
from paper_conf_sc_luxl0y024_b200 import smiless as S
p = W.make_config("C1")
pl = S.planner_for(p)
pl.plan(p.arrivals_us, p.sla_us, p.windows_us)
pl.plan(p.arrivals_us, p.sla_us, p.windows_us, flags=S.FLAG_NO_PRUNE | S.FLAG_FORCE_INT64)
pl.evaluate(np.arange(64, dtype=np.uint64), p.arrivals_us, p.sla_us, p.windows_us)
rng = np.random.default_rng(3)
q = W.random_problem(rng, 5, 3, 3, 300, sla_us=40_000)
plq = S.planner_for(q)
os.environ["SMILESS_BB_DEPTH"] = "3"
plq.plan(q.arrivals_us, q.sla_us, q.windows_us)
os.environ["SMILESS_BB_DEPTH"] = "0"
os.environ["SMILESS_HORIZON"] = "64"
plq.plan(q.arrivals_us, q.sla_us, q.windows_us)
plq.plan_sla_sweep(q.arrivals_us, [20_000, 40_000], q.windows_us)
print("sanitize workload done")
PY
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python /tmp/san.py > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$? $(grep -c 'ERROR SUMMARY' gpurun_out/sanitize_$tool.log) $(grep 'ERROR SUMMARY' gpurun_out/sanitize_$tool.log | tail -1)"
done
