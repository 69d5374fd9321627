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
# cost bound: two-level B&B with one shallow survivor per deep chunk and a cost cap
os.environ.pop("SMILESS_HORIZON")
os.environ.update(SMILESS_BB_DEPTH="3", SMILESS_BB_DEPTH_A="1", SMILESS_BB_FIRST="1")
r = plq.plan(q.arrivals_us, q.sla_us, q.windows_us)
if r.feasible:
    plq.plan(q.arrivals_us, q.sla_us, q.windows_us, cost_cap=r.cost)
for k in ("SMILESS_BB_DEPTH", "SMILESS_BB_DEPTH_A", "SMILESS_BB_FIRST"):
    os.environ.pop(k)
# prefix memoisation (throughput mode) and the wavefront exact evaluator on a 32-function DAG
os.environ["SMILESS_MEMO"] = "1"
plq.plan(q.arrivals_us, q.sla_us, q.windows_us, flags=S.FLAG_NO_PRUNE)
w = W.random_problem(rng, 32, 2, 2, 100, max_preds=8, sla_us=5 * 10**8)
S.planner_for(w).evaluate(rng.integers(0, w.space_size(), size=8, dtype=np.uint64), w.arrivals_us, w.sla_us,
                          w.windows_us)
# round 2: scale-out rings + prologue (plan, bound, memo upstream, virtual sink, exact),
# sharded B&B with split survivor lists, positive-time variants, the decomposition
for inst in ([2, 1, 3, 1, 2], [1, 2, 1, 1, 3]):       # last function 1 (memo, sink sharing) / 3 (virtual sink)
    plq.plan(q.arrivals_us, q.sla_us, q.windows_us, instances=inst)
    plq.plan(q.arrivals_us, q.sla_us, q.windows_us, instances=inst, flags=S.FLAG_NO_PRUNE)
    plq.evaluate(np.arange(32, dtype=np.uint64), q.arrivals_us, q.sla_us, q.windows_us, instances=inst)
os.environ.update(SMILESS_BB_DEPTH="3", SMILESS_BB_DEPTH_A="1", SMILESS_BB_LISTCAP="3")
for s_ in range(2):
    plq.plan(q.arrivals_us, q.sla_us, q.windows_us, shard=s_, n_shards=2, instances=[2, 1, 3, 1, 2])
for k in ("SMILESS_BB_DEPTH", "SMILESS_BB_DEPTH_A", "SMILESS_BB_LISTCAP"):
    os.environ.pop(k)
plq.decompose_plan(q.arrivals_us, q.sla_us, q.windows_us)
# round 2 (later): the fused producer/consumer memo kernel (mbarrier ring; plain and with a
# scaled-out upstream), the three-level B&B, smiless_plan_digits
rng2 = np.random.default_rng(11)
while True:
    f = W.random_problem(rng2, 4, 16, 2, 200, sla_us=60_000)
    if int(f.n_configs[-1]) >= 12:
        break
plf = S.planner_for(f)
os.environ["SMILESS_G"] = "1"
plf.plan(f.arrivals_us, f.sla_us, f.windows_us, flags=S.FLAG_NO_PRUNE)
plf.plan(f.arrivals_us, f.sla_us, f.windows_us, flags=S.FLAG_NO_PRUNE, instances=[2, 3, 1, 1])
os.environ["SMILESS_SPLITCOST"] = "0"
plf.plan(f.arrivals_us, f.sla_us, f.windows_us, flags=S.FLAG_NO_PRUNE, shard=1, n_shards=2)
os.environ.pop("SMILESS_SPLITCOST")
os.environ.pop("SMILESS_G")
os.environ.update(SMILESS_BB_DEPTH="4", SMILESS_BB_DEPTH_A="1", SMILESS_BB_DEPTH_M="2", SMILESS_BB_LISTCAP="5")
q6 = W.random_problem(rng2, 6, 3, 2, 200, sla_us=40_000)
pl6 = S.planner_for(q6)
pl6.plan(q6.arrivals_us, q6.sla_us, q6.windows_us)
pl6.plan(q6.arrivals_us, q6.sla_us, q6.windows_us, shard=0, n_shards=2)
for k in ("SMILESS_BB_DEPTH", "SMILESS_BB_DEPTH_A", "SMILESS_BB_DEPTH_M", "SMILESS_BB_LISTCAP"):
    os.environ.pop(k)
pl6.plan_digits(q6.arrivals_us, q6.sla_us, q6.windows_us, 0, int(q6.n_configs[0]) * 2, n_fixed=1, fixed_digits=[0])
print("sanitize workload done")
PY
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python /tmp/san.py > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$? $(grep -c 'ERROR SUMMARY' gpurun_out/sanitize_$tool.log) $(grep 'ERROR SUMMARY' gpurun_out/sanitize_$tool.log | tail -1)"
done
