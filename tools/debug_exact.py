import sys; sys.path.insert(0,'.')
import numpy as np, workloads as W
from oracle import OracleProblem
from paper_conf_sc_luxl0y024_b200 import smiless as S
rng = np.random.default_rng(2024)
nbad = 0
for t in range(120):
    n = int(rng.integers(1, 7))
    p = W.random_problem(rng, n, 4, int(rng.integers(1, 6)), int(rng.integers(1, 80)))
    if p.space_size() > 20000:
        continue
    flags = int(rng.choice([0, S.FLAG_NO_PRUNE, S.FLAG_FORCE_INT64]))
    sp = p.space_size()
    idx = np.arange(sp, dtype=np.uint64)
    pl = S.planner_for(p)
    gc, gl, gf = pl.evaluate(idx, p.arrivals_us, p.sla_us, p.windows_us)
    oc, ol, of = OracleProblem(p).evaluate(idx)
    bad = np.nonzero((gl != ol) | (gc.view(np.uint64) != oc.view(np.uint64)))[0]
    if len(bad):
        nbad += 1
        i = bad[0]
        print("case", t, "n", n, "J", len(p.arrivals_us), "preds", [p.preds(k) for k in range(n)], "nbad", len(bad), "of", sp,
              "idx", i, "gpu", gc[i], gl[i], "ora", oc[i], ol[i], flush=True)
        if nbad == 1:
            np.savez("gpurun_out/dbg_case.npz", arr=p.arrivals_us, bad=bad[:50])
    r = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, flags=flags) if not len(bad) else None
print("cases with mismatches:", nbad)
