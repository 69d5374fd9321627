"""Debug: per-candidate costs of the evaluator (cost_out) vs the oracle on a pickled case."""
import pickle, sys, numpy as np
sys.path.insert(0, '.')
from oracle import OracleProblem
from paper_conf_sc_luxl0y024_b200 import smiless as S
p = pickle.load(open(sys.argv[1], 'rb'))
o = OracleProblem(p)
n = o.space_size()
oc, ol, of = o.evaluate(np.arange(n, dtype=np.uint64))
pl = S.planner_for(p)
for flags in (1, 1 | 4):
    out = np.zeros(n)
    try:
        g = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, flags=flags, cost_out=out)
        print('flags', flags, 'winner', g.index, g.cost)
    except S.SmilessError as e:
        print('flags', flags, 'error', e)
    feas_g = ~np.isnan(out)
    print(' feasible mismatch', int((feas_g != of).sum()), 'of', n)
    both = feas_g & of
    bad = np.nonzero(both & (out != oc))[0]
    print(' cost mismatches', len(bad))
    Wn = len(p.windows_us)
    for i in bad[:12]:
        c, w = o.decode(int(i))
        print('  idx', i, 'cfg', c.tolist(), 'win', w.tolist(), 'gpu', out[i], 'oracle', oc[i], 'diff', out[i] - oc[i])
    fm = np.nonzero(feas_g != of)[0]
    for i in fm[:6]:
        c, w = o.decode(int(i))
        print('  feas idx', i, 'cfg', c.tolist(), 'win', w.tolist(), 'gpu feas', feas_g[i], 'oracle', of[i], ol[i], p.sla_us)
