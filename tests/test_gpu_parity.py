"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle (-m gpu).

Bar (BASELINE.json north star): chosen index / config / window bit-exact with
lowest-index tie-break, latencies exact in integer microseconds, cost within 1e-9
relative in fp64 -- the design reaches 0 ulp, so costs are compared bit for bit and
the 1e-9 bound is asserted as well.
"""
import numpy as np
import pytest

import workloads as W
from oracle import OracleProblem
from paper_conf_sc_luxl0y024_b200 import smiless as S

pytestmark = pytest.mark.gpu

COST_RTOL = 1e-9


def plan_both(p, **kw):
    pl = S.planner_for(p)
    g = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, **kw)
    nf = kw.get("n_fixed", 0)
    o = OracleProblem(p, n_fixed=nf, fixed_digits=kw.get("fixed_digits", ()))
    ref = o.plan(begin=kw.get("begin", 0), end=kw.get("end", 0))
    return pl, g, o, ref


def assert_same_plan(g, ref, o):
    if ref is None:
        assert g.status == S.INFEASIBLE and g.index is None and g.max_latency_us == -1
        assert (g.config == -1).all() and (g.window == -1).all()
        return
    assert g.status == S.OK
    assert g.index == ref[0]
    assert g.cost == ref[1] and abs(g.cost - ref[1]) <= COST_RTOL * abs(ref[1])
    assert g.max_latency_us == ref[2]
    c, w = o.decode(ref[0])
    assert g.config.tolist() == c.tolist() and g.window.tolist() == w.tolist()


def assert_same_eval(gc, gl, gf, oc, ol, of):
    assert (gf == of).all()
    assert (gl == ol).all()
    assert np.array_equal(gc.view(np.uint64), oc.view(np.uint64))


# ---------------------------------------------------------------------------------------
# C1 (configs[0]): every candidate, and the plan, in every mode
# ---------------------------------------------------------------------------------------

def test_c1_evaluate_every_candidate():
    p = W.make_config("C1")
    pl = S.planner_for(p)
    idx = np.arange(4096, dtype=np.uint64)
    gc, gl, gf = pl.evaluate(idx, p.arrivals_us, p.sla_us, p.windows_us)
    oc, ol, of = OracleProblem(p).evaluate(idx)
    assert_same_eval(gc, gl, gf, oc, ol, of)
    assert 0 < of.sum() < 4096


@pytest.mark.parametrize("flags", [0, S.FLAG_NO_PRUNE, S.FLAG_FORCE_INT64, S.FLAG_NO_PRUNE | S.FLAG_FORCE_INT64])
@pytest.mark.parametrize("sla", [300_000, 1_000_000, 1_500_000, 2_000_000, 3_000_000, 10_000_000])
def test_c1_plan(flags, sla):
    p = W.make_config("C1").replace(sla_us=sla)
    pl, g, o, ref = plan_both(p, flags=flags)
    assert_same_plan(g, ref, o)
    assert g.n_decided == 4096
    if flags & S.FLAG_NO_PRUNE:
        assert g.n_full_evals == 4096
    assert g.int64_path == bool(flags & S.FLAG_FORCE_INT64)


def test_c1_ranges_and_shards_compose():
    """[begin, end) sub-ranges (misaligned with W) and interleaved shards give the
    same winner as the full range after a lexicographic (cost, index) min."""
    p = W.make_config("C1")
    pl = S.planner_for(p)
    o = OracleProblem(p)
    for b, e in [(0, 4096), (1, 4095), (7, 9), (1000, 3001), (4095, 4096), (5, 5)]:
        g = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, begin=b, end=e)
        assert_same_plan(g, o.plan(begin=b, end=e), o)
        assert g.n_decided == e - b
    full = pl.plan(p.arrivals_us, p.sla_us, p.windows_us)
    for n in (2, 3, 8):
        parts = [pl.plan(p.arrivals_us, p.sla_us, p.windows_us, shard=s, n_shards=n) for s in range(n)]
        assert sum(r.n_decided for r in parts) == 4096
        best = min((r.cost, r.index) for r in parts if r.feasible)
        assert best == (full.cost, full.index)


def test_arrivals_on_device_tensor():
    import torch
    p = W.make_config("C1")
    pl = S.planner_for(p)
    host = pl.plan(p.arrivals_us, p.sla_us, p.windows_us)
    dev = torch.as_tensor(p.arrivals_us).cuda()
    d = pl.plan(dev, p.sla_us, p.windows_us)
    assert (d.index, d.cost, d.max_latency_us) == (host.index, host.cost, host.max_latency_us)
    bad = dev.clone()
    bad[5] = bad[4] - 1
    with pytest.raises(S.SmilessError) as e:
        pl.plan(bad, p.sla_us, p.windows_us)
    assert e.value.code == S.EINVAL


# ---------------------------------------------------------------------------------------
# Full-size configs: sampled exact evaluation at J = 10^4
# ---------------------------------------------------------------------------------------

@pytest.mark.parametrize("name,nf", [("C2", 0), ("C3", 0), ("C5", 2)])
def test_full_size_sampled_evaluate(name, nf):
    p = W.make_config(name)
    rng = np.random.default_rng(5)
    fixed = [int(rng.integers(0, p.n_configs[k] * len(p.windows_us))) for k in range(nf)]
    pl = S.planner_for(p)
    space = pl.space_size(len(p.windows_us), nf)
    idx = rng.integers(0, space, size=96, dtype=np.uint64)
    kw = dict(n_fixed=nf, fixed_digits=fixed)
    g = pl.evaluate(idx, p.arrivals_us, p.sla_us, p.windows_us, **kw)
    r = OracleProblem(p, n_fixed=nf, fixed_digits=fixed).evaluate(idx)
    assert_same_eval(*g, *r)


# ---------------------------------------------------------------------------------------
# Plan parity on oracle-sized sub-spaces of the real configs (pinned leading digits)
# ---------------------------------------------------------------------------------------

FAST = {"C2": 15, "C3": 11, "C4": 7, "C5": 7}   # GPU-100% config index per grid


@pytest.mark.parametrize("name,J", [("C2", 200), ("C3", 150), ("C4", 100), ("C5", 120)])
def test_plan_parity_on_subspaces(name, J):
    p = W.make_config(name, n_arrivals=J)
    Wn = len(p.windows_us)
    n = p.n_funcs
    rng = np.random.default_rng(11)
    checked_feasible = 0
    for trial in range(4):
        nf = n - 2
        fixed = []
        for k in range(nf):
            # trial 0: every pinned function on its fastest config, kept alive (feasible
            # prefix); later trials draw configs and windows at random
            c = FAST[name] if (trial == 0 or rng.random() < 0.7) else int(rng.integers(0, p.n_configs[k]))
            w = 0 if (trial == 0 or rng.random() < 0.6) else int(rng.integers(0, Wn))
            fixed.append(c * Wn + w)
        for sla in (p.sla_us, 4_000_000, 20_000_000):
            q = p.replace(sla_us=sla)
            for flags in (0, S.FLAG_NO_PRUNE):
                pl, g, o, ref = plan_both(q, n_fixed=nf, fixed_digits=fixed, flags=flags)
                assert_same_plan(g, ref, o)
                checked_feasible += ref is not None
    assert checked_feasible > 0


# ---------------------------------------------------------------------------------------
# Random DAGs: exhaustive plan parity, ragged configs, edge cases
# ---------------------------------------------------------------------------------------

def test_random_dags_exhaustive_plan_parity():
    rng = np.random.default_rng(2024)
    n_checked = 0
    for t in range(120):
        n = int(rng.integers(1, 7))
        p = W.random_problem(rng, n, 4, int(rng.integers(1, 6)), int(rng.integers(1, 80)))
        if p.space_size() > 20000:
            continue
        flags = int(rng.choice([0, S.FLAG_NO_PRUNE, S.FLAG_FORCE_INT64]))
        pl, g, o, ref = plan_both(p, flags=flags)
        assert_same_plan(g, ref, o)
        idx = rng.integers(0, p.space_size(), size=64, dtype=np.uint64)
        assert_same_eval(*pl.evaluate(idx, p.arrivals_us, p.sla_us, p.windows_us), *o.evaluate(idx))
        n_checked += 1
    assert n_checked > 60


@pytest.mark.parametrize("J", [1, 2, 3, 4, 5, 63, 64, 65, 127, 129, 257])
def test_horizon_edges_and_ragged_tail(J):
    """J = 1 (no steps), J - 1 below / at / above the chunk length and its multiples."""
    rng = np.random.default_rng(J)
    p = W.random_problem(rng, 4, 3, 3, J, sla_us=40_000)
    pl, g, o, ref = plan_both(p)
    assert_same_plan(g, ref, o)
    pl, g, o, ref = plan_both(p, flags=S.FLAG_NO_PRUNE)
    assert_same_plan(g, ref, o)


def test_ties_go_to_lowest_index():
    """Identical profiles for every config and zero prices: every candidate costs 0;
    the winner must be the lowest feasible index."""
    rng = np.random.default_rng(3)
    p = W.random_problem(rng, 3, 3, 3, 20, sla_us=10**8)
    p = p.replace(price_per_us=np.zeros_like(p.price_per_us))
    pl, g, o, ref = plan_both(p)
    assert ref[0] == 0 and g.index == 0 and g.cost == 0.0
    p2 = p.replace(price_per_us=np.ones_like(p.price_per_us) / 1024)
    pl, g, o, ref = plan_both(p2)
    assert_same_plan(g, ref, o)


def test_single_function_and_all_sources():
    rng = np.random.default_rng(4)
    for preds in ([[]], [[], []], [[], [], [], []]):
        base = W.random_problem(rng, len(preds), 4, 4, 40)
        ptr, idx = W.csr_from_preds(preds)
        p = base.replace(pred_ptr=ptr, pred_idx=idx)
        pl, g, o, ref = plan_both(p)
        assert_same_plan(g, ref, o)


def test_windows_without_keepalive_and_single_window():
    rng = np.random.default_rng(6)
    p = W.random_problem(rng, 3, 3, 4, 50)
    p = p.replace(windows_us=np.array([700, 2500, 9000], np.int32))
    pl, g, o, ref = plan_both(p)
    assert_same_plan(g, ref, o)
    p = p.replace(windows_us=np.array([0], np.int32))
    pl, g, o, ref = plan_both(p)
    assert_same_plan(g, ref, o)


def test_fully_pinned_and_empty_ranges():
    p = W.make_config("C1", n_arrivals=50)
    pl = S.planner_for(p)
    o = OracleProblem(p, n_fixed=3, fixed_digits=[15, 3, 0])
    g = pl.plan(p.arrivals_us, 10**8 - 1, p.windows_us, n_fixed=3, fixed_digits=[15, 3, 0])
    assert g.index == 0
    c, l, f = o.evaluate([0])
    assert g.cost == c[0] and g.max_latency_us == l[0]
    g = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, begin=100, end=100)
    assert g.status == S.INFEASIBLE and g.n_decided == 0


def test_large_gaps_exercise_clamp_and_int64_path_agree():
    """Gaps far above d_cap (clamped on the int32 path) and the int64 path give the
    oracle's answer; the natural int64 path (int32 range rule fails) as well."""
    rng = np.random.default_rng(8)
    for t in range(10):
        p = W.random_problem(rng, 4, 3, 3, 60)
        gaps = np.diff(p.arrivals_us, prepend=0)
        gaps[rng.random(len(gaps)) < 0.3] = int(rng.integers(10**9, 10**12))
        p = p.replace(arrivals_us=np.cumsum(gaps).astype(np.int64))
        for flags in (0, S.FLAG_FORCE_INT64):
            pl, g, o, ref = plan_both(p, flags=flags)
            assert_same_plan(g, ref, o)
    p = W.random_problem(rng, 3, 2, 3, 30, time_scale=10**7 // 8)
    p = p.replace(windows_us=np.array([0, 1 << 28, (1 << 29) - 1], np.int32),
                  init_us=np.minimum(p.init_us.astype(np.int64) * 8, (1 << 29) - 1).astype(np.int32),
                  sla_us=(1 << 29) - 1)
    pl, g, o, ref = plan_both(p)
    assert g.int64_path
    assert_same_plan(g, ref, o)


# ---------------------------------------------------------------------------------------
# The bench launch configuration at full size (C2, J = 10^4, 2^28-candidate slice)
# ---------------------------------------------------------------------------------------

def test_bench_configuration_split_cost_same_result(monkeypatch):
    """The bench slice at full size with the split-cost throughput path (every unit walked
    without the sum-of-u accumulators, units with a feasible candidate re-walked for their
    costs) returns the single-pass winner bit for bit and walks every candidate."""
    import bench
    p, kw = bench.workload("C2")
    pl = S.planner_for(p)
    monkeypatch.setenv("SMILESS_SPLITCOST", "0")
    one = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, flags=S.FLAG_NO_PRUNE, **kw)
    monkeypatch.setenv("SMILESS_SPLITCOST", "1")
    two = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, flags=S.FLAG_NO_PRUNE, **kw)
    assert (two.index, two.cost, two.max_latency_us) == (one.index, one.cost, one.max_latency_us)
    assert two.n_full_evals == two.n_decided == one.n_decided
    assert two.launches > one.launches                  # the cost pass ran


def test_bench_configuration_full_size_properties():
    """bench.py's step: C2 at J = 10^4, functions 0/1 pinned, 2^28 candidates, no pruning.
    The oracle cannot walk 2^28 x 10^4 x 6 steps, so we check (a) the winner on the
    oracle (cost bits, latency, feasibility), (b) no sampled feasible candidate beats it
    (lexicographic), (c) the pruned run returns the same winner, (d) the exact plan of
    the winner's own 2^14-candidate neighbourhood on the oracle contains it as OPT."""
    import bench
    p, kw = bench.workload("C2")
    pl = S.planner_for(p)
    full = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, flags=S.FLAG_NO_PRUNE, **kw)
    assert full.n_full_evals == full.n_decided == pl.space_size(len(p.windows_us), kw["n_fixed"])
    o = OracleProblem(p, **kw)
    pruned = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, **kw)
    assert (pruned.index, pruned.cost) == (full.index, full.cost)
    if full.feasible:
        c, l, f = o.evaluate([full.index])
        assert f[0] and c[0] == full.cost and l[0] == full.max_latency_us
        lo = full.index - full.index % (1 << 14)
        ref = o.plan(begin=lo, end=lo + (1 << 14))
        assert ref[0] == full.index and ref[1] == full.cost
    rng = np.random.default_rng(9)
    idx = rng.integers(0, full.n_decided, size=256, dtype=np.uint64)
    c, l, f = o.evaluate(idx)
    for i in range(len(idx)):
        if f[i]:
            assert full.feasible and (full.cost, full.index) <= (c[i], int(idx[i]))


# ---------------------------------------------------------------------------------------
# Per-candidate parity of the fast evaluator itself (cost_out), not only of its argmin
# ---------------------------------------------------------------------------------------

def assert_dump_matches(out, oc, of):
    feas = ~np.isnan(out)
    assert (feas == of).all(), np.nonzero(feas != of)[0][:10]
    bad = np.nonzero(feas & (out.view(np.uint64) != oc.view(np.uint64)))[0]
    assert len(bad) == 0, (bad[:10], out[bad[:10]], oc[bad[:10]])


def test_random_dags_per_candidate_costs():
    """Every candidate's cost as the int32/int64 evaluator computes it (sink sharing,
    rebasing, clamped gaps, negated time, busy mask) equals the oracle's, bit for bit;
    infeasible candidates are exactly the oracle's infeasible ones.  Joins of up to 3
    predecessors (the VIMNMX3 erratum pattern) are frequent here."""
    rng = np.random.default_rng(77)
    n_checked = 0
    for t in range(160):
        n = int(rng.integers(1, 7))
        p = W.random_problem(rng, n, 4, int(rng.integers(1, 6)), int(rng.integers(1, 140)))
        space = p.space_size()
        if space > 30000:
            continue
        flags = int(rng.choice([0, S.FLAG_NO_PRUNE, S.FLAG_FORCE_INT64]))
        pl = S.planner_for(p)
        out = np.empty(space)
        pl.plan(p.arrivals_us, p.sla_us, p.windows_us, flags=flags, cost_out=out)
        oc, ol, of = OracleProblem(p).evaluate(np.arange(space, dtype=np.uint64))
        assert_dump_matches(out, oc, of)
        n_checked += 1
    assert n_checked > 80


@pytest.mark.parametrize("name", ["C1", "C4"])
def test_config_per_candidate_costs(name):
    p = W.make_config(name)
    if name == "C4":
        p = p.replace(sla_us=3_000_000)
    pl = S.planner_for(p)
    space = min(pl.space_size(len(p.windows_us)), 1 << 14)
    for flags in (0, S.FLAG_NO_PRUNE):
        out = np.empty(space)
        pl.plan(p.arrivals_us, p.sla_us, p.windows_us, end=space, flags=flags, cost_out=out)
        oc, ol, of = OracleProblem(p).evaluate(np.arange(space, dtype=np.uint64))
        assert_dump_matches(out, oc, of)


def test_bench_slice_per_candidate_costs_full_J():
    """bench.py's C2 slice at J = 10^4: 2^12 consecutive candidates around the winner."""
    import bench
    p, kw = bench.workload("C2")
    pl = S.planner_for(p)
    full = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, **kw)
    lo = (full.index if full.feasible else 0) // 4096 * 4096
    out = np.empty(4096)
    pl.plan(p.arrivals_us, p.sla_us, p.windows_us, begin=lo, end=lo + 4096, flags=S.FLAG_NO_PRUNE,
            cost_out=out, **kw)
    oc, ol, of = OracleProblem(p, **kw).evaluate(np.arange(lo, lo + 4096, dtype=np.uint64))
    assert_dump_matches(out, oc, of)
    assert of.any() == full.feasible


@pytest.mark.parametrize("horizon", ["64", "128", "0"])
def test_stream_compaction_passes_are_exact(horizon, monkeypatch):
    """Prune mode runs pass 1 (all units, `horizon` steps, survivors compacted) and pass 2
    (survivors, all steps).  Every candidate's cost / feasibility and the winner must not
    depend on the horizon (0 = single pass)."""
    monkeypatch.setenv("SMILESS_HORIZON", horizon)
    rng = np.random.default_rng(31)
    n_checked = 0
    for t in range(40):
        n = int(rng.integers(2, 6))
        p = W.random_problem(rng, n, 3, int(rng.integers(2, 5)), int(rng.integers(130, 400)),
                             sla_us=int(rng.integers(20_000, 60_000)))
        space = p.space_size()
        if space > 20000:
            continue
        pl = S.planner_for(p)
        out = np.empty(space)
        g = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, cost_out=out)
        o = OracleProblem(p)
        oc, ol, of = o.evaluate(np.arange(space, dtype=np.uint64))
        assert_dump_matches(out, oc, of)
        assert_same_plan(g, o.plan(), o)
        assert g.n_decided == space
        n_checked += 1
    assert n_checked > 15


def test_branch_and_bound_prefix_pruning_is_exact(monkeypatch):
    """The B&B pre-pass (prefixes of D functions, the rest relaxed to keep-alive at their
    fastest config) only discards infeasible subtrees: every depth gives the oracle's
    per-candidate feasibility / cost, the same winner, and decides every candidate of the
    range exactly once (also for misaligned ranges and interleaved shards)."""
    rng = np.random.default_rng(47)
    n_checked = 0
    for t in range(40):
        if n_checked == 14:
            break
        n = int(rng.integers(3, 7))
        p = W.random_problem(rng, n, 3, int(rng.integers(2, 5)), int(rng.integers(20, 200)),
                             sla_us=int(rng.integers(15_000, 60_000)))
        space = p.space_size()
        if space > 30000:
            continue
        o = OracleProblem(p)
        oc, ol, of = o.evaluate(np.arange(space, dtype=np.uint64))
        ref = o.plan()
        for d in range(1, n):
            monkeypatch.setenv("SMILESS_BB_DEPTH", str(d))
            pl = S.planner_for(p)
            out = np.empty(space)
            g = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, cost_out=out)
            assert_dump_matches(out, oc, of)
            assert_same_plan(g, ref, o)
            assert g.n_decided == space
            b, e = int(rng.integers(0, space // 2)), int(rng.integers(space // 2, space + 1))
            g = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, begin=b, end=e)
            assert_same_plan(g, o.plan(begin=b, end=e), o)
            assert g.n_decided == e - b
            parts = [pl.plan(p.arrivals_us, p.sla_us, p.windows_us, shard=s_, n_shards=3) for s_ in range(3)]
            assert sum(r.n_decided for r in parts) == space
            feas = [(r.cost, r.index) for r in parts if r.feasible]
            assert (min(feas) if feas else None) == (None if ref is None else (ref[1], ref[0]))
        n_checked += 1
    assert n_checked > 10


# ---------------------------------------------------------------------------------------
# C4: SLA sweep in one pass (one argmin key per SLA)
# ---------------------------------------------------------------------------------------

def test_sla_sweep_matches_per_sla_oracle_plans():
    slas = W.C4_SLAS_US
    p = W.make_config("C4")
    Wn = len(p.windows_us)
    pl = S.planner_for(p)
    rng = np.random.default_rng(4)
    for trial in range(3):
        nf = 3
        fixed = [(7 if trial == 0 else int(rng.integers(0, 8))) * Wn + int(rng.integers(0, Wn)) for _ in range(nf)]
        rs = pl.plan_sla_sweep(p.arrivals_us, slas, p.windows_us, n_fixed=nf, fixed_digits=fixed)
        prev = None
        for sla, g in zip(slas, rs):
            o = OracleProblem(p.replace(sla_us=sla), n_fixed=nf, fixed_digits=fixed)
            assert_same_plan(g, o.plan(), o)
            single = pl.plan(p.arrivals_us, sla, p.windows_us, n_fixed=nf, fixed_digits=fixed)
            assert (single.index, single.cost) == (g.index, g.cost)
            if prev is not None and prev.feasible:       # OPT non-increasing in the SLA
                assert g.feasible and g.cost <= prev.cost
            prev = g


def test_sla_sweep_random_dags():
    rng = np.random.default_rng(5)
    for t in range(25):
        n = int(rng.integers(1, 6))
        p = W.random_problem(rng, n, 3, int(rng.integers(1, 5)), int(rng.integers(1, 90)))
        if p.space_size() > 20000:
            continue
        slas = sorted(set(int(v) for v in rng.integers(1_000, 40_000, size=int(rng.integers(2, 8)))))
        pl = S.planner_for(p)
        rs = pl.plan_sla_sweep(p.arrivals_us, slas, p.windows_us)
        for sla, g in zip(slas, rs):
            o = OracleProblem(p.replace(sla_us=sla))
            assert_same_plan(g, o.plan(), o)


# ---------------------------------------------------------------------------------------
# NEXT-1: config-only search under the paper's derived windows (per-row windows)
# ---------------------------------------------------------------------------------------

def test_derived_window_plans_match_oracle():
    rng = np.random.default_rng(61)
    n_checked = 0
    for t in range(30):
        n = int(rng.integers(1, 7))
        p = W.random_problem(rng, n, 6, 1, int(rng.integers(1, 150)))
        p = p.replace(windows_us=np.array([0], np.int32))
        if p.space_size() > 30000:
            continue
        pl = S.planner_for(p)
        it = int(np.diff(p.arrivals_us).mean()) if len(p.arrivals_us) > 1 else 0
        rw = pl.derive_windows(it)
        o = OracleProblem(p, row_windows=rw)
        space = p.space_size()
        for flags in (0, S.FLAG_NO_PRUNE, S.FLAG_FORCE_INT64):
            out = np.empty(space)
            g = pl.plan(p.arrivals_us, p.sla_us, [0], row_windows=rw, flags=flags, cost_out=out)
            assert_same_plan(g, o.plan(), o)
            oc, ol, of = o.evaluate(np.arange(space, dtype=np.uint64))
            assert_dump_matches(out, oc, of)
        idx = rng.integers(0, space, size=32, dtype=np.uint64)
        assert_same_eval(*pl.evaluate(idx, p.arrivals_us, p.sla_us, [0], row_windows=rw), *o.evaluate(idx))
        n_checked += 1
    assert n_checked > 15


def test_derived_window_c2_full_plan_with_bnb():
    """C2 (J = 10^4) under the paper's derived windows: 16^6 configurations, B&B pre-pass."""
    p = W.make_config("C2")
    q = p.replace(windows_us=np.array([0], np.int32))
    pl = S.planner_for(q)
    rw = pl.derive_windows(int(np.diff(p.arrivals_us).mean()))
    g = pl.plan(q.arrivals_us, q.sla_us, [0], row_windows=rw)
    o = OracleProblem(q, row_windows=rw)
    assert g.n_decided == 16 ** 6
    if g.feasible:
        c, l, f = o.evaluate([g.index])
        assert f[0] and c[0] == g.cost and l[0] == g.max_latency_us
        lo = g.index - g.index % 4096
        ref = o.plan(begin=lo, end=lo + 4096)
        assert ref[0] == g.index and ref[1] == g.cost


# ---------------------------------------------------------------------------------------
# NEXT-2: SMIless's Top-1 path search, GPU-evaluated nodes vs the oracle's walk
# ---------------------------------------------------------------------------------------

def test_top1_search_matches_oracle_walk():
    from oracle.top1 import top1_search
    rng = np.random.default_rng(71)
    for t in range(30):
        n = int(rng.integers(1, 7))
        p = W.random_problem(rng, n, 6, 1, int(rng.integers(2, 120)), sla_us=int(rng.integers(5_000, 40_000)))
        p = p.replace(windows_us=np.array([0], np.int32))
        it = int(np.diff(p.arrivals_us).mean()) if len(p.arrivals_us) > 1 else 0
        pl = S.planner_for(p)
        rw = pl.derive_windows(it)
        g, nodes = pl.top1_search(p.arrivals_us, p.sla_us, it, rw)
        cfg, cost, lat, ok, onodes = top1_search(p, it, rw, OracleProblem)
        assert nodes == onodes
        assert g.feasible == ok
        if ok:
            assert g.config.tolist() == cfg and g.cost == cost and g.max_latency_us == lat


def test_top1_never_beats_exhaustive_opt():
    """The heuristic's plan is a candidate of the derived-window space, so the exhaustive
    OPT of that space (and of the full window grid) costs no more."""
    rng = np.random.default_rng(72)
    for t in range(20):
        n = int(rng.integers(2, 6))
        p = W.random_problem(rng, n, 5, 1, int(rng.integers(10, 100)), sla_us=int(rng.integers(8_000, 40_000)))
        p = p.replace(windows_us=np.array([0], np.int32))
        it = int(np.diff(p.arrivals_us).mean())
        pl = S.planner_for(p)
        rw = pl.derive_windows(it)
        h, _ = pl.top1_search(p.arrivals_us, p.sla_us, it, rw)
        opt = pl.plan(p.arrivals_us, p.sla_us, [0], row_windows=rw)
        if h.feasible:
            assert opt.feasible and opt.cost <= h.cost


def test_two_level_branch_and_bound_is_exact(monkeypatch):
    """Shallow level (depth DA over every prefix) + deep level (depth D over the shallow
    survivors' children, list mode) + evaluator: same per-candidate results and winners."""
    rng = np.random.default_rng(53)
    n_checked = 0
    for t in range(30):
        if n_checked == 10:   # each (D, DA) pair is a separate NVRTC module; bound the compile time
            break
        n = int(rng.integers(4, 7))
        p = W.random_problem(rng, n, 3, int(rng.integers(2, 4)), int(rng.integers(20, 160)),
                             sla_us=int(rng.integers(15_000, 60_000)))
        space = p.space_size()
        if space > 30000:
            continue
        o = OracleProblem(p)
        oc, ol, of = o.evaluate(np.arange(space, dtype=np.uint64))
        ref = o.plan()
        for d in range(2, n):
            for da in range(1, d):
                monkeypatch.setenv("SMILESS_BB_DEPTH", str(d))
                monkeypatch.setenv("SMILESS_BB_DEPTH_A", str(da))
                pl = S.planner_for(p)
                out = np.empty(space)
                g = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, cost_out=out)
                assert_dump_matches(out, oc, of)
                assert_same_plan(g, ref, o)
                assert g.n_decided == space
                parts = [pl.plan(p.arrivals_us, p.sla_us, p.windows_us, shard=s_, n_shards=2) for s_ in range(2)]
                assert sum(r.n_decided for r in parts) == space
                # one shallow survivor per deep chunk: every later chunk's static prefix bound
                # prunes against the incumbent the earlier chunks set (cost bound on)
                monkeypatch.setenv("SMILESS_BB_FIRST", "1")
                g = pl.plan(p.arrivals_us, p.sla_us, p.windows_us)
                assert_same_plan(g, ref, o)
                assert g.n_decided == space
                if ref is not None:
                    g = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, cost_cap=ref[1])
                    assert_same_plan(g, ref, o)
                monkeypatch.delenv("SMILESS_BB_FIRST")
        n_checked += 1
    assert n_checked > 8


def test_branch_and_bound_with_pinned_digits(monkeypatch):
    """B&B levels count from the pinned prefix (n_fixed > 0): per-candidate parity with the
    oracle on the suffix space, for single and two-level schemes."""
    rng = np.random.default_rng(59)
    n_checked = 0
    for t in range(30):
        if n_checked == 10:
            break
        n = int(rng.integers(4, 7))
        p = W.random_problem(rng, n, 3, int(rng.integers(2, 4)), int(rng.integers(20, 150)),
                             sla_us=int(rng.integers(15_000, 60_000)))
        Wn = len(p.windows_us)
        nf = int(rng.integers(1, 3))
        fixed = [int(rng.integers(0, p.n_configs[k] * Wn)) for k in range(nf)]
        o = OracleProblem(p, n_fixed=nf, fixed_digits=fixed)
        space = o.space_size()
        if space > 30000 or space < 64:
            continue
        oc, ol, of = o.evaluate(np.arange(space, dtype=np.uint64))
        ref = o.plan()
        for d, da, dm in [(d, da, dm) for d in range(nf + 1, n) for da in [0] + list(range(nf + 1, d))
                          for dm in [0] + ([da + 1] if 0 < da and da + 1 < d else [])]:
                monkeypatch.setenv("SMILESS_BB_DEPTH", str(d))
                monkeypatch.setenv("SMILESS_BB_DEPTH_A", str(da))
                monkeypatch.setenv("SMILESS_BB_DEPTH_M", str(dm))          # three levels when dm > 0 (C5)
                pl = S.planner_for(p)
                out = np.empty(space)
                g = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, n_fixed=nf, fixed_digits=fixed, cost_out=out)
                assert_dump_matches(out, oc, of)
                assert_same_plan(g, ref, o)
                assert g.n_decided == space
        n_checked += 1
    assert n_checked > 8


# ---------------------------------------------------------------------------------------
# NEXT-3: DAG decomposition into sequential paths + combine
# ---------------------------------------------------------------------------------------

def test_decompose_search_matches_oracle_steps():
    from oracle.decompose import decompose_search
    rng = np.random.default_rng(91)
    for t in range(30):
        n = int(rng.integers(1, 8))
        p = W.random_problem(rng, n, 6, 1, int(rng.integers(2, 80)), sla_us=int(rng.integers(5_000, 40_000)))
        p = p.replace(windows_us=np.array([0], np.int32))
        it = int(np.diff(p.arrivals_us).mean()) if len(p.arrivals_us) > 1 else 0
        pl = S.planner_for(p)
        rw = pl.derive_windows(it)
        g, n_paths = pl.decompose_search(p.arrivals_us, p.sla_us, it, rw)
        cfg, cost, lat, ok, onp = decompose_search(p, it, rw, OracleProblem)
        assert n_paths == onp and g.feasible == ok
        if ok:
            assert g.config.tolist() == cfg and g.cost == cost and g.max_latency_us == lat


@pytest.mark.parametrize("memo,fused", [("0", "1"), ("1", "0"), ("1", "1")])
def test_throughput_mode_with_and_without_prefix_memoisation(memo, fused, monkeypatch):
    """Throughput mode runs the upstream once per prefix (memo = 1: the fused producer/consumer
    kernel where a tile fits, else upstream + variants kernels; fused = 0: always the two
    kernels) or per unit (memo = 0): per-candidate parity with the oracle either way."""
    monkeypatch.setenv("SMILESS_MEMO", memo)
    monkeypatch.setenv("SMILESS_FUSED", fused)
    rng = np.random.default_rng(97)
    n_checked = 0
    for t in range(40):
        n = int(rng.integers(1, 7))
        p = W.random_problem(rng, n, 4, int(rng.integers(1, 6)), int(rng.integers(1, 200)))
        space = p.space_size()
        if space > 30000:
            continue
        flags = S.FLAG_NO_PRUNE | (S.FLAG_FORCE_INT64 if rng.random() < 0.3 else 0)
        pl = S.planner_for(p)
        b = int(rng.integers(0, space // 3 + 1))
        out = np.empty(space - b)
        g = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, flags=flags, begin=b, cost_out=out)
        o = OracleProblem(p)
        oc, ol, of = o.evaluate(np.arange(b, space, dtype=np.uint64))
        assert_dump_matches(out, oc, of)
        assert_same_plan(g, o.plan(begin=b), o)
        assert g.n_full_evals == g.n_decided == space - b
        n_checked += 1
    assert n_checked > 20


@pytest.mark.parametrize("g,split,fmask", [("1", "1", "0"), ("1", "0", "0x54"), ("2", "1", "0xaa"), ("4", "0", "0"),
                                          ("2", "1", "0x54"), ("2", "0", "0xff"), ("1", "1", "0xffffffff")])
def test_memo_variants_shapes_are_exact(g, split, fmask, monkeypatch):
    """The variants kernel's tuning knobs (configs per lane G, split cost: every unit walked
    without the sum-of-u accumulators and the units with a feasible candidate re-walked for
    their costs, positive-time form per window variant) change only the instruction mix:
    per-candidate parity with the oracle for each."""
    monkeypatch.setenv("SMILESS_FMASK", fmask)
    monkeypatch.setenv("SMILESS_MEMO", "1")
    monkeypatch.setenv("SMILESS_FUSED", "0")
    monkeypatch.setenv("SMILESS_SPLITCOST", split)
    monkeypatch.setenv("SMILESS_G", g)
    rng = np.random.default_rng(131 + int(g) * 7 + int(fmask, 0) % 97)
    n_checked = 0
    for t in range(30):
        n = int(rng.integers(2, 6))
        p = W.random_problem(rng, n, 4, int(rng.integers(2, 5)), int(rng.integers(2, 300)))
        space = p.space_size()
        if space > 30000:
            continue
        pl = S.planner_for(p)
        out = np.empty(space)
        g_ = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, flags=S.FLAG_NO_PRUNE, cost_out=out)
        o = OracleProblem(p)
        oc, ol, of = o.evaluate(np.arange(0, space, dtype=np.uint64))
        assert_dump_matches(out, oc, of)
        assert_same_plan(g_, o.plan(), o)
        n_checked += 1
    assert n_checked > 10


@pytest.mark.parametrize("g,split", [("1", "1"), ("1", "0"), ("2", "1"), ("2", "0")])
def test_fused_memo_kernel_is_exact(g, split, monkeypatch):
    """The fused memoisation kernel (producer warps -> shared-memory ring of x -> consumer
    warps; split cost re-walked by the plan kernel in list mode) on random DAGs whose last
    function has enough config groups for a tile: per-candidate parity with the oracle over
    ragged ranges (partial tiles), several ring slots and a one-step tail, and every candidate
    counted once."""
    monkeypatch.setenv("SMILESS_MEMO", "1")
    monkeypatch.setenv("SMILESS_FUSED", "1")
    monkeypatch.setenv("SMILESS_SPLITCOST", split)
    monkeypatch.setenv("SMILESS_G", g)
    rng = np.random.default_rng(211 + 10 * int(g) + int(split))
    n_checked = 0
    for t in range(120):
        n = int(rng.integers(2, 5))
        p = W.random_problem(rng, n, 16, int(rng.integers(1, 4)), int(rng.choice([2, 5, 64, 65, 130, 257, 400])))
        space = p.space_size()
        if space > 40000 or int(p.n_configs[-1]) % int(g):
            continue
        pl = S.planner_for(p)
        flags = S.FLAG_NO_PRUNE
        if "#define SM_FUSED 1" not in pl.kernel_source(p.arrivals_us, p.sla_us, p.windows_us, flags=flags):
            continue                                   # too few config groups for a tile
        b = int(rng.integers(0, space // 4 + 1))
        out = np.empty(space - b)
        r = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, flags=flags, begin=b, cost_out=out)
        o = OracleProblem(p)
        oc, ol, of = o.evaluate(np.arange(b, space, dtype=np.uint64))
        assert_dump_matches(out, oc, of)
        assert_same_plan(r, o.plan(begin=b), o)
        assert r.n_full_evals == r.n_decided == space - b
        assert r.eval_path == S.PATH_MEMO_FUSED
        n_checked += 1
        if n_checked >= 12:
            break
    assert n_checked >= 6


def test_fused_memo_kernel_with_scaled_out_upstream(monkeypatch):
    """The fused kernel's producers with instance rings and the scale-out prologue (upstream
    functions with 2-4 round-robin instances, the last one with 1, as C3): per-candidate
    parity with the oracle."""
    monkeypatch.setenv("SMILESS_FUSED", "1")
    rng = np.random.default_rng(577)
    n_checked = 0
    for t in range(200):
        n = int(rng.integers(2, 5))
        p = W.random_problem(rng, n, 16, int(rng.integers(1, 4)), int(rng.choice([3, 9, 17, 70, 131])))
        space = p.space_size()
        if space > 40000:
            continue
        inst = [int(rng.integers(1, 5)) for _ in range(n - 1)] + [1]
        if max(inst) == 1:
            continue
        pl = S.planner_for(p)
        kw = dict(flags=S.FLAG_NO_PRUNE, instances=inst)
        if "#define SM_FUSED 1" not in pl.kernel_source(p.arrivals_us, p.sla_us, p.windows_us, **kw):
            continue
        o = OracleProblem(p, instances=inst)
        oc, ol, of = o.evaluate(np.arange(space, dtype=np.uint64))
        out = np.empty(space)
        r = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, cost_out=out, **kw)
        assert r.eval_path == S.PATH_MEMO_FUSED
        assert_dump_matches(out, oc, of)
        assert_same_plan(r, o.plan(), o)
        n_checked += 1
        if n_checked >= 10:
            break
    assert n_checked >= 5


def test_fused_memo_kernel_shards_and_matches_two_kernel_path(monkeypatch):
    """Fused vs two-kernel memoisation on the bench slice of C2 at J = 10^4 (2^28 candidates
    is too long here: a 2^22-candidate range around the winner), bit-identical winner; and the
    fused kernel's tiles interleaved over 3 shards decide the range exactly once."""
    import bench
    p, kw = bench.workload("C2")
    pl = S.planner_for(p)
    full = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, flags=S.FLAG_NO_PRUNE, **kw)
    lo = full.index - full.index % (1 << 22) if full.feasible else 0
    rng_kw = dict(kw, begin=lo + 77, end=lo + (1 << 22) - 5, flags=S.FLAG_NO_PRUNE)
    monkeypatch.setenv("SMILESS_FUSED", "0")
    two = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, **rng_kw)
    monkeypatch.setenv("SMILESS_FUSED", "1")
    assert "#define SM_FUSED 1" in pl.kernel_source(p.arrivals_us, p.sla_us, p.windows_us, **rng_kw)
    one = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, **rng_kw)
    assert (one.index, one.cost, one.max_latency_us) == (two.index, two.cost, two.max_latency_us)
    assert one.n_decided == two.n_decided == one.n_full_evals == (1 << 22) - 82
    assert (one.eval_path, two.eval_path) == (S.PATH_MEMO_FUSED, S.PATH_MEMO)
    parts = [pl.plan(p.arrivals_us, p.sla_us, p.windows_us, shard=s, n_shards=3, **rng_kw) for s in range(3)]
    assert sum(r.n_decided for r in parts) == one.n_decided
    assert all(r.n_decided > 0 for r in parts)
    best = min((r for r in parts if r.feasible), key=lambda r: (r.cost, r.index))
    assert (best.index, best.cost) == (one.index, one.cost)


# ---------------------------------------------------------------------------------------
# Cost-bound pruning against an incumbent, and the caller's cost cap (DESIGN.md section 5
# item 11): only candidates costing strictly more than a real feasible candidate (or the
# cap) are dropped, so the argmin and its lowest-index tie-break are unchanged
# ---------------------------------------------------------------------------------------

def _lex_min(oc, of, cap=np.inf):
    elig = np.nonzero(of & (oc <= cap))[0]
    if len(elig) == 0:
        return None
    best = elig[np.lexsort((elig, oc[elig]))[0]]
    return int(best), float(oc[best])


def test_cost_bound_and_cost_cap_are_exact(monkeypatch):
    rng = np.random.default_rng(61)
    checked = fewer = 0
    for t in range(120):
        if checked == 12:
            break
        n = int(rng.integers(2, 6))
        p = W.random_problem(rng, n, 4, int(rng.integers(2, 5)), int(rng.integers(150, 400)),
                             sla_us=int(rng.integers(15_000, 60_000)))
        space = p.space_size()
        if space > 40000:
            continue
        o = OracleProblem(p)
        oc, ol, of = o.evaluate(np.arange(space, dtype=np.uint64))
        ref = o.plan()
        assert (None if ref is None else (ref[0], ref[1])) == _lex_min(oc, of)
        pl = S.planner_for(p)
        args = (p.arrivals_us, p.sla_us, p.windows_us)
        assert_same_plan(pl.plan(*args), ref, o)                     # running incumbent
        monkeypatch.setenv("SMILESS_COST_PRUNE", "0")
        off = pl.plan(*args)
        monkeypatch.delenv("SMILESS_COST_PRUNE")
        assert_same_plan(off, ref, o)
        if ref is None:
            continue
        # the tightest valid cap is OPT itself: candidates tying it must survive; with the B&B
        # pre-pass at every depth the static prefix bound prunes against the cap as well
        for d in [None] + list(range(1, n)):
            if d is None:
                monkeypatch.delenv("SMILESS_BB_DEPTH", raising=False)
            else:
                monkeypatch.setenv("SMILESS_BB_DEPTH", str(d))
            for cap in (ref[1], float(np.nextafter(ref[1], np.inf)), 2 * ref[1] + 1e-3, np.inf):
                g = pl.plan(*args, cost_cap=cap)
                assert_same_plan(g, ref, o)
                assert g.n_decided == space
            g = pl.plan(*args)
            assert_same_plan(g, ref, o)
        monkeypatch.delenv("SMILESS_BB_DEPTH", raising=False)
        g = pl.plan(*args, cost_cap=ref[1])
        fewer += g.n_full_evals < off.n_full_evals
        # a cap below OPT leaves nothing eligible
        g = pl.plan(*args, cost_cap=float(np.nextafter(ref[1], 0)))
        assert g.status == S.INFEASIBLE and g.index is None
        # sub-ranges and shards with a cap between two feasible costs
        costs = np.unique(oc[of])
        if len(costs) > 1:
            cap = float(costs[len(costs) // 2])
            b, e = int(rng.integers(0, space // 2)), int(rng.integers(space // 2, space + 1))
            want = _lex_min(oc[b:e], of[b:e], cap)
            g = pl.plan(*args, begin=b, end=e, cost_cap=cap)
            assert (None if want is None else (want[0] + b, want[1])) == \
                (None if g.index is None else (g.index, g.cost))
            parts = [pl.plan(*args, shard=s_, n_shards=3, cost_cap=cap) for s_ in range(3)]
            feas = [(r.cost, r.index) for r in parts if r.feasible]
            want = _lex_min(oc, of, cap)
            assert (min(feas) if feas else None) == (None if want is None else (want[1], want[0]))
        checked += 1
    assert checked >= 8 and fewer >= 1


def test_cost_cap_ties_and_single_candidate():
    """Zero prices: every candidate costs 0, a cap of 0 keeps them all and the winner is the
    lowest feasible index; a fully pinned (single-candidate) plan honours the cap too."""
    rng = np.random.default_rng(3)
    p = W.random_problem(rng, 3, 3, 3, 20, sla_us=10**8)
    p = p.replace(price_per_us=np.zeros_like(p.price_per_us))
    pl = S.planner_for(p)
    g = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, cost_cap=0.0)
    assert g.index == 0 and g.cost == 0.0
    p2 = p.replace(price_per_us=np.ones_like(p.price_per_us) / 1024)
    o = OracleProblem(p2, n_fixed=3, fixed_digits=[0, 0, 0])
    c, l, f = o.evaluate([0])
    pl2 = S.planner_for(p2)
    kw = dict(n_fixed=3, fixed_digits=[0, 0, 0])
    g = pl2.plan(p2.arrivals_us, p2.sla_us, p2.windows_us, cost_cap=float(c[0]), **kw)
    assert g.index == 0 and g.cost == c[0]
    g = pl2.plan(p2.arrivals_us, p2.sla_us, p2.windows_us, cost_cap=float(np.nextafter(c[0], 0)), **kw)
    assert g.status == S.INFEASIBLE


def test_exact_evaluator_wide_dags():
    """The warp-per-candidate exact evaluator (lane k = function k, DAG levels in parallel) at
    the ABI limits: 32 functions, joins of up to 8 predecessors (past its 4 register-cached
    ones), several sinks; evaluated indices and a plan sub-range against the oracle."""
    rng = np.random.default_rng(71)
    for t in range(3):
        p = W.random_problem(rng, 32, 2, 1 + t % 2, 300, max_preds=8, sla_us=5 * 10**8)
        space = p.space_size()
        o = OracleProblem(p)
        idx = rng.integers(0, space, size=96, dtype=np.uint64)
        pl = S.planner_for(p)
        gc, gl, gf = pl.evaluate(idx, p.arrivals_us, p.sla_us, p.windows_us)
        assert_same_eval(gc, gl, gf, *o.evaluate(idx))
        b = int(rng.integers(0, space - 4096))
        g = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, begin=b, end=b + 4096)
        assert_same_plan(g, o.plan(begin=b, end=b + 4096), o)


@pytest.mark.parametrize("name", ["C2", "C3"])
def test_bench_full_space_seed_cap_same_opt(monkeypatch, name):
    """bench.full_space_opt with the window-0 seed cap (SMILESS_SEED_CAP=1: the best cost of
    the window-0 sub-space caps the whole-space plan) returns the uncapped run's OPT, and the
    winner re-checks on the oracle bit for bit (DESIGN.md §11 item 3)."""
    import torch
    import bench
    dev = torch.device("cuda:0")
    stream = torch.cuda.current_stream(dev)
    outs = {}
    for seed in ("0", "1"):
        monkeypatch.setenv("SMILESS_SEED_CAP", seed)
        outs[seed] = bench.full_space_opt(name, S, 0, 1, dev, dev, stream, 0, lambda: None)
    a, b = outs["0"], outs["1"]
    assert b["seed_cap"]["enabled"] and not a["seed_cap"]["enabled"]
    assert b["seed_cap"]["cap"] is not None and b["seed_cap"]["cap"] >= a["cost"]
    assert (b["cost"], b["index"], b["max_latency_us"]) == (a["cost"], a["index"], a["max_latency_us"])
    assert b["oracle_check"] == {"feasible": True, "cost_bits_equal": True, "latency_equal": True}


# ---------------------------------------------------------------------------------------
# Multi-GPU sharding of the exact pruned plans: interleaved deep B&B work
# ---------------------------------------------------------------------------------------

@pytest.mark.parametrize("listcap", ["0", "1", "5"])
def test_branch_and_bound_shards_and_list_splits_are_exact(listcap, monkeypatch):
    """Every (D, DA) pair, with and without a middle level DM (three-level B&B), 2 and 3
    shards, and a forced small survivor-list capacity (a survivor's children then span
    several launches): the shards' merged
    per-candidate costs equal the oracle's, each candidate is decided by exactly one shard,
    and the best shard winner is the oracle's OPT."""
    if listcap != "0":
        monkeypatch.setenv("SMILESS_BB_LISTCAP", listcap)
    rng = np.random.default_rng(61 + int(listcap))
    n_checked = 0
    for t in range(40):
        if n_checked == 6:
            break
        n = int(rng.integers(4, 7))
        p = W.random_problem(rng, n, 3, int(rng.integers(2, 4)), int(rng.integers(20, 120)),
                             sla_us=int(rng.integers(15_000, 60_000)))
        space = p.space_size()
        if space > 30000:
            continue
        o = OracleProblem(p)
        oc, ol, of = o.evaluate(np.arange(space, dtype=np.uint64))
        ref = o.plan()
        for d, da, dm in [(d, da, dm) for d in range(2, n) for da in [0] + list(range(1, d))
                          for dm in [0] + ([da + 1] if 0 < da and da + 1 < d else [])]:
                monkeypatch.setenv("SMILESS_BB_DEPTH", str(d))
                monkeypatch.setenv("SMILESS_BB_DEPTH_A", str(da))
                monkeypatch.setenv("SMILESS_BB_DEPTH_M", str(dm))
                pl = S.planner_for(p)
                assert ("#define SM_DM %d" % dm) in pl.kernel_source(p.arrivals_us, p.sla_us, p.windows_us)
                for world in (2, 3):
                    merged = np.full(space, np.nan)
                    parts = []
                    for s_ in range(world):
                        out = np.empty(space)
                        parts.append(pl.plan(p.arrivals_us, p.sla_us, p.windows_us, shard=s_, n_shards=world,
                                             cost_out=out))
                        hit = ~np.isnan(out)
                        assert np.isnan(merged[hit]).all()          # no candidate evaluated twice
                        merged[hit] = out[hit]
                    assert_dump_matches(merged, oc, of)
                    assert sum(r.n_decided for r in parts) == space
                    win = [(r.cost, r.index) for r in parts if r.feasible]
                    if ref is None:
                        assert not win
                    else:
                        assert min(win) == (ref[1], ref[0])
                    # with the cost bound (no dump): same OPT
                    parts = [pl.plan(p.arrivals_us, p.sla_us, p.windows_us, shard=s_, n_shards=world)
                             for s_ in range(world)]
                    assert sum(r.n_decided for r in parts) == space
                    win = [(r.cost, r.index) for r in parts if r.feasible]
                    assert (min(win) if win else None) == (None if ref is None else (ref[1], ref[0]))
        n_checked += 1
    assert n_checked >= 4


@pytest.mark.parametrize("name,world", [("C2", 2), ("C3", 2), ("C2", 4), ("C3", 3)])
def test_full_space_plan_shards_split_the_work(name, world):
    """The exact full-space plans of C2 (2^42) and C3 (7.2e15) sharded over `world` ranks
    (run one after the other on this GPU): every rank decides at least space / (2 world)
    candidates, the shares sum to the space, and the best rank winner is the single-rank
    OPT (which the oracle re-checks)."""
    import torch
    p = W.make_config(name)
    pl = S.planner_for(p)
    arr = torch.as_tensor(p.arrivals_us).cuda()
    one = pl.plan(arr, p.sla_us, p.windows_us)
    assert one.feasible
    oc, ol, of = OracleProblem(p).evaluate([one.index])
    assert of[0] and oc[0] == one.cost and ol[0] == one.max_latency_us
    space = p.space_size()
    parts = [pl.plan(arr, p.sla_us, p.windows_us, shard=s_, n_shards=world) for s_ in range(world)]
    assert sum(r.n_decided for r in parts) == space
    for r in parts:
        assert r.n_decided >= space // (2 * world), [q.n_decided for q in parts]
    assert sum(r.n_full_evals for r in parts) > 0      # (a rank's whole share may be pruned by the bounds)
    assert min((r.cost, r.index) for r in parts if r.feasible) == (one.cost, one.index)


@pytest.mark.parametrize("levels", ["two", "auto"])
def test_c5_heavy_subplan_children_split_over_launches(levels, monkeypatch):
    """C5s's sub-plan of function 0's digit 112 (2^63 candidates).  levels = two (DA = 4, no
    middle level): its shallow survivors have 2^28 deep children each, more than one survivor
    list holds, so their children run over several deep launches.  auto: the default three
    levels.  Single rank and 2 shards agree; the oracle re-checks the winner."""
    import torch
    if levels == "two":
        monkeypatch.setenv("SMILESS_BB_DEPTH_A", "4")
        monkeypatch.setenv("SMILESS_BB_DEPTH_M", "0")
    p = W.make_config("C5s")
    pl = S.planner_for(p)
    arr = torch.as_tensor(p.arrivals_us).cuda()
    kw = dict(n_fixed=1, fixed_digits=[112])
    one = pl.plan(arr, p.sla_us, p.windows_us, **kw)
    assert one.feasible
    oc, ol, of = OracleProblem(p, **kw).evaluate([one.index])
    assert of[0] and oc[0] == one.cost and ol[0] == one.max_latency_us
    parts = [pl.plan(arr, p.sla_us, p.windows_us, shard=s_, n_shards=2, **kw) for s_ in range(2)]
    assert sum(r.n_decided for r in parts) == 1 << 63
    assert min((r.cost, r.index) for r in parts if r.feasible) == (one.cost, one.index)


# ---------------------------------------------------------------------------------------
# Full-size parity (J = 10^4) of the fast evaluators around each config's OPT, and every
# int32 chunk length K
# ---------------------------------------------------------------------------------------

def _fastest_digit0(p):
    """Digit of function 0 on its fastest configuration, keep-alive (a feasible sub-space of
    C5 with scale-out)."""
    return int(np.argmin(p.exec_us[:int(p.n_configs[0])])) * len(p.windows_us)


@pytest.mark.parametrize("name,nf,fixed", [("C2", 0, []), ("C3", 0, []), ("C3s", 0, []), ("C5s", 1, [112]),
                                           ("C5", 1, None)])
def test_full_size_per_candidate_costs_around_opt(name, nf, fixed):
    """P:305 (OPT by exhaustive search): 4,096 consecutive candidates around the exact plan's
    winner at the full J = 10^4, evaluated by the memoised throughput kernels (no pruning)
    and by the prune-mode plan kernel, cost bits and feasibility per candidate against the
    oracle.  C5 pins function 0's digit (its space is 2^70)."""
    import torch
    p = W.make_config(name)
    if fixed is None:
        fixed = [_fastest_digit0(p)]
    kw = dict(n_fixed=nf, fixed_digits=fixed)
    pl = S.planner_for(p)
    arr = torch.as_tensor(p.arrivals_us).cuda()
    opt = pl.plan(arr, p.sla_us, p.windows_us, **kw)
    assert opt.feasible
    lo = opt.index // 4096 * 4096
    oc, ol, of = OracleProblem(p, **kw).evaluate(np.arange(lo, lo + 4096, dtype=np.uint64))
    assert of.any() and of[opt.index - lo] and oc[opt.index - lo] == opt.cost
    for flags in (S.FLAG_NO_PRUNE, 0):
        out = np.empty(4096)
        r = pl.plan(arr, p.sla_us, p.windows_us, begin=lo, end=lo + 4096, flags=flags, cost_out=out, **kw)
        assert_dump_matches(out, oc, of)
        assert r.index == opt.index and r.cost == opt.cost


@pytest.mark.parametrize("K", ["32", "16", "8", "4"])
def test_every_int32_chunk_length_is_exact(K, monkeypatch):
    """The int32 path rebases times every K steps; K in {32, 16, 8, 4} is chosen only for
    large windows/SLAs, so force it (SMILESS_FORCE_K) on random DAGs and on a full-size C3
    slice: per-candidate costs in throughput (memo) and prune mode equal the oracle's."""
    monkeypatch.setenv("SMILESS_FORCE_K", K)
    rng = np.random.default_rng(300 + int(K))
    n_checked = 0
    for t in range(60):
        n = int(rng.integers(2, 7))
        p = W.random_problem(rng, n, 4, int(rng.integers(1, 6)), int(rng.integers(2, 140)))
        space = p.space_size()
        if space > 20000:
            continue
        oc, ol, of = OracleProblem(p).evaluate(np.arange(space, dtype=np.uint64))
        pl = S.planner_for(p)
        for flags in (0, S.FLAG_NO_PRUNE):
            out = np.empty(space)
            r = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, flags=flags, cost_out=out)
            assert_dump_matches(out, oc, of)
            assert not r.int64_path
        n_checked += 1
        if n_checked == 12:
            break
    assert n_checked >= 8
    p = W.make_config("C3")
    pl = S.planner_for(p)
    opt = pl.plan(p.arrivals_us, p.sla_us, p.windows_us)          # exact full-space plan with this K
    assert opt.feasible and not opt.int64_path
    lo = opt.index // 2048 * 2048
    oc, ol, of = OracleProblem(p).evaluate(np.arange(lo, lo + 2048, dtype=np.uint64))
    assert of[opt.index - lo] and oc[opt.index - lo] == opt.cost
    out = np.empty(2048)
    r = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, begin=lo, end=lo + 2048, flags=S.FLAG_NO_PRUNE, cost_out=out)
    assert not r.int64_path
    assert_dump_matches(out, oc, of)


# ---------------------------------------------------------------------------------------
# NEXT-4 inside model M: scale-out instances (reading G26) on every kernel path
# ---------------------------------------------------------------------------------------

@pytest.mark.parametrize("lring", ["0", "1"])
def test_scale_out_golden_on_the_gpu(lring, monkeypatch):
    """Golden S_E7 (hand-worked) through smiless_evaluate and smiless_plan, with the
    scaled-out last function as the virtual sink (lring 0) or as ring variants (lring 1)."""
    monkeypatch.setenv("SMILESS_LRING", lring)
    import json, os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "S_E7_scale_out.json")))
    for case in g["cases"]:
        ptr, idx = W.csr_from_preds([[]])
        p = W.Problem("t", ptr, idx, np.ones(1, np.int32), np.asarray(case["exec_us"], np.int32),
                      np.asarray(case["init_us"], np.int32), np.ones(1), np.asarray(case["arrivals_us"], np.int64),
                      10**6, np.asarray(case["windows_us"], np.int32))
        pl = S.planner_for(p)
        c, l, f = pl.evaluate([0], p.arrivals_us, p.sla_us, p.windows_us, instances=case["instances"])
        assert c[0] == float(sum(case["billed"])) and l[0] == max(case["latency"])
        for flags in (0, S.FLAG_NO_PRUNE, S.FLAG_FORCE_INT64):
            r = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, instances=case["instances"], flags=flags)
            assert r.index == 0 and r.cost == c[0] and r.max_latency_us == l[0]


@pytest.mark.parametrize("lring", ["0", "1"])
@pytest.mark.parametrize("flags", [0, S.FLAG_NO_PRUNE, S.FLAG_FORCE_INT64, S.FLAG_NO_PRUNE | S.FLAG_FORCE_INT64])
def test_scale_out_random_dags_per_candidate_costs(flags, lring, monkeypatch):
    """Random DAGs with 1-4 round-robin instances per function (rings, prologue, virtual
    sink, scale-out billing): every candidate's cost bits and feasibility equal the oracle's,
    the winner is the oracle's OPT, and smiless_evaluate (the independent exact kernel)
    agrees too.  lring: a scaled-out last function as ring variants instead of the virtual
    sink (SMILESS_LRING)."""
    monkeypatch.setenv("SMILESS_LRING", lring)
    rng = np.random.default_rng(400 + flags)
    n_checked = 0
    for t in range(80):
        n = int(rng.integers(1, 7))
        p = W.random_problem(rng, n, 4, int(rng.integers(1, 5)), int(rng.integers(1, 140)))
        space = p.space_size()
        if space > 20000:
            continue
        inst = [int(rng.integers(1, 5)) for _ in range(n)]
        o = OracleProblem(p, instances=inst)
        idx = np.arange(space, dtype=np.uint64)
        oc, ol, of = o.evaluate(idx)
        pl = S.planner_for(p)
        out = np.empty(space)
        g = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, flags=flags, cost_out=out, instances=inst)
        assert_dump_matches(out, oc, of)
        assert_same_plan(g, o.plan(), o)
        gc, gl, gf = pl.evaluate(idx[:512], p.arrivals_us, p.sla_us, p.windows_us, instances=inst)
        assert_same_eval(gc, gl, gf, oc[:512], ol[:512], of[:512])
        n_checked += 1
        if n_checked == 25:
            break
    assert n_checked >= 15


@pytest.mark.parametrize("lring", ["0", "1"])
def test_scale_out_branch_and_bound_and_shards(lring, monkeypatch):
    """B&B depths with scale-out functions (lower-bound relaxation downstream of them),
    2 shards, and the cost bound: per-candidate parity and the oracle's OPT."""
    monkeypatch.setenv("SMILESS_LRING", lring)
    rng = np.random.default_rng(77)
    n_checked = 0
    for t in range(40):
        n = int(rng.integers(4, 7))
        p = W.random_problem(rng, n, 3, int(rng.integers(2, 4)), int(rng.integers(20, 120)),
                             sla_us=int(rng.integers(15_000, 60_000)))
        space = p.space_size()
        if space > 30000:
            continue
        inst = [int(rng.integers(1, 4)) for _ in range(n)]
        o = OracleProblem(p, instances=inst)
        oc, ol, of = o.evaluate(np.arange(space, dtype=np.uint64))
        ref = o.plan()
        for d in range(2, n):
            for da, dm in ((0, 0), (1, 0), (1, 2)):
                if da >= d or dm >= d:
                    continue
                monkeypatch.setenv("SMILESS_BB_DEPTH", str(d))
                monkeypatch.setenv("SMILESS_BB_DEPTH_A", str(da))
                monkeypatch.setenv("SMILESS_BB_DEPTH_M", str(dm))
                pl = S.planner_for(p)
                out = np.empty(space)
                g = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, cost_out=out, instances=inst)
                assert_dump_matches(out, oc, of)
                assert_same_plan(g, ref, o)
                g = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, instances=inst)      # cost bound on
                assert_same_plan(g, ref, o)
                parts = [pl.plan(p.arrivals_us, p.sla_us, p.windows_us, shard=s_, n_shards=2, instances=inst)
                         for s_ in range(2)]
                assert sum(r.n_decided for r in parts) == space
                win = [(r.cost, r.index) for r in parts if r.feasible]
                assert (min(win) if win else None) == (None if ref is None else (ref[1], ref[0]))
        n_checked += 1
        if n_checked == 8:
            break
    assert n_checked >= 5


@pytest.mark.parametrize("lring", ["0", "1"])
@pytest.mark.parametrize("K", ["64", "16", "8"])
def test_scale_out_chunk_lengths(K, lring, monkeypatch):
    """The prologue must sit inside chunk 0 (K >= prologue) and the rings span chunk
    rebases: forced K with up to 8 instances (prologue 8) against the oracle."""
    monkeypatch.setenv("SMILESS_FORCE_K", K)
    monkeypatch.setenv("SMILESS_LRING", lring)
    rng = np.random.default_rng(500 + int(K))
    for t in range(30):
        n = int(rng.integers(1, 5))
        p = W.random_problem(rng, n, 3, int(rng.integers(1, 4)), int(rng.integers(2, 100)))
        space = p.space_size()
        if space > 8000:
            continue
        inst = [int(rng.integers(1, 9)) for _ in range(n)]
        o = OracleProblem(p, instances=inst)
        oc, ol, of = o.evaluate(np.arange(space, dtype=np.uint64))
        pl = S.planner_for(p)
        for flags in (0, S.FLAG_NO_PRUNE):
            out = np.empty(space)
            pl.plan(p.arrivals_us, p.sla_us, p.windows_us, flags=flags, cost_out=out, instances=inst)
            assert_dump_matches(out, oc, of)


def test_c2_window0_subspace_matches_oracle_brute_force():
    """tests/golden/C2_window0_bruteforce.json: the plain oracle walked every one of the
    16^6 keep-alive candidates of C2 at J = 10^4 (tools/c2_window0_bruteforce.py, ~46 min on
    8 cores).  The GPU plan of that sub-space returns the same index and cost bits, and the
    full 2^42 plan's OPT is that same candidate (C2's optimum keeps every function alive)."""
    import json, os
    import torch
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "C2_window0_bruteforce.json")))
    p = W.make_config("C2")
    pl = S.planner_for(p)
    arr = torch.as_tensor(p.arrivals_us).cuda()
    for flags in (0, S.FLAG_NO_PRUNE):
        r = pl.plan(arr, p.sla_us, p.windows_us[:1], flags=flags)
        assert r.index == g["index_subspace"] and r.cost.hex() == g["cost_hex"]
        assert r.max_latency_us == g["max_latency_us"] and r.n_decided == g["space"]
    full = pl.plan(arr, p.sla_us, p.windows_us)
    assert full.index == g["index_full_space"] and full.cost.hex() == g["cost_hex"]
    assert full.config.tolist() == g["config"] and (full.window == 0).all()


# ---------------------------------------------------------------------------------------
# NEXT-3 with model M: per-path exhaustive GPU plans + the paper's combine
# ---------------------------------------------------------------------------------------

def test_decompose_plan_golden_on_the_gpu():
    """Golden P2m (hand-derived) through smiless_decompose_plan."""
    import json, os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "P2m_decompose_model_m.json")))
    ptr, idx = W.csr_from_preds(g["preds"])
    p = W.Problem("t", ptr, idx, np.asarray(g["n_configs"], np.int32), np.asarray(g["exec_us"], np.int32),
                  np.asarray(g["init_us"], np.int32), np.asarray(g["price_per_us"], np.float64),
                  np.asarray(g["arrivals_us"], np.int64), g["sla_us"], np.asarray(g["windows_us"], np.int32))
    r, n_paths = S.planner_for(p).decompose_plan(p.arrivals_us, p.sla_us, p.windows_us)
    assert n_paths == 2 and r.feasible
    assert r.config.tolist() == g["expected_configs"] and r.window.tolist() == [0] * 4
    assert r.max_latency_us == g["expected_latency_us"] and r.cost == g["expected_cost"]


def test_decompose_plan_matches_oracle_walk():
    """Random DAGs (joins, several sinks, instances): the library's per-path GPU plans and
    combine equal oracle/decompose_m.py step for step (configs, windows, cost bits)."""
    from oracle.decompose_m import decompose_plan
    rng = np.random.default_rng(808)
    n_checked = n_feasible = 0
    for t in range(60):
        n = int(rng.integers(2, 6))
        p = W.random_problem(rng, n, 3, int(rng.integers(1, 4)), int(rng.integers(2, 40)),
                             sla_us=int(rng.integers(8_000, 40_000)))
        if t % 2:
            p = p.replace(instances=np.asarray([int(rng.integers(1, 3)) for _ in range(n)], np.int32))
        pl = S.planner_for(p)
        r, n_paths = pl.decompose_plan(p.arrivals_us, p.sla_us, p.windows_us)
        cfg, win, cost, lat, ok, np_ = decompose_plan(p, OracleProblem)
        assert n_paths == np_
        assert r.feasible == ok
        if ok:
            assert r.config.tolist() == cfg and r.window.tolist() == win
            assert r.cost == cost and r.max_latency_us == lat
            n_feasible += 1
        n_checked += 1
        if n_checked == 30:
            break
    assert n_feasible >= 5


@pytest.mark.parametrize("name", ["C3", "C5"])
def test_decompose_plan_full_size(name):
    """C3 / C5 at J = 10^4 with scale-out: the per-path decomposition yields a plan; if it is
    feasible its cost is >= the exhaustive OPT's on the same space (C3) and it re-checks on
    the oracle."""
    p = W.make_config(name)
    pl = S.planner_for(p)
    r, n_paths = pl.decompose_plan(p.arrivals_us, p.sla_us, p.windows_us)
    assert n_paths >= 2
    if r.feasible:
        Wn = len(p.windows_us)
        kw = dict(n_fixed=1, fixed_digits=[int(r.config[0]) * Wn + int(r.window[0])]) if name == "C5" else {}
        oc, ol, of = OracleProblem(p, **kw).evaluate([r.index])
        assert of[0] and oc[0] == r.cost and ol[0] == r.max_latency_us
        if name != "C5":
            opt = pl.plan(p.arrivals_us, p.sla_us, p.windows_us)
            assert opt.feasible and opt.cost <= r.cost


def _decompose_rank(rank, world, port, name, out_q):
    import os
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    from paper_conf_sc_luxl0y024_b200.dist import decompose_plan_distributed
    p = W.make_config(name) if name != "rand" else W.random_problem(np.random.default_rng(9), 5, 3, 2, 60,
                                                                    sla_us=30_000)
    pl = S.planner_for(p)
    r, n_paths = decompose_plan_distributed(pl, p.arrivals_us, p.sla_us, p.windows_us, device="cpu")
    out_q.put((rank, (r.status, r.index, r.cost, r.max_latency_us, r.config.tolist(), r.window.tolist(), n_paths)))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("name,world", [("C3", 2), ("C2", 3), ("rand", 2)])
def test_decompose_plan_sharded_over_ranks(name, world):
    """NEXT-3 per-path GPU sharding: `world` ranks (processes on this one GPU,
    gloo collectives inside the library's reduce callback) each plan their share of every
    path; every rank returns the single-rank decomposition exactly."""
    import socket
    import torch.multiprocessing as mp
    p = W.make_config(name) if name != "rand" else W.random_problem(np.random.default_rng(9), 5, 3, 2, 60,
                                                                    sla_us=30_000)
    one, n_paths = S.planner_for(p).decompose_plan(p.arrivals_us, p.sla_us, p.windows_us)
    sock = socket.socket()
    sock.bind(("127.0.0.1", 0))
    port = sock.getsockname()[1]
    sock.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_decompose_rank, args=(r, world, port, name, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    out = dict(q.get(timeout=600) for _ in range(world))
    for pr in procs:
        pr.join(timeout=120)
        assert pr.exitcode == 0
    want = (one.status, one.index, one.cost, one.max_latency_us, one.config.tolist(), one.window.tolist(), n_paths)
    for r in range(world):
        assert out[r] == want


def test_arrivals_device_view_at_8_byte_offset():
    """Arrivals as a device tensor view 8 bytes into its allocation (only int64-aligned):
    the plan, its exact winner re-check (cp.async arrival ring) and smiless_evaluate agree
    with the oracle."""
    import torch
    p = W.make_config("C1")
    full = torch.as_tensor(np.concatenate([[0], p.arrivals_us])).cuda()
    view = full[1:]
    assert view.data_ptr() % 16 == 8
    pl = S.planner_for(p)
    g = pl.plan(view, p.sla_us, p.windows_us)
    o = OracleProblem(p)
    assert_same_plan(g, o.plan(), o)
    idx = np.arange(0, 4096, 13, dtype=np.uint64)
    assert_same_eval(*pl.evaluate(idx, view, p.sla_us, p.windows_us), *o.evaluate(idx))


# ---------------------------------------------------------------------------------------
# smiless_plan_digits: a range of values of the last pinned digit in one call
# ---------------------------------------------------------------------------------------

@pytest.mark.parametrize("flags", [0, S.FLAG_NO_PRUNE])
def test_plan_digits_matches_oracle_over_the_union(flags):
    """Every value of the last pinned digit in [d0, d1), one call, the incumbent carried on the
    device: the (cost, digit, index) minimum equals one oracle plan over the union of the digits'
    sub-spaces (ties to the lowest digit, then index), every candidate is counted once, and the
    shards of the call together decide the union; also with a cost cap at OPT."""
    rng = np.random.default_rng(909 + flags)
    n_checked = 0
    for t in range(60):
        n = int(rng.integers(3, 6))
        p = W.random_problem(rng, n, 4, int(rng.integers(2, 4)), int(rng.integers(20, 150)),
                             sla_us=int(rng.integers(15_000, 60_000)))
        Wn = len(p.windows_us)
        nf = int(rng.integers(1, 3))
        fixed = [int(rng.integers(0, p.n_configs[k] * Wn)) for k in range(nf)]
        radix = int(p.n_configs[nf - 1]) * Wn
        o_pre = OracleProblem(p, n_fixed=nf - 1, fixed_digits=fixed[:-1])
        S_ = OracleProblem(p, n_fixed=nf, fixed_digits=fixed).space_size()
        if S_ * radix > 40000 or radix < 3:
            continue
        d0 = int(rng.integers(0, radix - 1))
        d1 = int(rng.integers(d0 + 1, radix + 1))
        ref = o_pre.plan(begin=d0 * S_, end=d1 * S_)
        pl = S.planner_for(p)
        kw = dict(n_fixed=nf, fixed_digits=fixed, flags=flags)
        r = pl.plan_digits(p.arrivals_us, p.sla_us, p.windows_us, d0, d1, **kw)
        assert r.n_decided == (d1 - d0) * S_
        if ref is None:
            assert not r.feasible and r.digit is None
        else:
            assert r.feasible and (r.digit * S_ + r.index, r.cost, r.max_latency_us) == ref
            assert r.config.tolist() == o_pre.decode(ref[0])[0].tolist()
            rc = pl.plan_digits(p.arrivals_us, p.sla_us, p.windows_us, d0, d1, cost_cap=ref[1], **dict(kw, flags=0))
            assert (rc.digit * S_ + rc.index, rc.cost) == ref[:2]
        parts = [pl.plan_digits(p.arrivals_us, p.sla_us, p.windows_us, d0, d1, shard=s_, n_shards=3, **kw)
                 for s_ in range(3)]
        assert sum(q.n_decided for q in parts) == (d1 - d0) * S_
        win = [(q.cost, q.digit, q.index) for q in parts if q.feasible]
        assert (min(win) if win else None) == (None if ref is None else (ref[1], ref[0] // S_, ref[0] % S_))
        n_checked += 1
        if n_checked == 10:
            break
    assert n_checked >= 6


def test_plan_digits_c5_equals_the_per_digit_loop():
    """C5 (2^70 candidates, scale-out) in one smiless_plan_digits call over function 0's 128
    digits: the same OPT as planning the digits one call each with the running best as cost
    cap, 2^70 candidates decided (beyond 2^64: n_decided_hi), and the winner re-checks on the
    oracle."""
    p = W.make_config("C5")
    pl = S.planner_for(p)
    Wn = len(p.windows_us)
    radix = int(p.n_configs[0]) * Wn
    r = pl.plan_digits(p.arrivals_us, p.sla_us, p.windows_us, 0, radix, n_fixed=1, fixed_digits=[0])
    assert r.n_decided == 1 << 70
    best = None
    for d in range(radix):
        kw = dict(n_fixed=1, fixed_digits=[d])
        if best is not None:
            kw["cost_cap"] = best[0]
        q = pl.plan(p.arrivals_us, p.sla_us, p.windows_us, **kw)
        if q.feasible and (best is None or (q.cost, d, q.index) < best[:3]):
            best = (q.cost, d, q.index, q.max_latency_us)
    assert best is not None and (r.cost, r.digit, r.index, r.max_latency_us) == best
    c, l, f = OracleProblem(p, n_fixed=1, fixed_digits=[r.digit]).evaluate([r.index])
    assert f[0] and c[0] == r.cost and l[0] == r.max_latency_us
