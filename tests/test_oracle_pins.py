"""Pins of the CPU oracle against things other than itself (-m "not gpu").

Each test names the PAPER.md passage ("P:n") or the textbook result it pins.
A plausible mistake anywhere in the oracle (dropped billing term, wrong sign,
wrong predecessor, swapped case, wrong digit order, FMA in the cost) fails at
least one of them.
"""
import glob
import itertools
import json
import os
from fractions import Fraction

import numpy as np
import pytest

import workloads as W
from oracle import OracleProblem, des

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def mk(preds, exec_us, init_us, arrivals, windows, sla=10**9, prices=None, n_configs=None):
    ptr, idx = W.csr_from_preds(preds)
    n = len(preds)
    ncfg = np.ones(n, np.int32) if n_configs is None else np.asarray(n_configs, np.int32)
    tot = int(ncfg.sum())
    pr = np.ones(tot) if prices is None else np.asarray(prices, np.float64)
    return W.Problem("t", ptr, idx, ncfg, np.asarray(exec_us, np.int32), np.asarray(init_us, np.int32),
                     pr, np.asarray(arrivals, np.int64), int(sla), np.asarray(windows, np.int32))


# ---------------------------------------------------------------------------
# Worked examples (tests/golden, each with its citation and hand derivation)
# ---------------------------------------------------------------------------

@pytest.mark.parametrize("path", sorted(glob.glob(os.path.join(GOLDEN, "E*.json"))))
def test_golden_worked_examples(path):
    g = json.load(open(path))
    assert g["citation"]
    for case in g["cases"]:
        p = mk(g["preds"], g["exec_us"], g["init_us"], g["arrivals_us"], case["windows_us"])
        o = OracleProblem(p)
        cfg = [0] * p.n_funcs
        billed, lat = o.simulate(cfg, case["window_idx"])
        assert billed.tolist() == case["billed"], (path, case)
        assert lat.tolist() == case["latency"], (path, case)


# ---------------------------------------------------------------------------
# Closed forms from the paper
# ---------------------------------------------------------------------------

def test_eq5_case_I_chain_closed_form():
    """P:177-179 Eq. (5): with periodic arrivals and T_k + I_k < IT, the window
    IT - T_k - I_k hides every init: L = sum of I, C_k = (T_k + I_k) U per invocation."""
    rng = np.random.default_rng(11)
    for _ in range(200):
        n = int(rng.integers(1, 7))
        J = int(rng.integers(1, 30))
        IT = int(rng.integers(10_000, 100_000))
        I = rng.integers(0, IT // 3, size=n)
        T = rng.integers(0, IT // 3, size=n)
        windows = sorted(set(int(IT - T[k] - I[k]) for k in range(n)))
        r = np.arange(J, dtype=np.int64) * IT + int(rng.integers(0, 10**6))
        p = mk([[]] + [[k - 1] for k in range(1, n)], I, T, r, windows)
        widx = [windows.index(int(IT - T[k] - I[k])) for k in range(n)]
        billed, lat = OracleProblem(p).simulate([0] * n, widx)
        assert (lat == int(I.sum())).all()
        assert billed.tolist() == [J * int(T[k] + I[k]) for k in range(n)]


def test_case_II_keepalive_closed_form():
    """keep-alive (window 0) costs IT * U per invocation after the
    first (T + I); latency as Eq. (5)."""
    rng = np.random.default_rng(12)
    for _ in range(200):
        n = int(rng.integers(1, 6))
        J = int(rng.integers(1, 30))
        IT = int(rng.integers(1000, 100_000))
        I = rng.integers(0, IT // n + 1, size=n)    # sum I <= IT: never busy
        I = np.minimum(I, IT // n)
        T = rng.integers(0, 10 * IT, size=n)
        r = np.arange(J, dtype=np.int64) * IT
        p = mk([[]] + [[k - 1] for k in range(1, n)], I, T, r, [0])
        billed, lat = OracleProblem(p).simulate([0] * n, [0] * n)
        assert (lat == int(I.sum())).all()
        assert billed.tolist() == [int(T[k] + I[k]) + (J - 1) * IT for k in range(n)]


def test_theorem_5_1_window_minimises_cost():
    """P:184 Theorem 5.1: when I1 + I2 < SLA and T2 + I2 < IT, the Case-I window
    gives the minimum cost.  Over a dense window grid the lowest-index window of
    minimum F2 cost that also meets SLA = I1 + I2 is exactly IT - T2 - I2."""
    rng = np.random.default_rng(13)
    for _ in range(40):
        IT = int(rng.integers(2000, 20000))
        I1, I2 = (int(v) for v in rng.integers(1, IT // 4, size=2))
        T1, T2 = (int(v) for v in rng.integers(1, IT // 4, size=2))
        wstar = IT - T2 - I2
        grid = sorted(set([0, wstar] + [int(v) for v in rng.integers(1, 2 * IT, size=20)]))
        r = np.arange(12, dtype=np.int64) * IT
        p = mk([[], [0]], [I1, I2], [T1, T2], r, grid, sla=I1 + I2)
        o = OracleProblem(p)
        best = None
        for wi in range(len(grid)):
            billed, lat = o.simulate([0, 0], [0, wi])
            if lat.max() <= I1 + I2 and (best is None or billed[1] < best[1]):
                best = (wi, billed[1])
        assert grid[best[0]] == wstar
        assert best[1] == 12 * (T2 + I2)


# ---------------------------------------------------------------------------
# Textbook reductions
# ---------------------------------------------------------------------------

def test_case_III_lindley_single_server():
    """P:198 Fig. 5(c): a kept-alive function serves FIFO; waiting times follow
    Lindley's recursion W_j = max(0, W_{j-1} + I - (r_j - r_{j-1}))."""
    rng = np.random.default_rng(14)
    for _ in range(300):
        J = int(rng.integers(1, 60))
        I = int(rng.integers(0, 5000))
        T = int(rng.integers(0, 5000))
        r = np.cumsum(rng.integers(0, 2 * I + 2, size=J)).astype(np.int64)
        p = mk([[]], [I], [T], r, [0])
        billed, lat = OracleProblem(p).simulate([0], [0])
        w = 0
        exp = []
        for j in range(J):
            if j:
                w = max(0, w + I - int(r[j] - r[j - 1]))
            exp.append(w + I)
        assert lat.tolist() == exp
        # keep-alive: loaded from x_0 - T to the last completion
        assert int(billed[0]) == T + (int(r[-1]) + exp[-1]) - int(r[0])


def test_keepalive_tandem_queue_recursion():
    """Chain with keep-alive everywhere is a tandem of FIFO single servers:
    D_j^k = max(D_j^{k-1}, D_{j-1}^k) + I_k (max-plus recursion)."""
    rng = np.random.default_rng(15)
    for _ in range(200):
        n = int(rng.integers(1, 6))
        J = int(rng.integers(1, 40))
        I = rng.integers(0, 3000, size=n)
        T = rng.integers(0, 3000, size=n)
        r = np.cumsum(rng.integers(0, 4000, size=J)).astype(np.int64)
        p = mk([[]] + [[k - 1] for k in range(1, n)], I, T, r, [0])
        billed, lat = OracleProblem(p).simulate([0] * n, [0] * n)
        D = np.zeros((n, J), np.int64)
        for j in range(J):
            for k in range(n):
                up = r[j] if k == 0 else D[k - 1, j]
                prev = D[k, j - 1] if j else up
                D[k, j] = max(up, prev) + I[k]
        assert lat.tolist() == (D[n - 1] - r).tolist()
        first_start = [int(r[0])] + [int(D[k - 1, 0]) for k in range(1, n)]
        assert billed.tolist() == [int(T[k] + D[k, -1] - first_start[k]) for k in range(n)]


def _all_paths_longest(preds, I):
    """Brute-force longest I-weighted source->sink path by enumerating paths."""
    n = len(preds)
    succ = [[] for _ in range(n)]
    for k, ps in enumerate(preds):
        for q in ps:
            succ[q].append(k)
    best = 0

    def walk(k, acc):
        nonlocal best
        acc += int(I[k])
        if not succ[k]:
            best = max(best, acc)
        for s in succ[k]:
            walk(s, acc)

    for k in range(n):
        if not preds[k]:
            walk(k, 0)
    return best


def test_dag_latency_is_longest_path_when_sparse():
    """'sum along sequential stages, max over parallel branches':
    with warm (keep-alive) functions and gaps larger than every path, each
    request's latency is the longest I-weighted path of the DAG."""
    rng = np.random.default_rng(16)
    for _ in range(200):
        n = int(rng.integers(1, 8))
        p0 = W.random_problem(rng, n, 1, 1, int(rng.integers(1, 8)))
        preds = [p0.preds(k) for k in range(n)]
        I = rng.integers(0, 1000, size=n)
        r = np.cumsum(rng.integers(int(I.sum()) + 1, int(I.sum()) + 5000, size=p0.arrivals_us.shape[0]))
        p = mk(preds, I, rng.integers(0, 10**6, size=n), r.astype(np.int64), [0])
        billed, lat = OracleProblem(p).simulate([0] * n, [0] * n)
        assert (lat == _all_paths_longest(preds, I)).all()


def test_mixed_radix_decode_matches_numpy():
    """Index order: function 0 most significant, config-major digit
    d_k = c_k * W + w_k; checked against numpy.unravel_index (C order)."""
    rng = np.random.default_rng(17)
    for _ in range(50):
        n = int(rng.integers(1, 6))
        p = W.random_problem(rng, n, 4, int(rng.integers(1, 4)), 2)
        o = OracleProblem(p)
        Wn = len(p.windows_us)
        shape = tuple(int(p.n_configs[k]) * Wn for k in range(n))
        assert o.space_size() == int(np.prod(shape))
        for idx in rng.integers(0, o.space_size(), size=20):
            c, w = o.decode(int(idx))
            digits = np.unravel_index(int(idx), shape)
            assert [int(d) // Wn for d in digits] == c.tolist()
            assert [int(d) % Wn for d in digits] == w.tolist()


def test_n_fixed_prefix_pins_leading_digits():
    rng = np.random.default_rng(18)
    p = W.random_problem(rng, 4, 3, 2, 5)
    Wn = len(p.windows_us)
    full = OracleProblem(p)
    fixed = [int(rng.integers(0, p.n_configs[0] * Wn))]
    sub = OracleProblem(p, n_fixed=1, fixed_digits=fixed)
    S = sub.space_size()
    assert full.space_size() == S * int(p.n_configs[0]) * Wn
    for i in range(S):
        assert np.array_equal(sub.evaluate([i])[0], full.evaluate([fixed[0] * S + i])[0])


# ---------------------------------------------------------------------------
# Independent implementation: the event-driven simulator (oracle/des.py)
# ---------------------------------------------------------------------------

def test_oracle_matches_event_driven_simulator():
    """G3/G4/G5/G6/G7 are not fixed by the paper; two independent
    implementations of the stated rule (case split vs explicit instance state
    machine with loaded-time integration) must agree exactly."""
    rng = np.random.default_rng(19)
    for _ in range(3000):
        n = int(rng.integers(1, 7))
        p = W.random_problem(rng, n, 3, int(rng.integers(1, 5)), int(rng.integers(1, 13)))
        o = OracleProblem(p)
        c = [int(rng.integers(0, p.n_configs[k])) for k in range(n)]
        w = [int(rng.integers(0, len(p.windows_us))) for k in range(n)]
        billed, lat = o.simulate(c, w)
        b2, l2 = des.simulate(p, c, w)
        assert billed.tolist() == b2
        assert lat.tolist() == l2


def _des_cost(p, c, w):
    billed, lat = des.simulate(p, c, w)
    off = np.concatenate([[0], np.cumsum(p.n_configs)])
    cost = 0.0
    for k in range(p.n_funcs):
        cost = cost + float(p.price_per_us[off[k] + c[k]]) * float(billed[k])
    return cost, max(lat)


def test_plan_equals_brute_force_through_des():
    """OPT by brute force through the independent DES (P:305 'exhaustive
    search'): lowest index among minimum-cost SLA-feasible candidates."""
    rng = np.random.default_rng(20)
    checked = 0
    for _ in range(60):
        n = int(rng.integers(1, 4))
        p = W.random_problem(rng, n, 3, int(rng.integers(1, 4)), int(rng.integers(1, 8)))
        o = OracleProblem(p)
        S = o.space_size()
        if S > 600:
            continue
        best = None
        for i in range(S):
            c, w = o.decode(i)
            cost, ml = _des_cost(p, c.tolist(), w.tolist())
            if ml <= p.sla_us and (best is None or cost < best[1]):
                best = (i, cost, ml)
        got = o.plan(n_threads=3)
        assert got == best
        checked += 1
    assert checked > 20


def test_cost_is_exact_sum_for_dyadic_prices():
    """Eq. (3)/(4): cost = sum_k U_k * billed_k.  With dyadic prices every
    product and partial sum is exact, so the oracle's cost equals the exact
    rational sum (pins: no dropped/duplicated term, right price row)."""
    rng = np.random.default_rng(21)
    for _ in range(300):
        n = int(rng.integers(1, 7))
        p = W.random_problem(rng, n, 4, 2, int(rng.integers(1, 10)))
        o = OracleProblem(p)
        i = int(rng.integers(0, o.space_size()))
        c, w = o.decode(i)
        billed, _ = o.simulate(c, w)
        off = np.concatenate([[0], np.cumsum(p.n_configs)])
        exact = sum(Fraction(float(p.price_per_us[off[k] + c[k]])) * int(billed[k]) for k in range(n))
        cost, _, _ = o.evaluate([i])
        assert Fraction(float(cost[0])) == exact


def test_plan_thread_count_invariant():
    p = W.make_config("C1")
    a = OracleProblem(p).plan(n_threads=1)
    b = OracleProblem(p).plan(n_threads=7)
    assert a == b and a is not None


# ---------------------------------------------------------------------------
# Invariants
# ---------------------------------------------------------------------------

def test_sla_nesting_and_monotone_opt():
    """Eq. (4) constraint L <= SLA: the feasible set shrinks as the SLA
    tightens and the optimal cost is non-increasing in the SLA."""
    p = W.make_config("C1", n_arrivals=40)
    o = OracleProblem(p)
    idx = np.arange(o.space_size())
    cost, lat, _ = o.evaluate(idx)
    prev_set, prev_opt = None, None
    for sla in [400_000, 800_000, 1_200_000, 1_600_000, 2_000_000, 3_000_000, 10**9]:
        feas = set(np.nonzero(lat <= sla)[0].tolist())
        if prev_set is not None:
            assert prev_set <= feas
        got = OracleProblem(p, sla_us=sla).plan()
        opt = None if got is None else got[1]
        if prev_opt is not None:
            assert opt is not None and opt <= prev_opt
        prev_set, prev_opt = feas, opt


def test_price_power_of_two_scaling():
    """Scaling every U by 2 scales every cost exactly by 2 and keeps the argmin."""
    p = W.make_config("C1", n_arrivals=30)
    a = OracleProblem(p).plan()
    b = OracleProblem(p.replace(price_per_us=p.price_per_us * 2.0)).plan()
    assert a[0] == b[0] and b[1] == 2.0 * a[1] and a[2] == b[2]


def test_integer_time_scaling():
    """Scaling all times (I, T, windows, arrivals) by k scales latencies and
    billed times by k (the model is homogeneous of degree 1 in time)."""
    rng = np.random.default_rng(22)
    for _ in range(100):
        n = int(rng.integers(1, 6))
        p = W.random_problem(rng, n, 2, 3, int(rng.integers(1, 9)))
        k = int(rng.integers(2, 6))
        q = p.replace(exec_us=p.exec_us * k, init_us=p.init_us * k, windows_us=p.windows_us * k,
                      arrivals_us=p.arrivals_us * k, sla_us=p.sla_us * k)
        c = [int(rng.integers(0, p.n_configs[i])) for i in range(n)]
        w = [int(rng.integers(0, len(p.windows_us))) for i in range(n)]
        b1, l1 = OracleProblem(p).simulate(c, w)
        b2, l2 = OracleProblem(q).simulate(c, w)
        assert (b2 == k * b1).all() and (l2 == k * l1).all()


def test_keepalive_is_latency_lower_bound():
    """Keep-alive (all windows 0) never loads a cold instance, so every done
    time -- hence every latency -- is a lower bound for any window choice
    (basis of the exact keep-alive pre-pass prune)."""
    rng = np.random.default_rng(23)
    for _ in range(1000):
        n = int(rng.integers(1, 7))
        p = W.random_problem(rng, n, 2, 4, int(rng.integers(1, 12)))
        if p.windows_us[0] != 0:
            p = p.replace(windows_us=np.concatenate([[0], p.windows_us]).astype(np.int32))
        o = OracleProblem(p)
        c = [int(rng.integers(0, p.n_configs[i])) for i in range(n)]
        w = [int(rng.integers(0, len(p.windows_us))) for i in range(n)]
        _, l_any = o.simulate(c, w)
        _, l_ka = o.simulate(c, [0] * n)
        assert (l_ka <= l_any).all()


def test_cost_monotone_in_keepalive_when_never_busy():
    """North star invariant 'cost is monotone in keep-alive', in the form that
    holds under the model (G20): for a function whose every gap
    exceeds I + T, its billed time is non-increasing and its latency
    non-decreasing as the window grows, and keep-alive (window 0) bills the most."""
    rng = np.random.default_rng(24)
    for _ in range(300):
        I = int(rng.integers(0, 2000))
        T = int(rng.integers(0, 2000))
        J = int(rng.integers(2, 20))
        r = np.cumsum(rng.integers(I + T + 1, 20000, size=J)).astype(np.int64)
        grid = sorted(set([0] + rng.integers(1, 30000, size=12).tolist()))
        p = mk([[]], [I], [T], r, grid)
        o = OracleProblem(p)
        res = [o.simulate([0], [wi]) for wi in range(len(grid))]
        billed = [int(b[0]) for b, _ in res]
        lat = [int(l.max()) for _, l in res]
        assert all(billed[i] >= billed[i + 1] for i in range(len(grid) - 1))
        assert all(lat[i] <= lat[i + 1] for i in range(1, len(grid) - 1))
        assert billed[0] == max(billed)


def test_oracle_rejects_bad_args():
    p = mk([[]], [1], [1], [0], [0])
    o = OracleProblem(p)
    o.s.n_arrivals = 0
    with pytest.raises(ValueError):
        o.evaluate([0])


# ---------------------------------------------------------------------------
# NEXT-1: the paper's derived (adaptive) pre-warm windows as per-row windows
# ---------------------------------------------------------------------------

def paper_window(T, I, IT):
    """Case I (T + I < IT) -> IT - T - I; Case II -> 0 (keep alive)."""
    return IT - T - I if T + I < IT else 0


def test_derived_windows_reproduce_eq5_on_periodic_arrivals():
    """With the paper's derived windows and periodic arrivals the oracle gives Eq. (5):
    L = sum of I, C_k = (T_k + I_k) per invocation in Case I and IT per invocation after
    the first in Case II -- for every config of a random chain."""
    rng = np.random.default_rng(31)
    for _ in range(100):
        n = int(rng.integers(1, 5))
        M = int(rng.integers(1, 4))
        IT = int(rng.integers(20_000, 100_000))
        J = int(rng.integers(2, 25))
        I = rng.integers(0, IT // (n + 1), size=n * M)          # sum of I over a path < IT: never busy
        T = rng.integers(0, 2 * IT, size=n * M)
        p = mk([[]] + [[k - 1] for k in range(1, n)], I, T, np.arange(J, dtype=np.int64) * IT, [0],
               n_configs=[M] * n, prices=np.ones(n * M))
        rw = [paper_window(int(T[r]), int(I[r]), IT) for r in range(n * M)]
        o = OracleProblem(p, row_windows=rw)
        for _ in range(5):
            c = [int(rng.integers(0, M)) for _ in range(n)]
            billed, lat = o.simulate(c, [0] * n)
            rows = [k * M + c[k] for k in range(n)]
            assert (lat == sum(int(I[r]) for r in rows)).all()
            for k, r in enumerate(rows):
                if T[r] + I[r] < IT:
                    assert billed[k] == J * int(T[r] + I[r])
                else:
                    assert billed[k] == int(T[r] + I[r]) + (J - 1) * IT


# ---------------------------------------------------------------------------
# Hand-derived paper examples for the NEXT oracles and the cost rounding
# (tests/golden/P*.json, each with its citation and derivation)
# ---------------------------------------------------------------------------

def _golden(name):
    return json.load(open(os.path.join(GOLDEN, name)))


def _problem_from(g, windows=(0,)):
    return mk(g["preds"], g["exec_us"], g["init_us"], g["arrivals_us"], list(windows), sla=g.get("sla_us", 10**9),
              prices=g.get("price_per_us") or [float.fromhex(h) for h in g["price_per_us_hex"]],
              n_configs=g.get("n_configs"))


@pytest.mark.parametrize("name", ["P1_top1_walk_chain.json", "P1b_top1_ranking_case_I_II.json"])
def test_top1_walk_follows_fig6_narrative(name):
    """the Top-1 walk visits T^0 -> T^1_1 -> T^1_2 -> T^2_2 -> T^1_3 -> T^2_3 ->
    T^3_3 on the hand-built chain (golden P1), ranks configurations by the Case I / Case II
    per-invocation cost (golden P1b), and stops at the hand-derived leaf."""
    from oracle.top1 import top1_search
    g = _golden(name)
    p = _problem_from(g)
    trace = []
    cfg, cost, lat, ok, nodes = top1_search(p, g["it_us"], g["row_windows_us"], OracleProblem, trace=trace)
    assert [[l, c, f] for l, c, f in trace] == g["expected_walk"]
    assert cfg == g["expected_leaf"] and ok
    assert lat == g["expected_latency_us"] and cost == g["expected_cost"]


def test_decompose_combine_on_diamond():
    """paths of the diamond, each path's Top-1 choice, F_s/F_e take the fastest
    of their paths' choices, branch functions keep their path latency (golden P2)."""
    from oracle.decompose import decompose_search
    g = _golden("P2_decompose_diamond.json")
    p = _problem_from(g)
    tr = {}
    cfg, cost, lat, ok, n_paths = decompose_search(p, g["it_us"], g["row_windows_us"], OracleProblem, trace=tr)
    assert tr["paths"] == g["expected_paths"] and n_paths == 2
    assert tr["path_choices"] == g["expected_path_choices"]
    assert tr["path_latency"] == g["expected_path_latency"]
    assert cfg == g["expected_combined"] and ok
    assert lat == g["expected_latency_us"] and cost == g["expected_cost"]


def _autoscale_golden():
    g = _golden("P3_autoscale_eq7.json")

    class _P:
        n_funcs = len(g["n_configs"])
        n_configs = g["n_configs"]
        price_per_us = np.asarray([float.fromhex(h) for h in g["price_per_us_hex"]])
    exp = [(c, b, i, float(x)) for c, b, i, x in g["expected"]]
    return g, _P, exp


def test_autoscale_eq7_hand_worked_with_tie():
    """P:226-239 Eq. (7)/(8): the brute-force oracle gives the hand-worked (config, B,
    instances, cost) per function, including the lower-config tie-break (golden P3)."""
    from oracle.autoscale import autoscale
    g, prob, exp = _autoscale_golden()
    out = autoscale(prob, g["slope_us"], g["intercept_us"], g["invocations"], g["it_us"], g["target_us"])
    assert [tuple(o) for o in out] == exp


def test_autoscale_library_matches_hand_worked_golden():
    """The library's host-side bisection (smiless_autoscale) on the same golden."""
    from paper_conf_sc_luxl0y024_b200 import smiless as S
    g, prob, exp = _autoscale_golden()
    n = prob.n_funcs
    pl = S.Planner(device=0)
    pl.load_dag(*W.csr_from_preds([[]] * n))
    ncfg = np.asarray(g["n_configs"], np.int32)
    z = np.zeros(int(ncfg.sum()), np.int32)
    pl.load_profiles(ncfg, z + 1, z, prob.price_per_us)
    out = pl.autoscale(g["slope_us"], g["intercept_us"], g["invocations"], g["it_us"], g["target_us"])
    assert [(int(o[0]), int(o[1]), int(o[2]), float(o[3])) for o in out] == exp


def test_cost_is_left_to_right_without_fma_for_paper_prices():
    """G15 / Eq. (3)-(4) with the paper's non-dyadic prices (golden P4): the oracle's cost
    bits are the left-to-right correctly rounded sum, which differs from the FMA-contracted
    one, so an oracle (or kernel) that fuses a product into the sum fails here."""
    g = _golden("P4_cost_no_fma.json")
    p = _problem_from(g)
    c, l, f = OracleProblem(p).evaluate([0])
    assert c[0].hex() == g["expected_cost_hex"]
    assert g["expected_cost_hex"] != g["fma_contracted_cost_hex"]
    assert g["expected_cost_hex"] != g["right_to_left_cost_hex"]
    # the same numbers by exact rational arithmetic, rounding after every operation
    E = [t + i for t, i in zip(g["init_us"], g["exec_us"])]
    U = [Fraction(float.fromhex(h)) for h in g["price_per_us_hex"]]
    rnd = lambda q: float(q)  # noqa: E731  (correctly rounded)
    lr = rnd(U[0] * E[0])
    for k in (1, 2):
        lr = rnd(Fraction(lr) + Fraction(rnd(U[k] * E[k])))
    fused = rnd(U[0] * E[0])
    for k in (1, 2):
        fused = rnd(Fraction(fused) + U[k] * E[k])
    assert lr.hex() == g["expected_cost_hex"] and fused.hex() == g["fma_contracted_cost_hex"]
    rl = rnd(U[2] * E[2])
    for k in (1, 0):
        rl = rnd(Fraction(rl) + Fraction(rnd(U[k] * E[k])))
    assert rl.hex() == g["right_to_left_cost_hex"]


# ---------------------------------------------------------------------------
# NEXT-4 scale-out inside model M (reading G26: n_k round-robin instances)
# ---------------------------------------------------------------------------

def test_scale_out_worked_example():
    """Golden S_E7: one function on 1, 2, 3 instances under a Case III burst,
    and 2 instances with pre-warm windows (covered and partly covered)."""
    g = _golden("S_E7_scale_out.json")
    for case in g["cases"]:
        p = mk([[]], case["exec_us"], case["init_us"], case["arrivals_us"], case["windows_us"])
        billed, lat = OracleProblem(p, instances=case["instances"]).simulate([0], case["window_idx"])
        assert billed.tolist() == case["billed"], case
        assert lat.tolist() == case["latency"], case
        b2, l2 = des.simulate(p, [0], case["window_idx"], instances=case["instances"])
        assert b2 == case["billed"] and l2 == case["latency"]


def test_scale_out_oracle_matches_event_driven_simulator():
    """Random DAGs with 1-4 instances per function: the oracle's case split on
    D[k][j - n_k] equals the DES running n_k explicit instance state machines."""
    rng = np.random.default_rng(23)
    for _ in range(1500):
        n = int(rng.integers(1, 7))
        p = W.random_problem(rng, n, 3, int(rng.integers(1, 5)), int(rng.integers(1, 16)))
        inst = [int(rng.integers(1, 5)) for _ in range(n)]
        o = OracleProblem(p, instances=inst)
        c = [int(rng.integers(0, p.n_configs[k])) for k in range(n)]
        w = [int(rng.integers(0, len(p.windows_us))) for k in range(n)]
        billed, lat = o.simulate(c, w)
        b2, l2 = des.simulate(p, c, w, instances=inst)
        assert billed.tolist() == b2
        assert lat.tolist() == l2


def test_scale_out_keepalive_is_fcfs_multiserver_queue():
    """Textbook G/D/c: with keep-alive, deterministic service I and sorted arrivals, n
    round-robin instances serve each request exactly when the FCFS c-server queue does
    (the request starts at max(arrival, earliest server release); a heap of release
    times), so the completion times (latency) agree."""
    import heapq
    rng = np.random.default_rng(29)
    for _ in range(400):
        c = int(rng.integers(1, 6))
        J = int(rng.integers(1, 60))
        I = int(rng.integers(1, 500))
        arr = np.cumsum(rng.integers(0, 300, size=J)).astype(np.int64)
        p = mk([[]], [I], [int(rng.integers(0, 200))], arr, [0])
        billed, lat = OracleProblem(p, instances=[c]).simulate([0], [0])
        free = [int(arr[0])] * c                        # every server ready at the first arrival (G5)
        heapq.heapify(free)
        want = []
        for a in arr:
            s = max(int(a), heapq.heappop(free))
            heapq.heappush(free, s + I)
            want.append(s + I - int(a))
        assert lat.tolist() == want


def test_scale_out_periodic_closed_forms():
    """Periodic arrivals (period IT) with keep-alive on n instances, I <= n IT (no
    queueing: L = sum of I): every request's latency is the chain's sum of I, and
    each instance bills T + I + (its last - its first request) IT; with n >= J every
    request is an instance's first: billed = J (T + I)."""
    rng = np.random.default_rng(31)
    for _ in range(200):
        K = int(rng.integers(1, 4))
        J = int(rng.integers(1, 40))
        n = int(rng.integers(1, 6))
        IT = int(rng.integers(100, 1000))
        I = [int(rng.integers(1, n * IT // K + 1)) for _ in range(K)]
        T = [int(rng.integers(0, 500)) for _ in range(K)]
        p = mk([[]] + [[k] for k in range(K - 1)], I, T, [j * IT for j in range(J)], [0])
        billed, lat = OracleProblem(p, instances=[n] * K).simulate([0] * K, [0] * K)
        assert lat.tolist() == [sum(I)] * J
        for k in range(K):
            want = sum(T[k] + I[k] + ((J - 1 - i) // n * n) * IT for i in range(min(n, J)))
            assert billed[k] == want
        big = OracleProblem(p, instances=[J] * K).simulate([0] * K, [0] * K)[0]
        assert big.tolist() == [J * (T[k] + I[k]) for k in range(K)]


def test_scale_out_one_instance_is_model_m():
    """instances = [1] * N is exactly the single-instance model (every existing pin)."""
    rng = np.random.default_rng(37)
    for _ in range(300):
        n = int(rng.integers(1, 6))
        p = W.random_problem(rng, n, 3, int(rng.integers(1, 4)), int(rng.integers(1, 30)))
        o1, o2 = OracleProblem(p), OracleProblem(p, instances=[1] * n)
        idx = np.arange(min(p.space_size(), 64), dtype=np.uint64)
        a, b = o1.evaluate(idx), o2.evaluate(idx)
        assert all(np.array_equal(x.view(np.uint8), y.view(np.uint8)) for x, y in zip(a, b))


@pytest.mark.parametrize("name", ["C3", "C5"])
def test_workload_instances_are_the_autoscalers(name):
    """The scale-out instance counts of C3 / C5 (workloads.SCALE_OUT_INSTANCES, inputs of
    model M) are the paper's auto-scaler constraint (Eq. (7)/(8)) at each
    function's fastest configuration for the predicted peak G per 1-s window with
    IT = I_s = 1 s: the oracle's brute force and the library's bisection both give them."""
    from oracle.autoscale import autoscale_rows
    from paper_conf_sc_luxl0y024_b200 import smiless as S
    p = W.make_config(name)
    G = W.peak_window_count(p.arrivals_us)
    n = p.n_funcs
    b_o, n_o = autoscale_rows(p, p.batch_slope_us, p.batch_intercept_us, [G] * n, [10**6] * n)
    pl = S.planner_for(p)
    b_l, n_l = pl.autoscale_rows(p.batch_slope_us, p.batch_intercept_us, [G] * n, [10**6] * n)
    assert list(b_l) == b_o and list(n_l) == n_o
    off = np.concatenate([[0], np.cumsum(p.n_configs)])
    fastest = [off[k] + int(np.argmin(p.exec_us[off[k]:off[k + 1]])) for k in range(n)]
    assert [n_o[r] for r in fastest] == list(W.SCALE_OUT_INSTANCES[name]) == list(p.instances)


def test_decompose_model_m_on_diamond():
    """Golden P2m (P:214-218 with exhaustive per-path optima under model M): the paths, each
    path's optimum and latency, the F_s/F_e rule and the branch re-choice that moves F2 to
    its cheaper configuration, and the combined plan's latency and cost."""
    from oracle.decompose_m import decompose_plan
    g = _golden("P2m_decompose_model_m.json")
    p = mk(g["preds"], g["exec_us"], g["init_us"], g["arrivals_us"], g["windows_us"], sla=g["sla_us"],
           prices=g["price_per_us"], n_configs=g["n_configs"])
    tr = {}
    cfg, win, cost, lat, ok, n_paths = decompose_plan(p, OracleProblem, trace=tr)
    assert tr["paths"] == g["expected_paths"] and n_paths == 2
    assert tr["path_configs"] == g["expected_path_configs"] and tr["path_latency"] == g["expected_path_latency"]
    assert cfg == g["expected_configs"] and win == [0] * 4 and ok
    assert lat == g["expected_latency_us"] and cost == g["expected_cost"]
