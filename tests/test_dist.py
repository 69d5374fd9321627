"""Multi-process (gloo, CPU) tests of the cross-rank exchange of paper_conf_sc_luxl0y024_b200.dist.

The only collective of the path is the lexicographic (cost, index) MIN of
the per-rank winners.  On CPU we check it with world sizes 2 and 3: ties go to the lowest
index on any rank, infeasible ranks never win, all-infeasible stays infeasible, and the
decided counts sum.  The end-to-end check shards a small problem's candidate space the
way the kernel does (interleaved chunks of units) and compares the reduced winner with
the oracle's plan of the whole space.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_sc_luxl0y024_b200.dist import reduce_best, cost_bits, bits_cost, INF_BITS


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, cases, out_q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    res = []
    for case in cases:
        cost, idx, lat, dec = case[rank]
        res.append(reduce_best(cost, idx, lat, dec, "cpu"))
    out_q.put((rank, res))
    dist.barrier()
    dist.destroy_process_group()


def run_world(world, cases):
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, cases, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = dict(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    return out


def test_cost_bits_order_like_doubles():
    vals = [0.0, 1e-300, 0.5, 1.0, 3.25, 1e10, 8.3e1]
    bits = [cost_bits(v) for v in vals]
    assert sorted(range(len(vals)), key=lambda i: vals[i]) == sorted(range(len(vals)), key=lambda i: bits[i])
    assert all(bits_cost(b) == v for b, v in zip(bits, vals))
    assert cost_bits(None) == INF_BITS and bits_cost(INF_BITS) is None


@pytest.mark.parametrize("world", [2, 3])
def test_reduce_best_gloo(world):
    cases = [
        # (cost, index, latency, decided) per rank
        [(5.0, 10, 100, 7), (3.0, 20, 200, 5), (4.0, 1, 300, 1)][:world],
        [(3.0, 25, 100, 1), (3.0, 20, 200, 1), (3.0, 21, 300, 1)][:world],       # tie -> lowest index
        [(None, None, -1, 4), (2.0, 99, 50, 4), (None, None, -1, 4)][:world],     # infeasible ranks
        [(None, None, -1, 3), (None, None, -1, 3), (None, None, -1, 3)][:world],  # all infeasible
    ]
    out = run_world(world, cases)
    exp = [
        (3.0, 20, 200, sum([7, 5, 1][:world])),
        (3.0, 20, 200, world),
        (2.0, 99, 50, 4 * world),
        (None, None, -1, 3 * world),
    ]
    for r in range(world):
        assert out[r] == exp, (r, out[r])


def _shard_candidates(space, V, world, rank, chunk_units=256):
    """Candidates the kernel assigns to `rank`: units of V candidates, chunks of
    chunk_units units, chunk c belongs to rank c % world (csrc/evaluator.cuh)."""
    n_units = (space + V - 1) // V
    idx = []
    for u in range(n_units):
        if (u // chunk_units) % world == rank:
            idx.extend(range(u * V, min(space, u * V + V)))
    return np.asarray(idx, dtype=np.uint64)


def _plan_worker(rank, world, port, out_q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import workloads as W
    from oracle import OracleProblem
    p = W.make_config("C1", n_arrivals=40)
    o = OracleProblem(p)
    cand = _shard_candidates(o.space_size(), 4 * len(p.windows_us), world, rank, chunk_units=8)
    c, l, f = o.evaluate(cand)
    best = None
    for i in np.nonzero(f)[0]:
        if best is None or (c[i], int(cand[i])) < best[:2]:
            best = (c[i], int(cand[i]), int(l[i]))
    r = reduce_best(best[0] if best else None, best[1] if best else None, best[2] if best else -1,
                    len(cand), "cpu")
    out_q.put((rank, r))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_sharded_plan_reduces_to_global_opt(world):
    import workloads as W
    from oracle import OracleProblem
    p = W.make_config("C1", n_arrivals=40)
    ref = OracleProblem(p).plan()
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_plan_worker, args=(r, world, port, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    out = dict(q.get(timeout=180) for _ in range(world))
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    for r in range(world):
        cost, idx, lat, dec = out[r]
        assert (idx, cost, lat) == ref and dec == 4096


class _Res:
    def __init__(self, feasible, cost, index, lat, n):
        self.feasible, self.cost, self.index, self.max_latency_us = feasible, cost, index, lat
        self.n_decided, self.n_full_evals = n, n


def _pinned_worker(rank, world, port, zero_prices, out_q, seed=None):
    """C1 as 16 sub-spaces of function 0's digit (256 candidates each), planned round-robin
    with the global incumbent as cost cap; a sub-plan is emulated with the library's
    semantics (lowest (cost, index) among feasible candidates costing <= cap) on the oracle's
    per-candidate costs."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import workloads as W
    from oracle import OracleProblem
    from paper_conf_sc_luxl0y024_b200.dist import plan_pinned_rounds, reduce_lex
    p = W.make_config("C1", n_arrivals=40)
    if zero_prices:
        p = p.replace(price_per_us=np.zeros_like(p.price_per_us))
    c, l, f = OracleProblem(p).evaluate(np.arange(4096, dtype=np.uint64))

    def plan_digit(d, cap):
        s = np.arange(256)
        g = d * 256 + s
        ok = f[g] & (c[g] <= (np.inf if cap is None else cap))
        if not ok.any():
            return _Res(False, float("inf"), None, -1, 256)
        k = s[ok][np.lexsort((s[ok], c[g][ok]))[0]]
        return _Res(True, float(c[d * 256 + k]), int(k), int(l[d * 256 + k]), 256)

    init = None
    if seed == "opt":                     # a cap equal to OPT: candidates costing exactly the cap stay eligible
        init = float(c[f].min())
    elif seed == "max":                   # the loosest real cap: the most expensive feasible candidate
        init = float(c[f].max())
    best, dec, _, caps = plan_pinned_rounds(plan_digit, list(range(16)), rank, world, "cpu", initial_cap=init)
    keys = [cost_bits(best[0]) if best else INF_BITS, best[1] if best else 0, best[2] if best else 0]
    keys, pay = reduce_lex(keys, [best[3] if best else -1], "cpu")
    out_q.put((rank, (keys, pay, dec, caps)))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,zero_prices,seed", [(2, False, None), (3, False, None), (2, True, None),
                                                     (2, False, "opt"), (3, False, "max"), (2, True, "opt")])
def test_pinned_rounds_with_global_cost_cap(world, zero_prices, seed):
    """bench.py's C5 driver (dist.plan_pinned_rounds): the caps exchanged between rounds are
    real feasible costs (>= OPT), so the reduced (cost, digit, index) equals the oracle's
    global OPT, ties included (zero prices: every candidate costs 0, lowest index wins)."""
    import workloads as W
    from oracle import OracleProblem
    p = W.make_config("C1", n_arrivals=40)
    if zero_prices:
        p = p.replace(price_per_us=np.zeros_like(p.price_per_us))
    ref_idx, ref_cost, ref_lat = OracleProblem(p).plan()
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_pinned_worker, args=(r, world, port, zero_prices, q, seed)) for r in range(world)]
    for pr in procs:
        pr.start()
    out = dict(q.get(timeout=180) for _ in range(world))
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    n_caps = 0
    for r in range(world):
        keys, pay, dec, caps = out[r]
        assert bits_cost(keys[0]) == ref_cost and keys[1] * 256 + keys[2] == ref_idx and pay[0] == ref_lat
        assert all(cp is None or cp >= ref_cost for cp in caps)
        n_caps += sum(cp is not None for cp in caps)
    assert n_caps > 0                     # later rounds did run under a cap


def _range_rounds_worker(rank, world, port, rounds, zero_prices, out_q):
    """One exact plan of C1's 4096 candidates split into `rounds` index ranges; in each round
    every rank plans its interleaved shard (emulated with the library's semantics on the
    oracle's per-candidate costs: lowest (cost, index) among the shard's feasible candidates
    costing <= cap) and the ranks exchange the incumbent before the next round."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import workloads as W
    from oracle import OracleProblem
    from paper_conf_sc_luxl0y024_b200.dist import plan_range_rounds, reduce_lex
    p = W.make_config("C1", n_arrivals=40)
    if zero_prices:
        p = p.replace(price_per_us=np.zeros_like(p.price_per_us))
    c, l, f = OracleProblem(p).evaluate(np.arange(4096, dtype=np.uint64))

    def plan_range(b0, b1, cap):
        g = np.arange(b0, b1)
        g = g[g % world == rank]                       # this rank's interleaved share
        ok = f[g] & (c[g] <= (np.inf if cap is None else cap))
        if not ok.any():
            return _Res(False, float("inf"), None, -1, len(g))
        k = g[ok][np.lexsort((g[ok], c[g][ok]))[0]]
        return _Res(True, float(c[k]), int(k), int(l[k]), len(g))

    best, dec, _, caps = plan_range_rounds(plan_range, 4096, rounds, rank, world, "cpu")
    keys = [cost_bits(best[0]) if best else INF_BITS, best[1] if best else 0]
    keys, pay = reduce_lex(keys, [best[2] if best else -1, dec], "cpu")
    out_q.put((rank, (keys, pay, dec, caps)))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,rounds,zero_prices", [(2, 4, False), (3, 3, False), (2, 5, True), (3, 1, False)])
def test_range_rounds_with_in_plan_incumbent_exchange(world, rounds, zero_prices):
    """dist.plan_range_rounds (the exact full-space plans of C2/C3 on N GPUs): every rank
    decides its share of every round, the caps passed are real feasible costs (>= OPT), and
    the reduced (cost, index) is the oracle's OPT with the lowest-index tie-break."""
    import workloads as W
    from oracle import OracleProblem
    p = W.make_config("C1", n_arrivals=40)
    if zero_prices:
        p = p.replace(price_per_us=np.zeros_like(p.price_per_us))
    ref_idx, ref_cost, ref_lat = OracleProblem(p).plan()
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_range_rounds_worker, args=(r, world, port, rounds, zero_prices, q))
             for r in range(world)]
    for pr in procs:
        pr.start()
    out = dict(q.get(timeout=180) for _ in range(world))
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    total = sum(out[r][2] for r in range(world))
    assert total == 4096
    for r in range(world):
        keys, pay, dec, caps = out[r]
        assert dec >= 4096 // (2 * world)
        assert bits_cost(keys[0]) == ref_cost and keys[1] == ref_idx and pay[0] == ref_lat
        assert len(caps) == rounds and all(cp is None or cp >= ref_cost for cp in caps)
        if rounds > 1:
            assert caps[-1] is not None       # the global incumbent reached every rank's last round


def _digits_sharded_worker(rank, world, port, zero_prices, out_q, block=0):
    """C1 as 16 function-0 digits, EVERY rank planning every digit on its interleaved shard
    (emulated on the oracle's per-candidate costs with the library's semantics), the
    incumbent exchanged after each digit."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import workloads as W
    from oracle import OracleProblem
    from paper_conf_sc_luxl0y024_b200.dist import plan_digits_sharded, plan_digit_blocks_sharded, reduce_lex
    p = W.make_config("C1", n_arrivals=40)
    if zero_prices:
        p = p.replace(price_per_us=np.zeros_like(p.price_per_us))
    c, l, f = OracleProblem(p).evaluate(np.arange(4096, dtype=np.uint64))

    def plan_digit(d, cap):
        s_ = np.arange(256)
        s_ = s_[s_ % world == rank]                     # this rank's share of the digit
        g = d * 256 + s_
        ok = f[g] & (c[g] <= (np.inf if cap is None else cap))
        if not ok.any():
            return _Res(False, float("inf"), None, -1, len(s_))
        k = s_[ok][np.lexsort((s_[ok], c[g][ok]))[0]]
        return _Res(True, float(c[d * 256 + k]), int(k), int(l[d * 256 + k]), len(s_))

    def plan_block(lo, hi, cap):          # smiless_plan_digits: the (cost, digit, index) minimum of the block
        rs = [(plan_digit(d, cap), d) for d in range(lo, hi)]
        ok = [(r.cost, d, r.index, r) for r, d in rs if r.feasible]
        n = sum(r.n_decided for r, _ in rs)
        if not ok:
            out = _Res(False, float("inf"), None, -1, n)
            out.digit = None
            return out
        c_, d_, i_, r_ = min(ok, key=lambda t: t[:3])
        out = _Res(True, c_, i_, r_.max_latency_us, n)
        out.digit = d_
        return out

    if block:
        best, dec, _, caps = plan_digit_blocks_sharded(plan_block, 0, 16, block, rank, world, "cpu")
    else:
        best, dec, _, caps = plan_digits_sharded(plan_digit, list(range(16)), rank, world, "cpu")
    keys = [cost_bits(best[0]) if best else INF_BITS, best[1] if best else 0, best[2] if best else 0]
    keys, pay = reduce_lex(keys, [best[3] if best else -1], "cpu")
    out_q.put((rank, (keys, pay, dec, caps)))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,zero_prices,block", [(2, False, 0), (3, False, 0), (2, True, 0), (2, False, 4),
                                                     (3, False, 5), (2, True, 4)])
def test_digits_sharded_with_global_cost_cap(world, zero_prices, block):
    """bench.py's C5 driver (dist.plan_digits_sharded, or with block > 0
    dist.plan_digit_blocks_sharded: several digits per library call, exchange per block): every
    rank decides its share of every digit, the caps are real feasible costs, and the reduced
    (cost, digit, index) is the oracle's OPT with the lowest-index tie-break."""
    import workloads as W
    from oracle import OracleProblem
    p = W.make_config("C1", n_arrivals=40)
    if zero_prices:
        p = p.replace(price_per_us=np.zeros_like(p.price_per_us))
    ref_idx, ref_cost, ref_lat = OracleProblem(p).plan()
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_digits_sharded_worker, args=(r, world, port, zero_prices, q, block))
             for r in range(world)]
    for pr in procs:
        pr.start()
    out = dict(q.get(timeout=180) for _ in range(world))
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    assert sum(out[r][2] for r in range(world)) == 4096
    for r in range(world):
        keys, pay, dec, caps = out[r]
        assert dec >= 4096 // (2 * world)
        assert bits_cost(keys[0]) == ref_cost and keys[1] * 256 + keys[2] == ref_idx and pay[0] == ref_lat
        assert all(cp is None or cp >= ref_cost for cp in caps)


def _weak_worker(rank, world, port, zero_prices, out_q):
    """Weak scaling as bench.py runs it: rank r plans its own slice of C1 (function 0 pinned to
    digit 5, function 1 to digit 15 - r); the winners are reduced with their indices in the
    function-0-pinned space (dist.union_index)."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import workloads as W
    from oracle import OracleProblem
    from paper_conf_sc_luxl0y024_b200.dist import union_index
    p = W.make_config("C1", n_arrivals=40)
    if zero_prices:                       # every feasible candidate ties: the lowest union index wins
        p = p.replace(price_per_us=np.zeros_like(p.price_per_us))
    o = OracleProblem(p, n_fixed=2, fixed_digits=[5, 15 - rank])
    ref = o.plan()
    gi = union_index(15 - rank, o.space_size(), ref[0] if ref else None)
    r = reduce_best(ref[1] if ref else None, gi, ref[2] if ref else -1, o.space_size(), "cpu")
    out_q.put((rank, r))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,zero_prices", [(2, False), (3, False), (3, True)])
def test_weak_scaling_union_of_slices(world, zero_prices):
    """The bench's weak-scaled step: the reduced winner of the per-rank slices equals one oracle
    plan over the union of the slices (function 0 pinned, function 1 on the ranks' digits),
    with the lowest-index tie-break, and the decided counts sum to the union's size."""
    import workloads as W
    from oracle import OracleProblem
    p = W.make_config("C1", n_arrivals=40)
    if zero_prices:
        p = p.replace(price_per_us=np.zeros_like(p.price_per_us))
    o1 = OracleProblem(p, n_fixed=1, fixed_digits=[5])
    S = OracleProblem(p, n_fixed=2, fixed_digits=[5, 15]).space_size()
    best = None
    for r in range(world):                # the union: function 1's digits 15, 14, ...
        d1 = 15 - r
        ref = o1.plan(begin=d1 * S, end=(d1 + 1) * S)
        if ref and (best is None or (ref[1], ref[0]) < (best[1], best[0])):
            best = ref
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_weak_worker, args=(r, world, port, zero_prices, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    out = dict(q.get(timeout=180) for _ in range(world))
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    for r in range(world):
        cost, idx, lat, dec = out[r]
        assert (idx, cost, lat) == (best if best else (None, None, -1))
        assert dec == world * S
