"""Multi-GPU driver: shard the candidate space across ranks, one exchange at the end.

SURVEY 8(e): candidates are independent, so each rank (one process per GPU) plans the
chunks c with c % world == rank (interleaved for balance under pruning) through the
C ABI, then the ranks agree on the lexicographic (cost, index) minimum with two
8-byte MIN all-reduces over NCCL/NVLink (cost bits of a non-negative double order like
the double; then the index among ranks holding that cost).  No candidate data crosses
GPUs.  The same code runs on the gloo backend for the CPU tests.
"""
from __future__ import annotations

import struct
from typing import Optional

import numpy as np
import torch
import torch.distributed as dist

INF_BITS = (1 << 63) - 1          # "no feasible candidate" key (above every finite cost's bits)
NO_INDEX = (1 << 63) - 1


def cost_bits(cost: Optional[float]) -> int:
    if cost is None:
        return INF_BITS
    b = struct.unpack("<q", struct.pack("<d", float(cost)))[0]
    assert b >= 0, "costs are non-negative"
    return b


def bits_cost(bits: int) -> Optional[float]:
    if bits == INF_BITS:
        return None
    return struct.unpack("<d", struct.pack("<q", int(bits)))[0]


def reduce_best(local_cost: Optional[float], local_index: Optional[int], local_latency: int,
                n_decided: int, device, group=None):
    """All-reduce the per-rank winners to the global lexicographic (cost, index) minimum.

    Returns (cost or None, index or None, max_latency or -1, total decided)."""
    kb = cost_bits(local_cost)
    t = torch.tensor([kb], dtype=torch.int64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MIN, group=group)
    best_bits = int(t.item())
    mine = local_cost is not None and kb == best_bits
    v = torch.tensor([int(local_index) if mine else NO_INDEX], dtype=torch.int64, device=device)
    dist.all_reduce(v, op=dist.ReduceOp.MIN, group=group)
    best_index = int(v.item())
    # one SUM: the (unique) owner contributes the winner's latency; everyone its decided count
    s = torch.tensor([local_latency if (mine and local_index == best_index) else 0, int(n_decided)],
                     dtype=torch.int64, device=device)
    dist.all_reduce(s, op=dist.ReduceOp.SUM, group=group)
    lat, dec = (int(v) for v in s.tolist())
    if best_bits == INF_BITS:
        return None, None, -1, dec
    return bits_cost(best_bits), best_index, lat, dec


def union_index(pinned_digit: int, slice_size: int, index: Optional[int]) -> Optional[int]:
    """Index of a slice's candidate in the space with one digit fewer pinned: weak scaling gives
    every rank its own slice (the last pinned digit differs per rank), and the winner of the
    union is the lexicographic (cost, union index) minimum, the same tie-break as one plan over
    the union."""
    return None if index is None else int(pinned_digit) * int(slice_size) + int(index)


def plan_distributed(planner, arrivals, sla_us, windows_us, group=None, device=None, **kw):
    """Plan this rank's shard through the C ABI and reduce across ranks.

    Returns (cost, index, max_latency, config, window, n_decided, local PlanResult)."""
    rank = dist.get_rank(group)
    world = dist.get_world_size(group)
    if device is None:
        device = torch.device("cuda", torch.cuda.current_device()) if torch.cuda.is_available() else "cpu"
    r = planner.plan(arrivals, sla_us, windows_us, shard=rank, n_shards=world, **kw)
    cost, index, lat, decided = reduce_best(r.cost if r.feasible else None, r.index, r.max_latency_us,
                                            r.n_decided, device, group)
    if index is None:
        n = planner.n_funcs
        return None, None, -1, np.full(n, -1, np.int32), np.full(n, -1, np.int32), decided, r
    c, w = planner.decode(index, len(windows_us), kw.get("n_fixed", 0), kw.get("fixed_digits", ()))
    return cost, index, lat, c, w, decided, r


def reduce_lex(keys, payload, device, group=None):
    """Lexicographic MIN across ranks of an int64 key tuple (e.g. cost bits, pinned digit,
    suffix index) by successive MIN all-reduces, each over the ranks still tied; `payload`
    (int64s) comes from the unique owner of the minimum.  Returns (keys, payload)."""
    BIG = (1 << 63) - 1
    tied = True
    out = []
    for k in keys:
        t = torch.tensor([int(k) if tied else BIG], dtype=torch.int64, device=device)
        dist.all_reduce(t, op=dist.ReduceOp.MIN, group=group)
        v = int(t.item())
        tied = tied and int(k) == v
        out.append(v)
    s = torch.tensor([int(x) if tied else 0 for x in payload], dtype=torch.int64, device=device)
    dist.all_reduce(s, op=dist.ReduceOp.SUM, group=group)
    return out, [int(x) for x in s.tolist()]


def plan_pinned_rounds(plan_digit, digits, rank, world, device, group=None, initial_cap=None):
    """Plan sub-spaces (one per value of a pinned leading digit) round-robin over the ranks:
    round r gives digit r*world + rank to this rank.  After every round the ranks MIN-all-
    reduce their cheapest feasible cost (8 bytes) and the next sub-plan gets it as its cost
    cap, so every rank's cost bound prunes against the global incumbent.  A cap is always a
    real feasible candidate's cost, i.e. >= OPT, so each sub-plan still returns its own best
    candidate among those costing <= the cap, and the global (cost, digit, index) minimum is
    OPT with the lowest-index tie-break.

    plan_digit(d, cap) -> result with .feasible, .cost, .index, .max_latency_us, .n_decided,
    .n_full_evals (cap None = no cap).  Returns (best, decided, full_evals, caps) where best
    = (cost, digit, index, max_latency) of this rank or None and caps = the caps it passed.
    initial_cap: the cost of a feasible candidate known beforehand (the same on every rank),
    or None; it caps the first round too."""
    best, decided, full_evals, caps = None, 0, 0, []
    cap_bits = cost_bits(initial_cap) if initial_cap is not None else INF_BITS
    n_rounds = (len(digits) + world - 1) // world
    for rnd in range(n_rounds):
        i = rnd * world + rank
        if i < len(digits):
            d0 = digits[i]
            cap = bits_cost(cap_bits) if cap_bits != INF_BITS else None
            caps.append(cap)
            r = plan_digit(d0, cap)
            decided += r.n_decided
            full_evals += r.n_full_evals
            if r.feasible and (best is None or (r.cost, d0, r.index) < best[:3]):
                best = (r.cost, d0, r.index, r.max_latency_us)
        if best is not None:
            cap_bits = min(cap_bits, cost_bits(best[0]))
        if world > 1 and rnd + 1 < n_rounds:
            t = torch.tensor([cap_bits], dtype=torch.int64, device=device)
            dist.all_reduce(t, op=dist.ReduceOp.MIN, group=group)
            cap_bits = int(t.item())
    return best, decided, full_evals, caps


def plan_range_rounds(plan_range, space, rounds, rank, world, device, group=None, initial_cap=None):
    """One exact plan of [0, space) split into `rounds` contiguous index ranges, each planned
    by every rank on its interleaved shard (plan_range(begin, end, cap) calls smiless_plan with
    shard=rank, n_shards=world).  After every round the ranks MIN-all-reduce their cheapest
    feasible cost bits and the next round gets it as its cost cap, so each GPU's cost bound
    prunes against the global incumbent inside the plan (SURVEY 8(e) collective (1)).  A cap
    is always a real feasible candidate's cost, i.e. >= OPT, so every round still returns its
    best candidate among those costing <= the cap, and the lexicographic (cost, index) minimum
    over rounds and ranks is OPT with the lowest-index tie-break.

    Returns (best, decided, full_evals, caps): best = (cost, index, max_latency) of this rank
    or None; caps = the caps this rank passed (None = no cap)."""
    best, decided, full_evals, caps = None, 0, 0, []
    cap_bits = cost_bits(initial_cap) if initial_cap is not None else INF_BITS
    rounds = max(1, min(int(rounds), int(space)))
    for rnd in range(rounds):
        b0 = space * rnd // rounds
        b1 = space * (rnd + 1) // rounds
        cap = bits_cost(cap_bits) if cap_bits != INF_BITS else None
        caps.append(cap)
        r = plan_range(b0, b1, cap)
        decided += r.n_decided
        full_evals += r.n_full_evals
        if r.feasible and (best is None or (r.cost, r.index) < best[:2]):
            best = (r.cost, r.index, r.max_latency_us)
        if best is not None:
            cap_bits = min(cap_bits, cost_bits(best[0]))
        if world > 1 and rnd + 1 < rounds:
            t = torch.tensor([cap_bits], dtype=torch.int64, device=device)
            dist.all_reduce(t, op=dist.ReduceOp.MIN, group=group)
            cap_bits = int(t.item())
    return best, decided, full_evals, caps


def plan_digits_sharded(plan_digit, digits, rank, world, device, group=None, initial_cap=None):
    """Sub-spaces (one per value of a pinned leading digit, e.g. C5's 2^70 = 128 x 2^63) planned
    one after the other by EVERY rank on its interleaved shard (plan_digit(d, cap) calls
    smiless_plan with shard=rank, n_shards=world), so a heavy digit is split across the GPUs
    like any single plan.  After every digit the ranks MIN-all-reduce
    their cheapest feasible cost and pass it as the next digit's cost cap (exact for any cap
    >= OPT, see plan_range_rounds).

    Returns (best, decided, full_evals, caps) like plan_pinned_rounds: best = (cost, digit,
    index, max_latency) of this rank or None."""
    best, decided, full_evals, caps = None, 0, 0, []
    cap_bits = cost_bits(initial_cap) if initial_cap is not None else INF_BITS
    for i, d0 in enumerate(digits):
        cap = bits_cost(cap_bits) if cap_bits != INF_BITS else None
        caps.append(cap)
        r = plan_digit(d0, cap)
        decided += r.n_decided
        full_evals += r.n_full_evals
        if r.feasible and (best is None or (r.cost, d0, r.index) < best[:3]):
            best = (r.cost, d0, r.index, r.max_latency_us)
        if best is not None:
            cap_bits = min(cap_bits, cost_bits(best[0]))
        if world > 1 and i + 1 < len(digits):
            t = torch.tensor([cap_bits], dtype=torch.int64, device=device)
            dist.all_reduce(t, op=dist.ReduceOp.MIN, group=group)
            cap_bits = int(t.item())
    return best, decided, full_evals, caps


def plan_digit_blocks_sharded(plan_block, d_begin, d_end, block, rank, world, device, group=None, initial_cap=None):
    """plan_digits_sharded with blocks of consecutive digits per library call:
    plan_block(d_lo, d_hi, cap) plans digits d_lo .. d_hi - 1 on this rank's interleaved shard in
    one smiless_plan_digits call (the incumbent carried on the device inside the block) and
    returns a result with .digit; the ranks MIN-all-reduce their cheapest feasible cost after
    every block.  One GPU: one block of all digits, no host round trip per digit.

    Returns (best, decided, full_evals, caps) like plan_digits_sharded."""
    best, decided, full_evals, caps = None, 0, 0, []
    cap_bits = cost_bits(initial_cap) if initial_cap is not None else INF_BITS
    for lo in range(d_begin, d_end, block):
        hi = min(d_end, lo + block)
        cap = bits_cost(cap_bits) if cap_bits != INF_BITS else None
        caps.append(cap)
        r = plan_block(lo, hi, cap)
        decided += r.n_decided
        full_evals += r.n_full_evals
        if r.feasible and (best is None or (r.cost, r.digit, r.index) < best[:3]):
            best = (r.cost, r.digit, r.index, r.max_latency_us)
        if best is not None:
            cap_bits = min(cap_bits, cost_bits(best[0]))
        if world > 1 and hi < d_end:
            t = torch.tensor([cap_bits], dtype=torch.int64, device=device)
            dist.all_reduce(t, op=dist.ReduceOp.MIN, group=group)
            cap_bits = int(t.item())
    return best, decided, full_evals, caps


def decompose_plan_distributed(planner, arrivals, sla_us, windows_us, group=None, device=None, **kw):
    """NEXT-3 with model M on N GPUs: every rank plans its interleaved share of each source-to-
    sink path (smiless_decompose_plan_sharded) and the path winners are reduced with the same
    two MIN all-reduces as a plan (reduce_best), inside the library's callback.  Every rank
    returns the same combined plan: (PlanResult, number of paths)."""
    rank = dist.get_rank(group)
    world = dist.get_world_size(group)
    if device is None:
        device = torch.device("cuda", torch.cuda.current_device()) if torch.cuda.is_available() else "cpu"

    def reduce(path, res):
        feasible = res.index != (1 << 64) - 1
        cost, index, lat, _ = reduce_best(res.cost if feasible else None, res.index if feasible else None,
                                          res.max_latency_us, res.n_decided, device, group)
        if index is None:
            res.index, res.cost, res.max_latency_us = (1 << 64) - 1, float("inf"), -1
        else:
            res.index, res.cost, res.max_latency_us = index, cost, lat

    return planner.decompose_plan(arrivals, sla_us, windows_us, reduce=reduce, shard=rank, n_shards=world, **kw)
