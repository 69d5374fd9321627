#!/usr/bin/env python
"""Time-to-optimal of one workload's whole space on cuda:0 (exact pruned plan), winner
re-checked on the oracle.  C5-like spaces above 2^63 run as one sub-plan per value of
function 0's digit with the running best cost as cap (the single-rank form of
dist.plan_pinned_rounds).

    python tools/tto_full.py C3 [--sla US] [--limit-digits K]
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("name")
    ap.add_argument("--sla", type=int, default=None)
    ap.add_argument("--limit-digits", type=int, default=0)
    ap.add_argument("--per-digit", action="store_true",
                    help="one smiless_plan call per function-0 digit (default: one smiless_plan_digits call)")
    args = ap.parse_args()
    import torch
    from paper_conf_sc_luxl0y024_b200 import smiless as S
    from oracle import OracleProblem
    p = W.make_config(args.name)
    if args.sla:
        p = p.replace(sla_us=args.sla)
    pl = S.planner_for(p)
    arr = torch.as_tensor(p.arrivals_us).cuda()
    Wn = len(p.windows_us)
    try:
        space = pl.space_size(Wn)
        pinned = False
    except S.SmilessError:
        pinned = True
    warm = dict(n_fixed=1, fixed_digits=[0]) if pinned else {}
    pl.plan(arr, p.sla_us, p.windows_us, end=1 << 16, **warm)          # NVRTC outside the timing
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    best, decided, full, launches = None, 0, 0, 0
    per_digit = []
    if pinned:
        digits = list(range(int(p.n_configs[0]) * Wn))
        if args.limit_digits:
            digits = digits[:args.limit_digits]
        if not args.per_digit:
            r = pl.plan_digits(arr, p.sla_us, p.windows_us, digits[0], digits[-1] + 1, n_fixed=1, fixed_digits=[0])
            decided, full, launches = r.n_decided, r.n_full_evals, r.launches
            if r.feasible:
                best = (r.cost, r.digit, r.index, r.max_latency_us)
            digits = []
        for d in digits:
            td = time.perf_counter()
            kw = dict(n_fixed=1, fixed_digits=[d])
            if best is not None:
                kw["cost_cap"] = best[0]
            r = pl.plan(arr, p.sla_us, p.windows_us, **kw)
            per_digit.append(round((time.perf_counter() - td) * 1e3, 3))
            print(f"digit {d}: {per_digit[-1]} ms, feasible {r.feasible}, decided {r.n_decided}, "
                  f"full {r.n_full_evals}, best {best[0] if best else None}", file=sys.stderr, flush=True)
            decided += r.n_decided
            full += r.n_full_evals
            launches += r.launches
            if r.feasible and (best is None or (r.cost, d, r.index) < best[:3]):
                best = (r.cost, d, r.index, r.max_latency_us)
    else:
        r = pl.plan(arr, p.sla_us, p.windows_us)
        decided, full, launches = r.n_decided, r.n_full_evals, r.launches
        if r.feasible:
            best = (r.cost, 0, r.index, r.max_latency_us)
    torch.cuda.synchronize()
    sec = time.perf_counter() - t0
    out = {"workload": args.name, "sla_us": p.sla_us, "instances": None if p.instances is None else p.instances.tolist(),
           "time_to_optimal_s": sec, "decided": decided, "full_evals": full, "launches": launches,
           "prune_ratio": full / max(1, decided)}
    if best is not None:
        kw = dict(n_fixed=1, fixed_digits=[best[1]]) if pinned else {}
        c, w = pl.decode(best[2], Wn, **kw)
        oc, ol, of = OracleProblem(p, **kw).evaluate([best[2]])
        out.update(cost=best[0], index=best[2], digit0=best[1] if pinned else None, max_latency_us=best[3],
                   config=c.tolist(), window=w.tolist(), windows_nonzero=int((w != 0).sum()),
                   oracle_check={"feasible": bool(of[0]), "cost_bits_equal": bool(oc[0] == best[0]),
                                 "latency_equal": int(ol[0]) == best[3]})
    if per_digit:
        srt = sorted(per_digit)
        out["per_digit_ms"] = {"max": srt[-1], "median": srt[len(srt) // 2], "sum": round(sum(srt), 2)}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
