#!/usr/bin/env python
"""bench.py -- candidate plans evaluated/s (and time-to-optimal) of the SMIless hot path on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload C2] [--impl ours|reference]
    python -m torch.distributed.run --nproc-per-node N --master-addr 127.0.0.1 bench.py --gpus N ...

Step (BASELINE.json metric, configs[1]): one smiless_plan call = the whole hot path
(arrival prep, NVRTC-specialised evaluator over every candidate, argmin, exact
re-evaluation of the winner) over the fixed 2^28-candidate slice of C2 (IPA-6 DAG,
16 configs x 8 windows, 10^4 Poisson arrivals; functions 0 and 1 pinned to
GPU-100% / keep-alive), in throughput mode (no pruning: every candidate walked through
all 10^4 arrivals).  Weak scaling (the candidate space partitions, so per-GPU work is
fixed): rank r plans its own 2^28-candidate slice, function 1 pinned to config 15 - r
(rank 0 = the single-GPU slice), and the ranks exchange the winner of the union with
NCCL MIN all-reduces (16 bytes; no data-path collective).  SMILESS_BENCH_SCALING=strong
splits the one rank-0 slice over the ranks instead.

`value` = candidates of all ranks' slices / max-over-ranks device time per step (inputs resident
in HBM: arrivals passed as a device tensor).  `e2e` = the same through the public API
with the arrivals in pinned host memory (H2D inside the timed region) and the result
read back to the host.  Only rank 0 at N=1 times the CPU oracle (cpu_baseline) on a
bounded sample; `--impl reference` times the oracle as the reference arm.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402

METRIC = "candidate plans evaluated/sec and time-to-optimal-plan at 1/2/4/8 B200"
UNIT = "candidates/s"
ISSUE_LANES_PER_CLK_PER_SM = 4 * 32      # 4 SMSPs x 1 warp-instruction/clk x 32 lanes


def workload(name: str = "C2", rank: int = 0):
    """(Problem, plan kwargs) of the timed step.  Shared with tests/test_gpu_parity.py.
    rank r > 0 (weak scaling): function 1 pinned to config 15 - r instead of 15."""
    if name == "C2":
        p = W.make_config("C2")
        Wn = len(p.windows_us)
        gpu100 = 15                        # CONFIG_GRIDS[16][15] = ("gpu", 1.0)
        if not 0 <= rank < 16:
            raise ValueError("weak-scaling slices exist for ranks 0..15")
        fixed = [gpu100 * Wn + 0, (gpu100 - rank) * Wn + 0]   # SR, IR on GPU configs, keep-alive
        return p, dict(n_fixed=2, fixed_digits=fixed)
    if name == "C1":
        return W.make_config("C1"), dict(n_fixed=0, fixed_digits=[])
    raise KeyError(name)


def configs_per_lane(p) -> int:
    """Mirror of host.cpp configs_per_lane (G): last-function configs carried per lane."""
    M = int(p.n_configs[-1])
    Wn = len(p.windows_us)
    want = int(os.environ.get("SMILESS_G", "0")) or max(1, 16 // Wn)   # grid windows (no row windows)
    G = 1
    for g in range(1, want + 1):
        if M % g == 0 and g * Wn <= 32:
            G = g
    return G


def algorithmic_ops_per_candidate(p, memo: bool = True, split: bool = True) -> float:
    """Integer ops per candidate over the whole horizon for the algorithm as implemented
    (DESIGN.md "Roofline").  Per invocation j >= 1:
      upstream, once per prefix (memo) or per lane-unit: 7 per function-step (g, u, delta,
        busy mask, masked update, +I, sum u), +1 per extra join input, +1 per upstream sink;
      per last-function config 3 shared ops (x + CN, CN += -I, o + CN);
      per window variant 7 (g, u, delta, mask, update, sum u, latency), 4 for keep-alive;
      with the split cost (default, memo path): 6 per window variant -- the sum of u is not
      carried through the walk; the few units holding a feasible candidate are re-walked
      with it, which this count leaves out (it only lowers `achieved`);
    divided by the candidates sharing each part (prefix: M_{N-1} x W, unit: G x W)."""
    n = p.n_funcs
    Wn = len(p.windows_us)
    G = configs_per_lane(p)
    joins = sum(max(0, len(p.preds(k)) - 1) for k in range(n))
    listed = set(int(v) for v in p.pred_idx)
    up_sinks = sum(1 for k in range(n - 1) if k not in listed)
    w0 = 1 if int(p.windows_us[0]) == 0 else 0
    upstream = 7 * (n - 1) + joins + up_sinks
    per_unit = G * (3 + 4 * w0 + (6 if (memo and split) else 7) * (Wn - w0))
    up_share = int(p.n_configs[-1]) * Wn if memo else G * Wn
    per_cand_step = upstream / up_share + per_unit / (G * Wn)
    return per_cand_step * (len(p.arrivals_us) - 1)


class ClockSampler:
    """nvidia-smi-equivalent clocks/throttle sampling (NVML) during the timed region."""

    REASONS = {
        0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
        0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
        0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting",
    }

    def __init__(self, device_index: int, period_s: float = 0.2):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = threading.Event()
        self._thr = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self._nv = pynvml
            self._h = pynvml.nvmlDeviceGetHandleByIndex(device_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self._h, pynvml.NVML_CLOCK_SM)
        except Exception as e:  # pragma: no cover
            self._nv = None
            self.error = str(e)
        self.period = period_s

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self._nv.nvmlDeviceGetClockInfo(self._h, self._nv.NVML_CLOCK_SM))
                r = self._nv.nvmlDeviceGetCurrentClocksEventReasons(self._h)
                for bit, name in self.REASONS.items():
                    if r & bit and bit != 0x1:
                        self.reasons.add(name)
            except Exception:
                pass
            self._stop.wait(self.period)

    def __enter__(self):
        if self._nv is not None:
            self._thr = threading.Thread(target=self._run, daemon=True)
            self._thr.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._thr:
            self._thr.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons),
                    "samples": 0}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


def full_space_opt(name, S, rank, world, dev, xdev, stream, local, barrier, sla=None):
    """Exact OPT of a whole BASELINE config space with pruning + multi-level B&B, sharded over
    the ranks (C2 / C3: interleaved prefix batches of one plan; C5, 2^70 candidates: the 128
    values of function 0's digit, each a 2^63-candidate plan, planned in blocks of digits per
    smiless_plan_digits call on every rank's interleaved shard), reduced lexicographically on
    (cost bits, digit, index) across ranks."""
    import torch
    import torch.distributed as dist
    from paper_conf_sc_luxl0y024_b200.dist import (cost_bits, bits_cost, reduce_lex, plan_pinned_rounds,
                                                   plan_range_rounds, plan_digits_sharded,
                                                   plan_digit_blocks_sharded, INF_BITS)
    rounds = int(os.environ.get("SMILESS_BENCH_ROUNDS", "1" if world == 1 else "2"))
    p = W.make_config(name)
    if sla is not None:
        p = p.replace(sla_us=int(sla))
    Wn = len(p.windows_us)
    pl = S.planner_for(p, device=local, stream=stream.cuda_stream)
    arr = torch.as_tensor(p.arrivals_us).to(dev)
    pinned = name in ("C5", "C5s")
    digits = list(range(int(p.n_configs[0]) * Wn)) if pinned else [None]
    warm = dict(n_fixed=1, fixed_digits=[0]) if pinned else {}
    seed = os.environ.get("SMILESS_SEED_CAP", "0") == "1"
    seed_w = p.windows_us[:1]                                            # window 0 only: configs-only sub-space
    pl.plan(arr, p.sla_us, p.windows_us, end=1 << 20, **warm)            # NVRTC compile outside the timing
    if seed:
        pl.plan(arr, p.sla_us, seed_w, end=1 << 16)
    barrier()
    a = torch.cuda.Event(enable_timing=True)
    b = torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    a.record(stream)
    cap0, seed_ms = None, None
    if seed:
        # Incumbent from the window-0 sub-space (every window fixed to grid value 0; a subset of the
        # full space, so its best feasible cost is >= OPT and a valid cost cap: the full plan stays exact)
        ts = time.perf_counter()
        rs = pl.plan(arr, p.sla_us, seed_w, shard=rank, n_shards=world)
        cb = torch.tensor([cost_bits(rs.cost) if rs.feasible else INF_BITS], dtype=torch.int64, device=xdev)
        if world > 1:
            dist.all_reduce(cb, op=dist.ReduceOp.MIN)
        cap0 = bits_cost(int(cb.item())) if int(cb.item()) != INF_BITS else None
        seed_ms = (time.perf_counter() - ts) * 1e3
    if pinned:
        # every rank plans every function-0 digit on its interleaved shard (a heavy digit is split
        # across the GPUs), a block of digits per smiless_plan_digits call (incumbent carried on
        # the device inside a block, exchanged across ranks after each block: one block on one
        # GPU, 16 digits with N > 1); SMILESS_BENCH_DIGITS=sharded plans one digit per call,
        # =rr deals whole digits round-robin (dist.plan_pinned_rounds)
        scheme = os.environ.get("SMILESS_BENCH_DIGITS", "blocks")
        if scheme == "blocks":
            block = int(os.environ.get("SMILESS_BENCH_DIGIT_BLOCK", "0")) or (len(digits) if world == 1 else 16)
            best, decided, full_evals, _ = plan_digit_blocks_sharded(
                lambda d_lo, d_hi, cap: pl.plan_digits(arr, p.sla_us, p.windows_us, d_lo, d_hi, n_fixed=1,
                                                       fixed_digits=[0], shard=rank, n_shards=world,
                                                       **({"cost_cap": cap} if cap is not None else {})),
                digits[0], digits[-1] + 1, block, rank, world, xdev, initial_cap=cap0)
        elif scheme == "rr":
            best, decided, full_evals, _ = plan_pinned_rounds(
                lambda d0, cap: pl.plan(arr, p.sla_us, p.windows_us, n_fixed=1, fixed_digits=[d0],
                                        **({"cost_cap": cap} if cap is not None else {})),
                digits, rank, world, xdev, initial_cap=cap0)
        else:
            best, decided, full_evals, _ = plan_digits_sharded(
                lambda d0, cap: pl.plan(arr, p.sla_us, p.windows_us, n_fixed=1, fixed_digits=[d0], shard=rank,
                                        n_shards=world, **({"cost_cap": cap} if cap is not None else {})),
                digits, rank, world, xdev, initial_cap=cap0)
    else:
        # one exact plan, every rank on its interleaved share of every B&B survivor's subtree;
        # with N > 1 the index range runs in `rounds` pieces and the ranks exchange the
        # incumbent cost between them (dist.plan_range_rounds; exact for any cap >= OPT)
        rb, decided, full_evals, _ = plan_range_rounds(
            lambda b0, b1, cap: pl.plan(arr, p.sla_us, p.windows_us, begin=b0, end=b1, shard=rank, n_shards=world,
                                        **({"cost_cap": cap} if cap is not None else {})),
            p.space_size(), rounds, rank, world, xdev, initial_cap=cap0)
        best = (rb[0], 0, rb[1], rb[2]) if rb is not None else None
    local_decided = decided
    keys = [cost_bits(best[0]) if best else INF_BITS, best[1] if best else 0, best[2] if best else 0]
    payload = [best[3] if best else -1]
    if world > 1:
        keys, pay = reduce_lex(keys, payload, xdev)
        # C5 decides 2^70 candidates: exceeds int64, so sum as two int64 halves
        hi_lo = torch.tensor([decided >> 32, decided & 0xffffffff], dtype=torch.int64, device=xdev)
        dist.all_reduce(hi_lo)
        decided = (int(hi_lo[0].item()) << 32) + int(hi_lo[1].item())
        lat = pay[0]
        # every rank's share (balanced under pruning), as hi/lo int64 halves
        mine = torch.tensor([local_decided >> 32, local_decided & 0xffffffff, full_evals], dtype=torch.int64,
                            device=xdev)
        allv = [torch.zeros_like(mine) for _ in range(world)]
        dist.all_gather(allv, mine)
        per_rank = [(int(v[0].item()) << 32) + int(v[1].item()) for v in allv]
        per_rank_full = [int(v[2].item()) for v in allv]
    else:
        lat = payload[0]
        per_rank, per_rank_full = [local_decided], [full_evals]
    b.record(stream)
    torch.cuda.synchronize(dev)
    wall = time.perf_counter() - t0
    tt = torch.tensor([a.elapsed_time(b)], dtype=torch.float64, device=xdev)
    if world > 1:
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
    sec = float(tt.item()) / 1e3
    cost = bits_cost(keys[0])
    out = {"candidates": decided, "time_to_optimal_s": sec, "wall_s": wall, "decided_per_s": decided / sec,
           "sla_us": p.sla_us, "instances": None if p.instances is None else p.instances.tolist(),
           "full_evals_local": full_evals, "digits": os.environ.get("SMILESS_BENCH_DIGITS", "blocks") if pinned else None, "decided_per_rank": per_rank, "full_evals_per_rank": per_rank_full,
           "rounds": 1 if pinned else rounds,
           "cost": cost, "max_latency_us": lat if cost is not None else -1,
           "seed_cap": {"enabled": seed, "cap": cap0, "wall_ms": seed_ms}}
    if cost is not None:
        kw = dict(n_fixed=1, fixed_digits=[keys[1]]) if pinned else {}
        c, w = pl.decode(keys[2], Wn, **kw)
        out.update({"index": keys[2], "config": c.tolist(), "window": w.tolist(),
                    "windows_nonzero": int((w != 0).sum()), "full_evals_fraction": full_evals / max(1, decided)})
        if pinned:
            out["digit0"] = keys[1]
        if rank == 0:
            from oracle import OracleProblem
            oc, ol, of = OracleProblem(p, **kw).evaluate([keys[2]])
            out["oracle_check"] = {"feasible": bool(of[0]), "cost_bits_equal": bool(oc[0] == cost),
                                   "latency_equal": int(ol[0]) == out["max_latency_us"]}
    return out


def plan_kernel_ops_per_candidate(p) -> float:
    """Integer ops per candidate of smiless_plan_kernel (no prefix memoisation: every lane
    walks its own upstream) over the horizon, counted like algorithmic_ops_per_candidate.  A
    scale-out plan's kernel DAG ends in the virtual sink (one keep-alive variant joining the
    real sinks), so every real function is upstream; ring shifts are register moves and are
    not counted."""
    n = p.n_funcs
    Wn = len(p.windows_us)
    listed = set(int(v) for v in p.pred_idx)
    sinks = [k for k in range(n) if k not in listed]
    joins = sum(max(0, len(p.preds(k)) - 1) for k in range(n))
    if virtual_sink(p):
        upstream = 7 * n + joins + (len(sinks) - 1)       # + the virtual sink's join
        per_unit = 3 + 4                                   # one keep-alive variant
        share = 1
    else:
        G = configs_per_lane(p)
        up_sinks = sum(1 for k in sinks if k != n - 1)
        upstream = 7 * (n - 1) + joins + up_sinks
        w0 = 1 if int(p.windows_us[0]) == 0 else 0
        per_unit = G * (3 + 4 * w0 + 7 * (Wn - w0))
        share = G * Wn
    return (upstream + per_unit) / share * (len(p.arrivals_us) - 1)


SLICE_PINNED = {"C3": 4, "C5": 6, "C3s": 4, "C5s": 6}   # leading functions pinned (fastest, keep-alive)


def virtual_sink(p) -> bool:
    """Mirror of host.cpp virt_sink: with SMILESS_LRING=0 a scaled-out LAST function makes the
    kernels append the virtual sink (no sink sharing, no memoised path); by default its window
    variants carry instance rings instead."""
    return (p.instances is not None and int(p.instances[-1]) > 1 and
            os.environ.get("SMILESS_LRING", "1") == "0")


def throughput_slice(name, S, dev, stream, local, steps=2, n_cand=1 << 24):
    """Throughput mode (no pruning) over a fixed slice of C3 / C5: the first n_cand candidates
    with the leading functions pinned to their fastest configuration, keep-alive.  Reports
    candidates/s, function-steps/s and the evaluator's fraction of the issue peak for the
    kernel path it takes (scale-out plans: smiless_plan_kernel; else the memoised kernels)."""
    import torch
    p = W.make_config(name)
    Wn = len(p.windows_us)
    nf = SLICE_PINNED[name]
    M = int(p.n_configs[0])
    fixed = [int(np.argmin(p.exec_us[k * M:(k + 1) * M])) * Wn for k in range(nf)]
    pl = S.planner_for(p, device=local, stream=stream.cuda_stream)
    arr = torch.as_tensor(p.arrivals_us).to(dev)
    kw = dict(n_fixed=nf, fixed_digits=fixed, end=n_cand, flags=S.FLAG_NO_PRUNE)
    pl.plan(arr, p.sla_us, p.windows_us, **kw)                          # NVRTC + warm-up
    torch.cuda.synchronize(dev)
    a = torch.cuda.Event(enable_timing=True)
    b = torch.cuda.Event(enable_timing=True)
    kms = 0.0
    a.record(stream)
    for _ in range(steps):
        r = pl.plan(arr, p.sla_us, p.windows_us, **kw)
        kms += r.eval_kernel_ms
    b.record(stream)
    torch.cuda.synchronize(dev)
    sec = a.elapsed_time(b) / 1e3
    scale_out = virtual_sink(p)
    memo = r.eval_path in (S.PATH_MEMO, S.PATH_MEMO_FUSED)
    ops = (plan_kernel_ops_per_candidate(p) if scale_out else
           algorithmic_ops_per_candidate(p, memo=memo, split=os.environ.get("SMILESS_SPLITCOST", "1") != "0"))
    value = steps * r.n_decided / sec
    return {"candidates_per_step": r.n_decided, "value": value, "unit": UNIT,
            "function_steps_per_s": value * p.n_funcs * (len(p.arrivals_us) - 1),
            "slice": f"first {n_cand} candidates, functions 0..{nf - 1} pinned to digits {fixed}",
            "kernel": ("smiless_plan_kernel (scaled-out last function: virtual sink)" if scale_out else
                       KERNEL_LABEL.get(r.eval_path, "smiless_plan_kernel") +
                       (" (scale-out upstream rings)" if p.instances is not None else "")),
            "int_ops_per_candidate": ops, "achieved_int_ops_per_s": ops * r.n_decided / (kms / steps / 1e3),
            "instances": None if p.instances is None else p.instances.tolist(),
            "winner": {"index": r.index, "cost": r.cost} if r.feasible else None}


def gap_fractions(p):
    """fraction of inter-arrival gaps longer than T + I per function and
    configuration (both Case I and Case II must occur for the window dimension to matter)."""
    gaps = np.diff(np.asarray(p.arrivals_us, dtype=np.int64))
    off = np.concatenate([[0], np.cumsum(p.n_configs)])
    per_fn = []
    for k in range(p.n_funcs):
        fr = [float((gaps > int(p.init_us[r]) + int(p.exec_us[r])).mean()) for r in range(off[k], off[k + 1])]
        per_fn.append({"min": min(fr), "median": float(np.median(fr)), "max": max(fr)})
    return {"per_function_over_configs": per_fn, "gaps": int(len(gaps))}


# The paper's own numbers (BASELINE.md sections 1-2), quoted as context: other hardware, other
# quantities (its planner is a heuristic with a closed-form latency, no per-candidate walk)
PAPER_CONTEXT = {
    "hardware": "8-node cluster, 2x Intel Xeon Gold 5320 + 1x RTX 3090 per node, 10 GbE (PAPER.md:299)",
    "top1_strategy_search": "< 20 ms for a DAG whose longest path has 12 functions (PAPER.md:367, Fig. 16a)",
    "autoscaler_solve": "< 0.1 ms per function (PAPER.md:367, Fig. 16b)",
    "cost_vs_icebreaker": "up to 5.73x lower cost with 0 SLA violations (PAPER.md:17, :305-311)",
    "vs_opt": "OPT by exhaustive search; 'additional total cost of 50%' (PAPER.md:305, likely garbled)",
    "default_sla": "2 s (PAPER.md:283)",
}


TRAFFIC_BASIS = {
    3: "ncu dram__bytes_read+write per plan call (profiles/ncu_memo_summary.json): the memoised x-buffer "
       "round trip, ~5.4 GB per 65,536 prefixes",
    4: "ncu dram__bytes_read+write per plan call (profiles/ncu_fused_summary.json): the fused kernel keeps "
       "the x stream in a shared-memory ring; what is left is the tables, offsets and the cost re-walk",
}
KERNEL_LABEL = {
    3: "smiless_variants_kernel + smiless_upstream_kernel (prefix memoisation, x stream through HBM)",
    4: "smiless_fused_kernel (prefix memoisation: producer warp -> shared-memory ring -> consumer warps)",
}


def measured_peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


def ncu_traffic(path: int, plan_launches: int, split: bool = True):
    """DRAM bytes of the timed kernels per plan call (the unit `achieved` uses), from the
    committed ncu --set full summaries.  Fused memo path (PATH_MEMO_FUSED): one plan call =
    prep + B x (fused[, plan-kernel cost re-walk]) + reduce + exact; the x stream stays in
    shared memory, so a batch moves only the tables, offsets and the re-walked units' inputs.
    Two-kernel memo path: B x (upstream, variants[, variants cost]), each batch moving the
    upstream kernel's x-buffer write and the variants kernel's read of it."""
    PATH_MEMO, PATH_MEMO_FUSED = 3, 4
    try:
        if path == PATH_MEMO_FUSED:
            d = json.load(open(os.path.join(ROOT, "profiles", "ncu_fused_summary.json")))
            per = sum(k["dram_bytes_per_launch"] for k in d.get("launches", [d])
                      if k["dram_bytes_per_launch"] == k["dram_bytes_per_launch"])      # skip NaN
            return per * max(1, (plan_launches - 3) // (2 if split else 1))
        if path == PATH_MEMO:
            d = json.load(open(os.path.join(ROOT, "profiles", "ncu_memo_summary.json")))
            pair = sum(k["dram_bytes_per_launch"] for k in d["launches"])
            return pair * max(1, (plan_launches - 3) // (3 if split else 2))
        d = json.load(open(os.path.join(ROOT, "profiles", "ncu_evaluator_summary.json")))
        return d.get("dram_bytes_per_launch")
    except Exception:
        return None


def host_cpu():
    """CPU model and clock of this host (lscpu, else /proc/cpuinfo) for the oracle timings."""
    info = {"model": None, "mhz": None, "max_mhz": None, "nproc": os.cpu_count()}
    try:
        import subprocess
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            k, _, v = line.partition(":")
            k, v = k.strip(), v.strip()
            if k == "Model name":
                info["model"] = v
            elif k == "CPU MHz":
                info["mhz"] = float(v)
            elif k == "CPU max MHz":
                info["max_mhz"] = float(v)
    except Exception:
        pass
    if info["mhz"] is None:
        try:
            for line in open("/proc/cpuinfo"):
                if line.startswith("cpu MHz"):
                    info["mhz"] = float(line.split(":")[1])
                    break
                if line.startswith("model name") and not info["model"]:
                    info["model"] = line.split(":")[1].strip()
        except Exception:
            pass
    return info


def cpu_oracle_rate(p, kw, n_random: int = 1 << 16, n_first: int = 1 << 16, threads=None, seed: int = 8):
    """Oracle (as it stands) on the host cores, SURVEY 8(d) sample: 2^16 seeded random indices
    of the space plus its first 2^16 indices, evaluated by `threads` threads (ctypes releases
    the GIL).  Returns (candidates/s, sample size, seconds, threads)."""
    from concurrent.futures import ThreadPoolExecutor
    import numpy as np_
    from oracle import OracleProblem
    threads = threads or os.cpu_count() or 1
    o = OracleProblem(p, n_fixed=kw["n_fixed"], fixed_digits=kw["fixed_digits"])
    space = o.space_size()
    rng = np_.random.default_rng(seed)
    idx = np_.concatenate([rng.integers(0, space, size=n_random, dtype=np_.uint64),
                           np_.arange(min(n_first, space), dtype=np_.uint64)])
    parts = np_.array_split(idx, threads)
    t0 = time.perf_counter()
    with ThreadPoolExecutor(threads) as ex:
        list(ex.map(o.evaluate, parts))
    dt = time.perf_counter() - t0
    return len(idx) / dt, len(idx), dt, threads


def run_reference(args):
    """--impl reference: the CPU oracle as the reference arm (rank 0 only)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    weak = os.environ.get("SMILESS_BENCH_SCALING", "weak") != "strong" and args.workload == "C2"
    p, kw = workload(args.workload)
    from oracle import OracleProblem
    threads = os.cpu_count() or 1
    o = OracleProblem(p, n_fixed=kw["n_fixed"], fixed_digits=kw["fixed_digits"])
    # size one step so the whole --steps K --warmup W run takes ~2 minutes of host work
    probe = max(threads, 8)
    t0 = time.perf_counter()
    o.plan(0, probe, n_threads=threads)
    per = (time.perf_counter() - t0) / probe
    step_s = max(1.0, min(8.0, 120.0 / max(1, args.steps)))
    n_step = max(threads, int(step_s / max(per, 1e-9)))
    for _ in range(args.warmup):
        o.plan(0, min(n_step, threads * 2), n_threads=threads)
    t0 = time.perf_counter()
    for s in range(args.steps):
        o.plan(s * n_step, (s + 1) * n_step, n_threads=threads)
    dt = time.perf_counter() - t0
    value = args.steps * n_step / dt
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt / args.steps * 1e3,
        "higher_is_better": True, "scaling": "weak" if weak else "strong", "vs_baseline": None,
        "dtype": "i64+f64", "data": "synthetic", "config": config_block(p, kw, args, weak),
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle",
                         "sample": f"{n_step} consecutive candidates of the slice per step",
                         "cpu_model": host_cpu()["model"], "cpu_mhz": host_cpu()["mhz"]},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def config_block(p, kw, args, weak=False):
    space = 1
    for k in range(kw["n_fixed"], p.n_funcs):
        space *= int(p.n_configs[k]) * len(p.windows_us)
    n_slices = args.gpus if weak else 1
    per_rank = (f"; rank r plans the slice with function 1 on config 15 - r (digit {kw['fixed_digits'][1]} - 8r)"
                if weak and args.gpus > 1 else "")
    return {
        "workload": f"{p.name}: {p.n_funcs}-function DAG, {int(p.n_configs[0])} configs x {len(p.windows_us)} "
                    f"windows, J={len(p.arrivals_us)} arrivals, SLA {p.sla_us} us; slice of {space} candidates "
                    f"(functions 0..{kw['n_fixed'] - 1} pinned to digits {list(kw['fixed_digits'])}){per_rank}; "
                    f"throughput mode (no pruning)",
        "candidates_per_step": space * n_slices,
        "arrivals": len(p.arrivals_us),
        "l2": "256 MiB buffer written between timed steps (L2 flushed); working set < 1 MB",
        "parallelism": (f"weak scaling: one {space}-candidate slice per rank x{args.gpus}" if weak
                        else f"candidate-space sharding x{args.gpus}"),
    }


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--workload", default="C2")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-pruned", action="store_true")
    ap.add_argument("--no-full-space", action="store_true",
                    help="skip the exhaustive pruned plan of the whole workload space (time-to-optimal)")
    ap.add_argument("--no-c4", action="store_true", help="skip the C4 SLA-sweep re-planning rate")
    ap.add_argument("--no-extra", action="store_true",
                    help="skip C1 time-to-optimal, the C3/C5 throughput slices and the live-window SLAs")
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist
    from paper_conf_sc_luxl0y024_b200 import smiless as S
    from paper_conf_sc_luxl0y024_b200.dist import reduce_best, union_index as dist_union_index

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # SMILESS_BENCH_SAME_GPU=1 (testing the multi-rank flow on a one-GPU box): every rank
    # uses cuda:0 and the exchange runs on gloo; the real runs use one GPU per rank + NCCL
    same_gpu = os.environ.get("SMILESS_BENCH_SAME_GPU") == "1"
    if same_gpu:
        local = 0
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    xdev = torch.device("cpu") if same_gpu else dev           # device of the collective tensors
    if world > 1:
        if same_gpu:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)

    weak = os.environ.get("SMILESS_BENCH_SCALING", "weak") != "strong" and args.workload == "C2"
    p, kw = workload(args.workload, rank if weak else 0)
    stream = torch.cuda.current_stream(dev)
    pl = S.planner_for(p, device=local, stream=stream.cuda_stream)
    arr_dev = torch.as_tensor(p.arrivals_us).to(dev)                 # HBM-resident inputs
    arr_pin = torch.as_tensor(p.arrivals_us).pin_memory()            # e2e: pinned host inputs
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    # weak: every rank its own slice (no sharding inside); strong: the rank-0 slice split
    shard_kw = dict(shard=0, n_shards=1) if weak else dict(shard=rank, n_shards=world)
    plan_kw = dict(kw, flags=S.FLAG_NO_PRUNE, **shard_kw)
    slice_size = pl.space_size(len(p.windows_us), kw["n_fixed"])

    def union_index(r):
        # index in the function-0-pinned space (function 1's digit is the rank's slice), so
        # the lowest-index tie-break is the same for every world size
        if not (weak and r.feasible):
            return r.index
        return dist_union_index(kw["fixed_digits"][1], slice_size, r.index)

    def step(arrivals):
        r = pl.plan(arrivals, p.sla_us, p.windows_us, **plan_kw)
        if world > 1:
            reduce_best(r.cost if r.feasible else None, union_index(r), r.max_latency_us, r.n_decided, xdev)
        return r

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize(dev)

    t_first = time.perf_counter()
    first_call_s = None
    for w_ in range(args.warmup):
        r = step(arr_dev)
        if w_ == 0:
            torch.cuda.synchronize(dev)
            first_call_s = time.perf_counter() - t_first      # includes the NVRTC specialisation
    barrier()
    # NVRTC compile of the DAG-specialised module, timed on its own (SURVEY 8(d) ii): a fresh
    # planner for the same DAG compiles once on its first call
    t_c = time.perf_counter()
    pl_c = S.planner_for(p, device=local, stream=stream.cuda_stream)
    pl_c.jit_compile(p.arrivals_us, p.sla_us, p.windows_us, **dict(kw, flags=S.FLAG_NO_PRUNE))
    nvrtc_s = time.perf_counter() - t_c
    del pl_c

    def timed(arrivals, n):
        evs = []
        res = None
        launches = 0
        kernel_ms = 0.0
        for _ in range(n):
            flush.fill_(1)                                           # L2 flush, outside the events
            a = torch.cuda.Event(enable_timing=True)
            b = torch.cuda.Event(enable_timing=True)
            a.record(stream)
            res = step(arrivals)
            b.record(stream)
            evs.append((a, b))
            launches += res.launches
            kernel_ms += res.eval_kernel_ms
        torch.cuda.synchronize(dev)
        ms = sum(a.elapsed_time(b) for a, b in evs)
        t = torch.tensor([ms], dtype=torch.float64, device=xdev)
        if world > 1:
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item()), res, launches, kernel_ms

    barrier()
    with ClockSampler(local) as clk:
        ms, res, launches, kernel_ms = timed(arr_dev, args.steps)
    barrier()
    barrier()
    ms_e2e, res_e2e, _, _ = timed(arr_pin, args.steps)
    barrier()

    cands = int(res.n_decided)
    if world > 1:
        t = torch.tensor([cands], dtype=torch.int64, device=xdev)
        dist.all_reduce(t)
        cands = int(t.item())
    steps_e2e = args.steps
    value = cands * args.steps / (ms / 1e3)
    e2e_value = cands * steps_e2e / (ms_e2e / 1e3)

    # pruned (exact plan with early exit): time-to-optimal of the same slice
    pruned = None
    if not args.no_pruned:
        kwp = dict(kw, flags=0, **shard_kw)
        pl.plan(arr_dev, p.sla_us, p.windows_us, **kwp)          # NVRTC compile of the prune-mode kernels
        barrier()
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record(stream)
        rp = pl.plan(arr_dev, p.sla_us, p.windows_us, **kwp)
        if world > 1:
            reduce_best(rp.cost if rp.feasible else None, union_index(rp), rp.max_latency_us, rp.n_decided, xdev)
        b.record(stream)
        torch.cuda.synchronize(dev)
        pruned = {"time_to_optimal_ms": a.elapsed_time(b), "index": rp.index, "cost": rp.cost,
                  "max_latency_us": rp.max_latency_us, "full_evals_fraction": rp.n_full_evals / max(1, rp.n_decided)}

    # time-to-optimal of the WHOLE configuration space (C2: 2^42 candidates): exact plan with
    # pruning, sharded over the ranks (interleaved chunks) + NCCL reduction of the winner
    full = None
    if not args.no_full_space:
        full = {}
        for name in os.environ.get("SMILESS_BENCH_FULL", "C2,C3,C3s,C5,C5s").split(","):
            full[name] = full_space_opt(name, S, rank, world, dev, xdev, stream, local, barrier)
        if not args.no_extra:
            # SURVEY 8(d) / VERDICT: instances where the pre-warm windows are live at J = 10^4
            for sla in (4_000_000, 8_000_000):
                full[f"C2@SLA{sla // 1_000_000}s"] = full_space_opt("C2", S, rank, world, dev, xdev, stream, local,
                                                                   barrier, sla=sla)

    # C1 time-to-optimal, C3 / C5 throughput slices (N = 1)
    extra = None
    if not args.no_extra and world == 1:
        extra = {}
        p1 = W.make_config("C1")
        pl1 = S.planner_for(p1, device=local, stream=stream.cuda_stream)
        arr1 = torch.as_tensor(p1.arrivals_us).to(dev)
        pl1.plan(arr1, p1.sla_us, p1.windows_us)
        barrier()
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record(stream)
        r1 = pl1.plan(arr1, p1.sla_us, p1.windows_us)
        b.record(stream)
        torch.cuda.synchronize(dev)
        from oracle import OracleProblem
        ref1 = OracleProblem(p1).plan()
        extra["C1_time_to_optimal"] = {"time_to_optimal_ms": a.elapsed_time(b), "candidates": 4096,
                                       "index": r1.index, "cost": r1.cost, "max_latency_us": r1.max_latency_us,
                                       "oracle_plan_equal": ref1 == (r1.index, r1.cost, r1.max_latency_us)}
        for name in ("C3", "C5"):
            extra[f"{name}_throughput_slice"] = throughput_slice(name, S, dev, stream, local)
        extra["C2_gaps_longer_than_T_plus_I"] = gap_fractions(p)

    # C4 (configs[3]): 1,000 re-plans of 100 predicted arrivals, 6 SLAs per pass, exhaustive each
    c4 = None
    if not args.no_c4 and world == 1:
        p4 = W.make_config("C4")
        pl4 = S.planner_for(p4, device=local, stream=stream.cuda_stream)
        wins = [torch.as_tensor(w).to(dev) for w in W.c4_replans(1000)]
        pl4.plan_sla_sweep(wins[0], W.C4_SLAS_US, p4.windows_us)
        barrier()
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record(stream)
        feas = [0] * len(W.C4_SLAS_US)
        mono = True
        for w in wins:
            rs = pl4.plan_sla_sweep(w, W.C4_SLAS_US, p4.windows_us)
            cs = [r.cost if r.feasible else float("inf") for r in rs]
            mono &= all(cs[i + 1] <= cs[i] for i in range(len(cs) - 1))
            for i, r in enumerate(rs):
                feas[i] += r.feasible
        b.record(stream)
        torch.cuda.synchronize(dev)
        sec = a.elapsed_time(b) / 1e3
        c4 = {"replans": len(wins), "slas": W.C4_SLAS_US, "candidates_per_replan": pl4.space_size(len(p4.windows_us)),
              "replans_per_s": len(wins) / sec, "seconds": sec, "feasible_per_sla": feas,
              "opt_non_increasing_in_sla": bool(mono)}

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return 0

    peaks = measured_peaks()
    props = torch.cuda.get_device_properties(dev)
    clocks = clk.summary()
    sm_mhz = clocks["sm_mhz"] or peaks.get("sm_max_mhz", 1965.0)
    peak_ops = props.multi_processor_count * ISSUE_LANES_PER_CLK_PER_SM * float(clocks["sm_max_mhz"] or 1965.0) * 1e6
    memo = res.eval_path in (S.PATH_MEMO, S.PATH_MEMO_FUSED)
    split = os.environ.get("SMILESS_SPLITCOST", "1") != "0"
    ops_per_cand = algorithmic_ops_per_candidate(p, memo=memo, split=split)
    ops = ops_per_cand * res.n_decided
    kernel_ms_per_step = kernel_ms / args.steps
    achieved = ops / (kernel_ms_per_step / 1e3)
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True,
        "scaling": "weak" if weak else "strong", "vs_baseline": None, "dtype": "i32+f64", "data": "synthetic",
        "config": config_block(p, kw, args, weak),
        "time_to_optimal_ms": ms / args.steps,
        "winner": {"index": res.index, "cost": res.cost, "max_latency_us": res.max_latency_us,
                   "config": res.config.tolist(), "window": res.window.tolist()} if world == 1 else None,
        "pruned": pruned,
        "time_to_optimal_full_space": full,
        "c4_sla_sweep_replanning": c4,
        "extra": extra,
        "paper_context": PAPER_CONTEXT,
        "gpu_launches": launches,
        "e2e": {"value": e2e_value, "unit": UNIT, "h2d_bytes_per_step": int(res_e2e.h2d_bytes),
                "d2h_bytes_per_step": int(res_e2e.d2h_bytes), "steps": steps_e2e,
                "bytes_basis": "counted by the library per smiless_plan call (smiless_plan_result)"},
        "clocks": clocks,
        "roofline": {"bound": "alu", "achieved": achieved, "peak": peak_ops, "unit": "int-ops/s",
                     "frac": achieved / peak_ops, "traffic": ncu_traffic(res.eval_path, res.launches, split),
                     "traffic_basis": TRAFFIC_BASIS.get(res.eval_path, "ncu dram__bytes_read+write per plan call"),
                     "kernel": KERNEL_LABEL.get(res.eval_path, "smiless_plan_kernel"),
                     "kernel_ms_per_launch": kernel_ms_per_step,
                     "int_ops_per_candidate": ops_per_cand, "configs_per_lane": configs_per_lane(p),
                     "peak_basis": "issue peak: SMs x 4 SMSP x 32 lanes x sm_max_mhz (DESIGN.md Roofline)"},
        "kernel_share_of_step": kernel_ms_per_step / (ms / args.steps),
        # SURVEY 8(d) i/ii: function-steps/s (N functions x (J-1) transitions per candidate) and
        # the NVRTC specialisation, reported apart from the timed steps
        "function_steps_per_s": value * p.n_funcs * (len(p.arrivals_us) - 1),
        "nvrtc_compile_s": nvrtc_s,
        "first_call_s": first_call_s,
    }
    if world == 1 and not args.no_cpu_baseline:
        rate, n, dt, threads = cpu_oracle_rate(p, kw)
        rate1, n1, dt1, _ = cpu_oracle_rate(p, kw, n_random=1 << 12, n_first=1 << 12, threads=1)  # SURVEY 8(d) iii
        cpu = host_cpu()
        line["cpu_baseline"] = {"value": rate, "unit": UNIT, "cores": threads, "kind": "oracle",
                                "sample": f"2^16 seeded random + the first 2^16 candidates of the slice ({n} in "
                                          f"{dt:.1f} s, J={len(p.arrivals_us)})",
                                "cpu_model": cpu["model"], "cpu_mhz": cpu["mhz"], "cpu_max_mhz": cpu["max_mhz"],
                                "function_steps_per_s": rate * p.n_funcs * (len(p.arrivals_us) - 1),
                                "single_core_value": rate1,
                                "single_core_sample": f"2^12 random + first 2^12 candidates, 1 thread ({dt1:.1f} s)"}
        if full:
            for name, f in full.items():          # what the same exhaustive search costs on the oracle
                f["oracle_extrapolated_s"] = f["candidates"] / rate
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
