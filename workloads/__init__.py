"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module holds NO arithmetic of the method (no simulation, no cost, no
latency, no argmin).  It only draws the inputs the paper's workloads have:

* DAG topologies (topologically ordered CSR over predecessors), shaped after
  the paper's applications (PAPER.md:25 conversational pipeline ASR->LLM->TTS;
  PAPER.md:60 IPA with NLP/IR/QA/TTS stages; PAPER.md:285 AMBER-alert fan-out).
* Per-function x per-config profiles from the paper's own models:
  inference time Eq. (1)/(2) (batch B = 1), init time
  mu + 3 sigma, prices from PAPER.md:299.
* Window grids (the cold-start policy set S; 0 = keep-alive,
  PAPER.md:194).
* Predicted arrival sequences: Poisson, bursty 2-state MMPP, and
  Azure-Functions-shaped (per-1-s-window counts, variance/mean
  >= 2, compressed 1 min -> 2 s).

Every generator takes a numpy Generator; `make_config(name)` seeds it with
``default_rng(1000 + config#)``.
"""
from __future__ import annotations

import dataclasses
from typing import Dict, List, Optional, Sequence

import numpy as np

US_PER_S = 1_000_000
US_PER_H = 3_600 * US_PER_S

# ---------------------------------------------------------------------------
# DAGs: predecessor CSR, topological order (every pred index < its function).
# ---------------------------------------------------------------------------

def csr_from_preds(preds: Sequence[Sequence[int]]):
    ptr = [0]
    idx: List[int] = []
    for p in preds:
        idx.extend(int(v) for v in p)
        ptr.append(len(idx))
    return np.asarray(ptr, dtype=np.int32), np.asarray(idx, dtype=np.int32)


DAGS: Dict[str, List[List[int]]] = {
    # C1: ASR -> LLM -> TTS chain
    "chain3": [[], [0], [1]],
    # C2/C4: IPA-shaped: 0 SR, 1 IR sources; 2 NLP<-0;
    # 3 QA<-{1,2}; 4 TG<-3; 5 TTS<-4
    "ipa6": [[], [], [0], [1, 2], [3], [4]],
    # C3: fan-out/fan-in (AMBER alert): 0 OD -> {1..6 TRS} -> 7
    "fan8": [[], [0], [0], [0], [0], [0], [0], [1, 2, 3, 4, 5, 6]],
    # C5: 10-function mixed chain/parallel
    "mixed10": [[], [0], [1], [2], [1], [3, 4], [5], [5], [7], [6, 8]],
}

# ---------------------------------------------------------------------------
# Config grids (CPU 1/2/4/8/16 cores; GPU in 10% MPS units,
# PAPER.md:124).  ("cpu", cores) or ("gpu", fraction).
# ---------------------------------------------------------------------------

CONFIG_GRIDS = {
    16: [("cpu", c) for c in (1, 2, 4, 8, 16, 32)] + [("gpu", f / 10) for f in range(1, 11)],
    12: [("cpu", c) for c in (1, 2, 4, 8, 16)] + [("gpu", f) for f in (0.1, 0.2, 0.3, 0.4, 0.6, 0.8, 1.0)],
    8: [("cpu", c) for c in (2, 4, 8, 16)] + [("gpu", f) for f in (0.2, 0.4, 0.7, 1.0)],
    4: [("cpu", 4), ("cpu", 16), ("gpu", 0.3), ("gpu", 1.0)],
}

# Window grids in microseconds (strictly increasing; 0 = keep-alive).
WINDOW_GRIDS = {
    4: [0, 500_000, 2_000_000, 8_000_000],
    8: [0, 250_000, 500_000, 1_000_000, 2_000_000, 4_000_000, 8_000_000, 16_000_000],
    16: [0] + [int(round(v)) for v in np.geomspace(1e5, 3.2e7, 15)],
}

CPU_PRICE_PER_CORE_H = 0.034   # PAPER.md:299 (AWS c6g)
GPU_PRICE_FULL_H = 3.06        # PAPER.md:299 (10% GPU = 10% of p3.2xlarge)


def window_grid(w: int) -> np.ndarray:
    return np.asarray(WINDOW_GRIDS[w], dtype=np.int32)


def gen_profiles(rng: np.random.Generator, n_funcs: int, n_configs: int):
    """Per function x config: exec_us (int32), init_us (int32), price_per_us (f64).

    Inference time via Eq. (1) (CPU) / Eq. (2) (GPU) with batch size B = 1
    (PAPER.md:128-137); init time mu + 3 sigma with sigma = 0.1 mu
    (PAPER.md:120, :329); GPU init longer than CPU.  Times are
    rounded to integer microseconds (reading G14).
    """
    grid = CONFIG_GRIDS[n_configs]
    slope = np.zeros((n_funcs, n_configs), dtype=np.float64)      # lambda * (alpha / x + beta)
    icept = np.zeros((n_funcs, n_configs), dtype=np.float64)      # gamma
    ex = np.zeros((n_funcs, n_configs), dtype=np.int64)
    ini = np.zeros((n_funcs, n_configs), dtype=np.int64)
    price = np.zeros((n_funcs, n_configs), dtype=np.float64)
    for k in range(n_funcs):
        a_c = rng.uniform(0.3, 3.0) * US_PER_S     # alpha_c: s * core
        b_c = rng.uniform(5e3, 5e4)                 # beta_c
        l_c = rng.uniform(1.0, 1.2)                 # lambda_c
        g_c = rng.uniform(2e3, 2e4)                 # gamma_c (network)
        a_g = a_c / rng.uniform(8.0, 30.0)          # GPU ~10x faster
        b_g = rng.uniform(2e3, 1e4)
        l_g = rng.uniform(1.0, 1.1)
        g_g = g_c
        mu_c = rng.uniform(0.5, 2.5) * US_PER_S
        mu_g = mu_c + rng.uniform(1.5, 5.0) * US_PER_S
        for c, (kind, amount) in enumerate(grid):
            jitter = rng.uniform(0.97, 1.03)
            if kind == "cpu":
                slope[k, c], icept[k, c] = l_c * (a_c / amount + b_c), g_c
                t_inf = l_c * 1 * (a_c / amount + b_c) + g_c          # Eq. (1), B = 1
                mu = mu_c * jitter
                p = amount * CPU_PRICE_PER_CORE_H
            else:
                slope[k, c], icept[k, c] = l_g * (a_g / amount + b_g), g_g
                t_inf = l_g * 1 * (a_g / amount + b_g) + g_g          # Eq. (2), B = 1
                mu = mu_g * jitter
                p = amount * GPU_PRICE_FULL_H
            sigma = 0.1 * mu
            ex[k, c] = int(round(t_inf))
            ini[k, c] = int(round(mu + 3.0 * sigma))                   # mu + n sigma, n = 3
            price[k, c] = p / US_PER_H
    gen_profiles.last_batch_model = (slope.reshape(-1), icept.reshape(-1))
    return ex.astype(np.int32), ini.astype(np.int32), price


# ---------------------------------------------------------------------------
# Arrivals (absolute integer microseconds, non-decreasing).
# ---------------------------------------------------------------------------

def poisson_arrivals(rng: np.random.Generator, n: int, rate_per_s: float) -> np.ndarray:
    gaps = np.rint(rng.exponential(US_PER_S / rate_per_s, size=n)).astype(np.int64)
    gaps[0] = 0
    return np.cumsum(gaps)


def mmpp_arrivals(rng: np.random.Generator, n: int, rates=(0.2, 10.0), dwell_s=(60.0, 5.0)) -> np.ndarray:
    """Bursty 2-state Markov-modulated Poisson process: 0.2 req/s, mean dwell 60 s, and
    10 req/s bursts of mean 5 s.  C3 serves the bursts with scale-out
    instances (NEXT-4); the single-instance variant C3s softens the bursts to 3 req/s."""
    out = np.empty(n, dtype=np.int64)
    t = 0.0
    state = 0
    left = rng.exponential(dwell_s[state] * US_PER_S)
    i = 0
    while i < n:
        g = rng.exponential(US_PER_S / rates[state])
        if g <= left:
            left -= g
            t += g
            out[i] = int(round(t))
            i += 1
        else:
            t += left
            state ^= 1
            left = rng.exponential(dwell_s[state] * US_PER_S)
    out -= out[0]
    return np.maximum.accumulate(out)


def azure_arrivals(rng: np.random.Generator, n: int, mean_per_window: float = 0.25,
                   vmr: float = 3.0, period_windows: int = 720) -> np.ndarray:
    """Azure-Functions-shaped: per-1-s-window counts, negative
    binomial with variance/mean = vmr >= 2 under a sinusoidal
    diurnal envelope compressed 1 min -> 2 s; uniform within
    each window."""
    out: List[np.ndarray] = []
    total = 0
    w = 0
    while total < n:
        block = 4096
        ws = np.arange(w, w + block)
        env = mean_per_window * (1.0 + 0.8 * np.sin(2 * np.pi * ws / period_windows))
        env = np.maximum(env, 1e-3)
        # NB(r, p) with mean m and variance vmr * m: p = 1/vmr, r = m / (vmr - 1)
        r = env / (vmr - 1.0)
        counts = rng.negative_binomial(r, 1.0 / vmr)
        for i, c in enumerate(counts):
            if c:
                ts = (ws[i] + np.sort(rng.uniform(0.0, 1.0, size=c))) * US_PER_S
                out.append(np.rint(ts).astype(np.int64))
                total += c
        w += block
    arr = np.concatenate(out)[:n]
    arr -= arr[0]
    return np.maximum.accumulate(arr)


# ---------------------------------------------------------------------------
# The BASELINE.json configs as concrete inputs.
# ---------------------------------------------------------------------------

@dataclasses.dataclass
class Problem:
    name: str
    pred_ptr: np.ndarray      # int32 [N+1]
    pred_idx: np.ndarray      # int32 [E]
    n_configs: np.ndarray     # int32 [N]
    exec_us: np.ndarray       # int32 [sum M]
    init_us: np.ndarray       # int32 [sum M]
    price_per_us: np.ndarray  # f64   [sum M]
    arrivals_us: np.ndarray   # int64 [J]
    sla_us: int
    windows_us: np.ndarray    # int32 [W]
    # Eq. (1)/(2) batch model per row: inference time of a batch of B = slope * B + intercept
    batch_slope_us: Optional[np.ndarray] = None      # f64 [sum M]
    batch_intercept_us: Optional[np.ndarray] = None  # f64 [sum M]
    # scale-out: instances of each function (NEXT-4, reading G26); None = one each
    instances: Optional[np.ndarray] = None           # int32 [N]

    @property
    def n_funcs(self) -> int:
        return int(self.pred_ptr.shape[0] - 1)

    def preds(self, k: int) -> List[int]:
        return [int(v) for v in self.pred_idx[self.pred_ptr[k]:self.pred_ptr[k + 1]]]

    def space_size(self, n_fixed: int = 0) -> int:
        s = 1
        for k in range(n_fixed, self.n_funcs):
            s *= int(self.n_configs[k]) * int(self.windows_us.shape[0])
        return s

    def replace(self, **kw) -> "Problem":
        return dataclasses.replace(self, **kw)


def build_problem(name: str, dag: str, m: int, w: int, arrivals: np.ndarray,
                  rng: np.random.Generator, sla_us: int = 2 * US_PER_S) -> Problem:
    preds = DAGS[dag]
    ptr, idx = csr_from_preds(preds)
    n = len(preds)
    ex, ini, pr = gen_profiles(rng, n, m)
    slope, icept = gen_profiles.last_batch_model
    return Problem(
        name=name, pred_ptr=ptr, pred_idx=idx,
        n_configs=np.full(n, m, dtype=np.int32),
        exec_us=ex.reshape(-1), init_us=ini.reshape(-1), price_per_us=pr.reshape(-1),
        arrivals_us=np.ascontiguousarray(arrivals, dtype=np.int64), sla_us=int(sla_us),
        windows_us=window_grid(w), batch_slope_us=slope, batch_intercept_us=icept)


CONFIG_NUMBER = {"C1": 1, "C2": 2, "C3": 3, "C4": 4, "C5": 5, "C3s": 3, "C5s": 5}


def peak_window_count(arrivals_us, window_us: int = US_PER_S) -> int:
    """Largest number of predicted invocations in one 1-s window (the predictor
    forecasts invocations per 1-s window): the G the auto-scaler provisions for."""
    a = np.asarray(arrivals_us, dtype=np.int64)
    return int(np.bincount((a - a[0]) // window_us).max())


# Scale-out instance counts of C3 / C5 (inputs of model M, reading G26): for every function,
# the instances the paper's auto-scaler constraint (Eq. (7)/(8)) needs at the
# function's fastest configuration to keep up with the predicted peak G = peak_window_count()
# per window IT = I_s = 1 s: ceil(G / B) with B the largest batch meeting I_s.  Written here as
# data; tests/test_oracle_pins.py::test_workload_instances_are_the_autoscalers re-derives them
# with oracle/autoscale.py and the library's smiless_autoscale_rows.
SCALE_OUT_INSTANCES = {
    "C3": [2, 1, 4, 2, 3, 3, 2, 1],
    "C5": [2, 2, 2, 2, 3, 2, 1, 2, 2, 3],
}


def make_config(name: str, n_arrivals: Optional[int] = None) -> Problem:
    """BASELINE.json configs as seeded synthetic inputs.

    n_arrivals overrides J (parity tests use shorter horizons of the same
    distribution)."""
    rng = np.random.default_rng(1000 + CONFIG_NUMBER[name])
    if name == "C1":
        # 3-function chain, 4 configs x 4 windows, 100 Poisson arrivals at 0.25 req/s
        prof_rng = rng
        j = n_arrivals or 100
        arr_seed = rng.integers(1 << 62)
        arr = poisson_arrivals(np.random.default_rng(arr_seed), j, 0.25)
        return build_problem("C1", "chain3", 4, 4, arr, prof_rng)
    if name == "C2":
        j = n_arrivals or 10_000
        arr_seed = rng.integers(1 << 62)
        arr = poisson_arrivals(np.random.default_rng(arr_seed), j, 0.25)
        return build_problem("C2", "ipa6", 16, 8, arr, rng)
    if name in ("C3", "C3s"):
        # C3: 10 req/s bursts served by scale-out instances (NEXT-4);
        # C3s: the single-instance variant with the bursts softened to 3 req/s (round 1)
        j = n_arrivals or 10_000
        arr_seed = rng.integers(1 << 62)
        rates = (0.2, 10.0) if name == "C3" else (0.2, 3.0)
        arr = mmpp_arrivals(np.random.default_rng(arr_seed), j, rates=rates)
        p = build_problem(name, "fan8", 12, 8, arr, rng)
        if name == "C3":
            p.instances = np.asarray(SCALE_OUT_INSTANCES["C3"], dtype=np.int32)
        return p
    if name == "C4":
        # one re-plan window of the SLA x rate sweep (100 arrivals at 0.25 req/s)
        j = n_arrivals or 100
        arr_seed = rng.integers(1 << 62)
        arr = poisson_arrivals(np.random.default_rng(arr_seed), j, 0.25)
        return build_problem("C4", "ipa6", 8, 4, arr, rng)
    if name in ("C5", "C5s"):
        # C5: Azure-shaped 0.25 invocations per 1-s window with VMR 3 served by
        # scale-out instances (NEXT-4); C5s: the single-instance variant at 0.2 per window,
        # VMR 2.2 (round 1: the fastest single-instance plan meets 2 s)
        j = n_arrivals or 10_000
        arr_seed = rng.integers(1 << 62)
        mpw, vmr = (0.25, 3.0) if name == "C5" else (0.2, 2.2)
        arr = azure_arrivals(np.random.default_rng(arr_seed), j, mean_per_window=mpw, vmr=vmr)
        p = build_problem(name, "mixed10", 8, 16, arr, rng)
        if name == "C5":
            p.instances = np.asarray(SCALE_OUT_INSTANCES["C5"], dtype=np.int32)
        return p
    raise KeyError(name)


def c4_replans(n_replans: int = 1000, per_plan: int = 100, seed: int = 1004):
    """C4: re-planning windows of predicted invocations over rates {0.1, 0.25, 1}."""
    rng = np.random.default_rng(seed)
    rates = (0.1, 0.25, 1.0)
    return [poisson_arrivals(rng, per_plan, rates[i % 3]) for i in range(n_replans)]


C4_SLAS_US = [500_000, 1_000_000, 1_500_000, 2_000_000, 2_500_000, 3_000_000]


def random_problem(rng: np.random.Generator, n_funcs: int, max_configs: int, n_windows: int,
                   n_arrivals: int, time_scale: int = 1000, max_preds: int = 3,
                   sla_us: Optional[int] = None, zero_gap_p: float = 0.15) -> Problem:
    """Small random DAG problem for cross-checks (ragged configs, zero gaps,
    huge gaps, joins, multiple sinks)."""
    preds: List[List[int]] = []
    for k in range(n_funcs):
        if k == 0 or rng.random() < 0.25:
            preds.append([])
        else:
            npred = int(rng.integers(1, min(k, max_preds) + 1))
            preds.append(sorted(rng.choice(k, size=npred, replace=False).tolist()))
    ptr, idx = csr_from_preds(preds)
    ncfg = rng.integers(1, max_configs + 1, size=n_funcs).astype(np.int32)
    tot = int(ncfg.sum())
    ex = rng.integers(0, 5 * time_scale, size=tot).astype(np.int32)
    ini = rng.integers(0, 5 * time_scale, size=tot).astype(np.int32)
    price = rng.integers(1, 64, size=tot).astype(np.float64) / 1024.0
    wins = np.sort(rng.choice(np.arange(1, 8 * time_scale), size=n_windows, replace=False)).astype(np.int32)
    if rng.random() < 0.7:
        wins[0] = 0
    gaps = rng.integers(0, 12 * time_scale, size=n_arrivals).astype(np.int64)
    gaps[rng.random(n_arrivals) < zero_gap_p] = 0
    big = rng.random(n_arrivals) < 0.1
    gaps[big] = rng.integers(10**6, 10**8, size=int(big.sum()))
    gaps[0] = int(rng.integers(0, 10**6))
    arr = np.cumsum(gaps)
    if sla_us is None:
        sla_us = int(rng.integers(2 * time_scale, 30 * time_scale))
    return Problem(name="random", pred_ptr=ptr, pred_idx=idx, n_configs=ncfg,
                   exec_us=ex, init_us=ini, price_per_us=price, arrivals_us=arr.astype(np.int64),
                   sla_us=int(sla_us), windows_us=wins)
