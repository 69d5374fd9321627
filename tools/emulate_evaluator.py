#!/usr/bin/env python
"""Step-by-step CPU emulation of the evaluator kernel's arithmetic (debugging aid only).

Mirrors paper_conf_sc_luxl0y024_b200/csrc/evaluator.cuh for ONE lane-unit (upstream
prefix x all W windows of the last function): chunk-relative clamped offsets, negated
time, the busy mask, the shared per-lane offset C, rebase, telescoped billing.  It
asserts every intermediate fits in int32 (the int32 path's range rule).  Not used by
the product or by the tests; compare its output with oracle/ when a GPU parity test
fails.
"""
import numpy as np

I32 = (-(1 << 31), (1 << 31) - 1)


def chk(v):
    assert I32[0] <= v <= I32[1], v
    return v


def emulate_unit(p, digits, c_last, K, sla):
    """digits: full digits (c*W + w) of functions 0..N-2; c_last: config of N-1.
    Returns per window v: (feasible, billed list) like the kernel computes."""
    N = p.n_funcs
    Wn = len(p.windows_us)
    row0 = np.concatenate([[0], np.cumsum(p.n_configs)])
    r = [int(v) for v in p.arrivals_us]
    J = len(r)
    T = [int(v) for v in p.init_us]
    I = [int(v) for v in p.exec_us]
    wmax = int(p.windows_us[-1])
    d_cap = sla + wmax + max(T) + 1
    # offsets (prep_offsets_kernel)
    n_steps = J - 1
    off = []
    for s in range(n_steps):
        if s % K == 0:
            acc = 0
        acc += min(r[s + 1] - r[s], d_cap)
        off.append(acc)
    preds = [p.preds(k) for k in range(N)]
    listed = set(int(v) for v in p.pred_idx)
    sinks_up = [k for k in range(N - 1) if k not in listed]
    NI, Te, Wk, Tk, rows = [], [], [], [], []
    for k in range(N - 1):
        row = row0[k] + digits[k] // Wn
        w = int(p.windows_us[digits[k] % Wn])
        rows.append(row)
        NI.append(-I[row]); Wk.append(w); Te.append(0 if w == 0 else T[row]); Tk.append(T[row])
    rowL = row0[N - 1] + c_last
    IL, TL = I[rowL], T[rowL]
    # j = 0
    NF = [0] * (N - 1)
    st0 = [0] * N
    nlu = (1 << 31) - 1
    for k in range(N - 1):
        x = 0 if not preds[k] else -min(NF[q] for q in preds[k])
        st0[k] = x
        NF[k] = NI[k] - x
    xl = 0 if not preds[N - 1] else -min(NF[q] for q in preds[N - 1])
    for k in sinks_up:
        nlu = min(nlu, NF[k])
    st0[N - 1] = xl
    C = 0
    Q = [-xl - IL] * Wn
    NLM = list(Q)
    SU = [0] * (N - 1)
    SUL = [0] * Wn
    acc = [0] * (N - 1 + Wn)
    w0zero = int(p.windows_us[0]) == 0

    def step(o):
        nonlocal xl, nlu, C
        for k in range(N - 1):
            if not preds[k]:
                g = chk(o + NF[k])
            else:
                g = chk(NF[k] - min(NF[q] for q in preds[k]))
            u = max(min(g, Wk[k]), 0)
            dl = chk(max(u + Te[k], g))
            m = -1 if g > 0 else 0
            NF[k] = chk(NF[k] + NI[k] + dl * m)
            SU[k] = chk(SU[k] + u)
        xl = o if not preds[N - 1] else -min(NF[q] for q in preds[N - 1])
        for k in sinks_up:
            nlu = min(NF[k] + o, nlu)
        xc = chk(xl - C)
        C = chk(C + IL)
        oc = chk(o - C)
        for v in range(Wn):
            g = xc + Q[v]
            if w0zero and v == 0:
                Q[v] = Q[v] - max(g, 0)
            else:
                u = max(min(g, int(p.windows_us[v])), 0)
                dl = max(u + TL, g)
                Q[v] = Q[v] + dl * (-1 if g > 0 else 0)
                SUL[v] += u
            NLM[v] = min(Q[v] + oc, NLM[v])

    def rebase(sh):
        nonlocal C
        for k in range(N - 1):
            NF[k] += sh
        d = sh - C
        for v in range(Wn):
            Q[v] += d
        C = 0

    def flush():
        for k in range(N - 1):
            acc[k] += SU[k]; SU[k] = 0
        for v in range(Wn):
            acc[N - 1 + v] += SUL[v]; SUL[v] = 0

    nfc = n_steps // K
    for qc in range(nfc):
        if qc > 0:
            rebase(off[qc * K - 1])
        for t in range(K):
            step(off[qc * K + t])
        flush()
    t0 = nfc * K
    if t0 < n_steps:
        if nfc > 0:
            rebase(off[t0 - 1])
        for s in range(t0, n_steps):
            step(off[s])
        flush()
    o_last = off[n_steps - 1] if n_steps else 0
    R = r[-1] - r[0]
    billed_up = [Tk[k] - NF[k] - o_last + R - st0[k] - acc[k] for k in range(N - 1)]
    out = []
    for v in range(Wn):
        FLv = C - Q[v]
        b = TL + FLv - o_last + R - st0[N - 1] - acc[N - 1 + v]
        feas = nlu >= -sla and NLM[v] >= -sla
        out.append((feas, billed_up + [b], -min(NLM[v], nlu)))
    return out
