"""The paper's auto-scaler (Eq. (7)/(8)) by brute force -- TEST
INFRASTRUCTURE ONLY (the oracle of smiless_autoscale).

For each function: every configuration c and every batch size B in [1, G] with
slope_c * B + intercept_c <= I_s (Eq. (1)/(2) with the batch B) costs
ceil(G / B) * IT * U(c) (Eq. (7): (G / B) instances, whole instances -- reading G24);
the cheapest wins, ties to the lower configuration then the larger B.
"""
import math


def autoscale(prob, slope, intercept, invocations, it_us, target_us):
    off = [0]
    for m in prob.n_configs:
        off.append(off[-1] + int(m))
    out = []
    for k in range(prob.n_funcs):
        G = int(invocations[k])
        if G <= 0:
            out.append((-1, 0, 0, 0.0))
            continue
        best = (-1, 0, 0, math.inf)
        for c in range(int(prob.n_configs[k])):
            r = off[k] + c
            for B in range(G, 0, -1):                  # largest B first: fewest instances
                if float(slope[r]) * float(B) + float(intercept[r]) <= float(target_us[k]):
                    inst = -(-G // B)
                    cost = (float(inst) * float(it_us)) * float(prob.price_per_us[r])
                    if cost < best[3]:
                        best = (c, B, inst, cost)
                    break
        out.append(best)
    return out


def autoscale_rows(prob, slope, intercept, invocations, target_us):
    """Eq. (7)/(8) constraint per (function, configuration) row by brute force: the largest
    B in [1, G] with slope * B + intercept <= I_s, and ceil(G / B) instances; (0, 0) when
    even B = 1 misses I_s or G <= 0."""
    off = [0]
    for m in prob.n_configs:
        off.append(off[-1] + int(m))
    batch, inst = [], []
    for k in range(prob.n_funcs):
        G = int(invocations[k])
        for c in range(int(prob.n_configs[k])):
            r = off[k] + c
            best = 0
            for B in range(1, G + 1):
                if float(slope[r]) * float(B) + float(intercept[r]) <= float(target_us[k]):
                    best = B
            batch.append(best)
            inst.append(-(-G // best) if best else 0)
    return batch, inst
