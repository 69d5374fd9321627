#!/usr/bin/env python
"""Mutation check of the oracle pins: copy the repo's test inputs, apply one plausible
mistake to oracle/ at a time, run the -m "not gpu" pins against the mutated copy, and
report which pins turn red.  A mutation no pin catches is a gap in the pins.

    python tools/mutation_check.py [--out profiles/r02_oracle_mutations.md]
"""
import argparse
import re
import os
import shutil
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

# (name, file, old text, new text)
MUTATIONS = [
    ("top1: layer 1 starts at the cheapest config (P:210 says second cheapest)", "oracle/top1.py",
     "range(1 if k == 0 else 0, M[k])", "range(0, M[k])"),
    ("top1: later functions on the cheapest instead of the fastest config", "oracle/top1.py",
     "[fastest[q] for q in range(k + 1, n)]", "[rank[q][0] for q in range(k + 1, n)]"),
    ("top1: rank by price only, not U*(T+I) / U*IT", "oracle/top1.py",
     "costs.append((float(prob.price_per_us[r]) * per_inv, m))", "costs.append((float(prob.price_per_us[r]), m))"),
    ("decompose: F_s/F_e take the slowest of their paths' choices", "oracle/decompose.py",
     "if cfg[k] < 0 or I(k, m) < I(k, cfg[k]):", "if cfg[k] < 0 or I(k, m) > I(k, cfg[k]):"),
    ("decompose: branch functions not re-chosen after combining", "oracle/decompose.py",
     "            if n_on[k] != 1:\n                continue", "            if True:\n                continue"),
    ("decompose (model M): F_s/F_e take the slowest of their paths' choices", "oracle/decompose_m.py",
     "if cfg[k] < 0 or prob.exec_us[off[k] + c[q]] < prob.exec_us[off[k] + cfg[k]]:",
     "if cfg[k] < 0 or prob.exec_us[off[k] + c[q]] > prob.exec_us[off[k] + cfg[k]]:"),
    ("decompose (model M): no re-choice of branch functions", "oracle/decompose_m.py",
     "            if n_on[k] != 1:\n                continue\n            R =", "            if True:\n                continue\n            R ="),
    ("decompose (model M): re-choice may raise the path latency", "oracle/decompose_m.py",
     "if lat[d] <= pl and (best is None or cost[d] < cost[best]):", "if (best is None or cost[d] < cost[best]):"),
    ("scale-out: previous completion from request j-1 instead of j-n_k", "oracle/smiless_oracle.c",
     "int64_t f = D[(int64_t)k * J + (j - n_inst[k])];", "int64_t f = D[(int64_t)k * J + (j - 1)];"),
    ("autoscale: ties go to the higher configuration", "oracle/autoscale.py",
     "if cost < best[3]:", "if cost <= best[3]:"),
    ("autoscale: smallest feasible batch instead of the largest", "oracle/autoscale.py",
     "for B in range(G, 0, -1):", "for B in range(1, G + 1):"),
    ("autoscale: fractional instances G/B", "oracle/autoscale.py",
     "inst = -(-G // B)", "inst = G / B"),
    ("cost_of: product fused into the running sum (FMA)", "oracle/smiless_oracle.c",
     "        cost = cost + term;", "        cost = __builtin_fma(u, (double)billed[k], cost); (void)term;"),
    ("cost_of: summed right to left", "oracle/smiless_oracle.c",
     "    for (int k = 0; k < P->n_funcs; ++k) {\n        double u = P->price_per_us[row0(P, k) + config[k]];",
     "    for (int k = P->n_funcs - 1; k >= 0; --k) {\n        double u = P->price_per_us[row0(P, k) + config[k]];"),
    ("model M: the +I of billing dropped", "oracle/smiless_oracle.c",
     "billed[k] += bill + I[k];", "billed[k] += bill;"),
    ("model M: arrival during init counted as covered (G4 boundary)", "oracle/smiless_oracle.c",
     "} else if (x < s + T[k]) {", "} else if (x < s) {"),
    ("model M: first invocation cold instead of pre-warmed (G5)", "oracle/smiless_oracle.c",
     "                start = x;\n                bill = T[k];", "                start = x + T[k];\n                bill = T[k];"),
]

COPY = ["oracle", "tests", "workloads", "paper_conf_sc_luxl0y024_b200", "include", "pytest.ini", "bench.py"]


def run_one(mut, tmp):
    name, path, old, new = mut
    dst = os.path.join(tmp, "r")
    if os.path.exists(dst):
        shutil.rmtree(dst)
    os.makedirs(dst)
    for c in COPY:
        s = os.path.join(ROOT, c)
        d = os.path.join(dst, c)
        if os.path.isdir(s):
            shutil.copytree(s, d, ignore=shutil.ignore_patterns("__pycache__", "liboracle.so*", "generated"))
        else:
            shutil.copy2(s, d)
    f = os.path.join(dst, path)
    src = open(f).read()
    assert src.count(old) == 1, (name, src.count(old))
    open(f, "w").write(src.replace(old, new))
    r = subprocess.run([sys.executable, "-m", "pytest", "tests/test_oracle_pins.py", "-q", "-m", "not gpu",
                        "-p", "no:cacheprovider", "--tb=no", "-rf"],
                       cwd=dst, capture_output=True, text=True, timeout=1800)
    failed = [ln.split(" ")[1].split("::")[-1] for ln in r.stdout.splitlines() if ln.startswith("FAILED")]
    return r.returncode, failed


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r02_oracle_mutations.md"))
    args = ap.parse_args()
    rows = []
    with tempfile.TemporaryDirectory() as tmp:
        for mut in MUTATIONS:
            rc, failed = run_one(mut, tmp)
            caught = rc != 0 and failed
            failed = [re.sub(r"\[/.*/tests/golden/", "[", f) for f in failed]
            rows.append((mut[0], mut[1], "caught" if caught else "SURVIVED", ", ".join(failed[:6])))
            print(rows[-1], flush=True)
    with open(args.out, "w") as fo:
        fo.write("# Oracle mutation check (tools/mutation_check.py)\n\n")
        fo.write("Each row applies one plausible mistake to a copy of `oracle/` and runs "
                 "`tests/test_oracle_pins.py -m \"not gpu\"` against it.\n\n")
        fo.write("| mutation | file | result | pins that turned red |\n|---|---|---|---|\n")
        for r in rows:
            fo.write("| %s | `%s` | %s | %s |\n" % r)
    return 0 if all(r[2] == "caught" for r in rows) else 1


if __name__ == "__main__":
    sys.exit(main())
