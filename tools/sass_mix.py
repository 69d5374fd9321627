#!/usr/bin/env python
"""Static pipe mix of the memoised variants kernel's innermost loop (NVRTC on the CPU, no
GPU): instructions per loop iteration split by pipe, and the resulting per-warp cycle
bounds on one SMSP (issue: 1 instruction/clk; ALU and FMA-heavy pipes: 16 lanes/clk, i.e.
2 clk per warp instruction; IMAD.HI: 4 clk).

    SMILESS_FMASK=0xfe python tools/sass_mix.py
"""
import os
import re
import subprocess
import sys
import tempfile
from collections import Counter

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

ALU = ("VIMNMX", "VIADDMNMX", "IADD3", "ISETP", "SEL", "LOP3", "SHF", "VIADD", "IMNMX", "FSEL", "PRMT", "LEA")


def loop_body(name="smiless_variants_kernel", workload="C2"):
    import bench
    from paper_conf_sc_luxl0y024_b200 import smiless as S
    p, kw = bench.workload(workload)
    pl = S.planner_for(p)
    log, cubin = pl.jit_compile(p.arrivals_us, p.sla_us, p.windows_us, want_cubin=True, flags=S.FLAG_NO_PRUNE, **kw)
    with tempfile.NamedTemporaryFile(suffix=".cubin") as f:
        f.write(cubin)
        f.flush()
        sass = subprocess.run(["cuobjdump", "-sass", f.name], capture_output=True, text=True, check=True).stdout
    funcs, cur = {}, None
    for line in sass.split("\n"):
        m = re.search(r"Function : (\w+)", line)
        if m:
            cur = funcs.setdefault(m.group(1), [])
            continue
        m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(.*?);", line)
        if m and cur is not None:
            cur.append((int(m.group(1), 16), m.group(2)))
    ins = funcs[name]
    loops = []
    for addr, txt in ins:
        m = re.search(r"BRA(?:\.\w+)*\s+(?:!?U?P\w+,\s*)?0x([0-9a-f]+)", txt)
        if m and int(m.group(1), 16) < addr:
            loops.append((int(m.group(1), 16), addr))
    # the hot loop: the innermost loop holding a 4-step body (>= 32 VIADDMNMX: 16 variants x 2
    # per step... at least two steps' worth)
    def n_dpx(l):
        return sum("VIADDMNMX" in t for a, t in ins if l[0] <= a <= l[1])
    # the main loop walks 4 steps per iteration (>= 4 x 16 min/max of the variants); the
    # one-step tail loop is what remains below that
    big = [l for l in loops if n_dpx(l) >= 100]
    best = min(big or [l for l in loops if n_dpx(l) >= 32], key=lambda l: l[1] - l[0])
    body = [t for a, t in ins if best[0] <= a <= best[1]]
    return body, log


def classify(body):
    c = Counter()
    for t in body:
        op = re.sub(r"^@!?U?P\w+\s+", "", t).split()[0]
        base = op.split(".")[0]
        if op.startswith("IMAD.HI"):
            c["fma_quarter"] += 1
        elif base in ("IMAD",):
            c["fma"] += 1
        elif base in ALU:
            c["alu"] += 1
        else:
            c["other:" + base] += 1
    return c


def main():
    body, log = loop_body()
    c = classify(body)
    n = len(body)
    alu, fma, q = c["alu"], c["fma"], c["fma_quarter"]
    print({"instructions": n, **c})
    print("cycles/iteration: issue %d, ALU %d, FMA-heavy %d -> bound %d (issue frac ceiling %.3f)" % (
        n, 2 * alu, 2 * fma + 4 * q, max(n, 2 * alu, 2 * fma + 4 * q), n / max(n, 2 * alu, 2 * fma + 4 * q)))
    spill = [l for l in log.splitlines() if "spill" in l]
    print(spill[:3])


if __name__ == "__main__":
    main()
