#!/usr/bin/env python
"""Per-kernel warp-stall breakdown (share of all warp samples) from an ncu report's source page.

    python tools/ncu_stalls.py gpurun_out/X_prof.ncu-rep smiless_variants_kernel
"""
import collections
import csv
import io
import subprocess
import sys


def stalls(rep, kernel):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass", "-k", kernel],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr = rows[1]
    ix = {h: i for i, h in enumerate(hdr)}
    cols = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
    agg = collections.Counter()
    for r in rows[2:]:
        if len(r) != len(hdr):
            continue
        for c in cols:
            agg[c] += int(r[ix[c]] or 0)
    tot = sum(agg.values()) or 1
    return {c[6:]: round(v / tot, 3) for c, v in agg.most_common() if v}


if __name__ == "__main__":
    print(stalls(sys.argv[1], sys.argv[2]))
