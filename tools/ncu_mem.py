#!/usr/bin/env python
"""Global-memory instructions of an ncu capture ranked by L2 theoretical sectors
(source page, SASS), with executions and the CUDA source line (-lineinfo).
Usage: ncu_mem.py REP [N]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 30


def page(extra):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", *extra], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return rows[1], rows[2:]


h, body = page(["--print-source=sass"])
ix = {k: h.index(k) for k in ("Address", "Source", "Instructions Executed", "L2 Theoretical Sectors Global",
                              "L2 Theoretical Sectors Global Excessive", "Warp Stall Sampling (All Samples)")}


def num(r, k):
    try:
        return float(r[ix[k]])
    except ValueError:
        return 0.0


mem = [r for r in body if num(r, "L2 Theoretical Sectors Global") > 0]
tot = sum(num(r, "L2 Theoretical Sectors Global") for r in mem) or 1
print(f"total L2 theoretical sectors (global): {tot:.4g}")
for r in sorted(mem, key=lambda r: -num(r, "L2 Theoretical Sectors Global"))[:N]:
    s = num(r, "L2 Theoretical Sectors Global")
    print(f"{100 * s / tot:5.1f}%  sect={s:10.4g} exc={num(r, 'L2 Theoretical Sectors Global Excessive'):9.3g} "
          f"inst={num(r, 'Instructions Executed'):9.3g}  {r[ix['Source']].strip()[:80]}")
