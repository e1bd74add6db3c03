#!/usr/bin/env python
"""Top SASS instructions of an ncu capture by warp-stall samples, with the
instruction that produced the awaited value (scoreboard waits show up on the
consumer).  Usage: ncu_hot.py REP [N]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[1]
i_src, i_s = h.index("Source"), h.index("Warp Stall Sampling (All Samples)")
cols = [i for i, x in enumerate(h) if x.startswith("stall_") and "Not Issued" not in x]
body = rows[2:]
tot = sum(int(r[i_s]) for r in body if r[i_s].isdigit()) or 1
ranked = sorted(range(len(body)), key=lambda j: -int(body[j][i_s]) if body[j][i_s].isdigit() else 0)
for j in ranked[:N]:
    r = body[j]
    top = sorted(((h[i], int(r[i])) for i in cols if r[i].isdigit() and int(r[i]) > 0), key=lambda x: -x[1])[:2]
    prev = " | ".join(body[k][i_src].strip()[:40] for k in range(max(0, j - 2), j))
    print(f"{100 * int(r[i_s]) / tot:5.1f}%  {r[i_src].strip()[:60]:60s} {top}  <- {prev}")
