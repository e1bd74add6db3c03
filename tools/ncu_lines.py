#!/usr/bin/env python
"""Per CUDA source line aggregates of an ncu capture (needs -lineinfo and
--import-source on): warp-stall samples, instructions executed, L2 sectors.
Usage: ncu_lines.py REP [N] [sort: stall|inst|sect]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 30
key = sys.argv[3] if len(sys.argv) > 3 else "stall"
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=cuda,sass"],
                     capture_output=True, text=True).stdout
rows, hdr, f = [], None, ""
for r in csv.reader(io.StringIO(out)):
    if not r:
        continue
    if r[0] == "File Path":
        f = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or len(r) != len(hdr) or r[2] != "-":
        continue  # only the per-line aggregate rows (address "-")
    try:
        s = int(r[4])
    except ValueError:
        continue
    def num(name):
        try:
            return float(r[hdr.index(name)])
        except (ValueError, IndexError):
            return 0.0
    st = sorted(((hdr[i][6:], int(r[i])) for i, x in enumerate(hdr) if x.startswith("stall_") and "Not Issued" not in x
                 and r[i].isdigit() and int(r[i]) > 0), key=lambda x: -x[1])[:2]
    rows.append(dict(stall=s, inst=num("Instructions Executed"), sect=num("L2 Theoretical Sectors Global"),
                     where=f"{f}:{r[0]}", src=r[1].strip(), top=st))
tot = {k: sum(x[k] for x in rows) or 1 for k in ("stall", "inst", "sect")}
print(f"totals: stall samples {tot['stall']:.4g}, warp instructions {tot['inst']:.4g}, L2 sectors {tot['sect']:.4g}")
for x in sorted(rows, key=lambda x: -x[key])[:N]:
    print(f"st {100 * x['stall'] / tot['stall']:5.1f}%  in {100 * x['inst'] / tot['inst']:5.1f}%  "
          f"sec {100 * x['sect'] / tot['sect']:5.1f}%  {x['where']:>22} {x['src'][:64]:64s} {x['top']}")
