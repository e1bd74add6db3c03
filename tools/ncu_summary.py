#!/usr/bin/env python
"""Summarise the round's ncu captures into profiles/ (text + JSON)."""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
WANT = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "lts__t_sector_hit_rate.pct", "l1tex__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "launch__shared_mem_per_block_dynamic", "smsp__inst_executed.sum",
        "lts__t_sectors_srcunit_tex_op_atom.sum", "lts__t_sectors_srcunit_tex_op_read.sum",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active"]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, u, v = rows[0], rows[1], rows[2]
    return {h[i]: (v[i], u[i]) for i in range(len(h))}


def stalls(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h = rows[1]
    cols = [i for i, x in enumerate(h) if x.startswith("stall_") and "Not Issued" not in x]
    agg = {}
    for r in rows[2:]:
        for i in cols:
            try:
                agg[h[i]] = agg.get(h[i], 0) + int(r[i])
            except ValueError:
                pass
    tot = sum(agg.values()) or 1
    return {k: round(100 * v / tot, 1) for k, v in sorted(agg.items(), key=lambda x: -x[1])[:8]}


def main():
    rnd = sys.argv[1] if len(sys.argv) > 1 else "r01"
    src = os.path.join(ROOT, "gpurun_out")
    summary, lines = {}, []
    for cfg in ("road", "rmat", "er", "batch"):
        rep = os.path.join(src, f"{rnd}_full_{cfg}.ncu-rep")
        if not os.path.exists(rep):
            continue
        m = raw(rep)
        get = lambda k: float(m[k][0]) if k in m else None  # noqa: E731
        unit = lambda k: m[k][1] if k in m else ""  # noqa: E731
        scale = {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1.0}
        rd = get("dram__bytes_read.sum") * scale.get(unit("dram__bytes_read.sum"), 1)
        wr = get("dram__bytes_write.sum") * scale.get(unit("dram__bytes_write.sum"), 1)
        st = stalls(rep)
        shape = lambda k: int(float(m[k][0])) if k in m else None  # noqa: E731
        summary[cfg] = {"block": shape("launch__block_size"), "grid": shape("launch__grid_size"), "round": rnd,
                        "dram_bytes_per_launch": rd + wr, "dram_read": rd, "dram_write": wr,
                        "duration_ms_under_ncu": get("gpu__time_duration.sum"),
                        "metrics": {k: m[k][0] + " " + m[k][1] for k in WANT if k in m}, "stalls_pct": st}
        lines.append(f"== {cfg}: persistent kernel, one launch, ncu --set full ({rnd})")
        for k in WANT:
            if k in m:
                lines.append(f"  {k:60s} {m[k][0]:>16s} {m[k][1]}")
        lines.append(f"  dram read+write per launch: {(rd + wr) / 1e9:.3f} GB")
        lines.append("  top stall reasons (% of samples): " + ", ".join(f"{k}={v}" for k, v in st.items()))
    # launch list: share of the persistent kernel in the step
    lc = os.path.join(src, f"{rnd}_launches.csv")
    if os.path.exists(lc):
        rows = [r for r in csv.reader(open(lc)) if len(r) > 10]
        h = rows[0]
        ik, iv = h.index("Kernel Name"), h.index("Metric Value")
        per = {}
        for r in rows[1:]:
            name = r[ik].split("(")[0].split("<")[0].replace("void ", "").strip()
            per.setdefault(name, []).append(float(r[iv].replace(",", "")))
        tot = sum(sum(v) for v in per.values())
        lines.append(f"== launch list of `bench.py --steps 1 --warmup 3` (default workload), ncu gpu__time_duration ({rnd})")
        share = {}
        for k, v in sorted(per.items(), key=lambda x: -sum(x[1])):
            share[k] = {"launches": len(v), "total_ns": sum(v), "share": sum(v) / tot}
            lines.append(f"  {k:45s} launches={len(v):3d} total={sum(v) / 1e6:9.3f} ms share={100 * sum(v) / tot:5.1f}%")
        summary["launch_list"] = share
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    with open(os.path.join(ROOT, "profiles", f"{rnd}_ncu_summary.txt"), "w") as f:
        f.write("\n".join(lines) + "\n")
    with open(os.path.join(ROOT, "profiles", "ncu_summary.json"), "w") as f:
        json.dump(summary, f, indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
