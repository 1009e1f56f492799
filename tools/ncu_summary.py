"""Dev tool: summarise an ncu report (key metrics + top source lines by stall samples)."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
ntop = int(sys.argv[2]) if len(sys.argv) > 2 else 25
KEYS = ["Duration", "Elapsed Cycles", "Compute (SM) Throughput", "Memory Throughput", "DRAM Throughput",
        "L2 Cache Throughput", "Executed Ipc Active", "Issue Slots Busy", "Registers Per Thread",
        "Achieved Occupancy", "Theoretical Occupancy", "Warp Cycles Per Issued Instruction",
        "Avg. Active Threads Per Warp", "Executed Instructions", "L2 Hit Rate", "Dynamic Shared Memory Per Block",
        "Block Limit Registers", "Block Limit Shared Mem", "Grid Size"]
out = subprocess.run(["ncu", "-i", rep, "--page", "details", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[0]
kern = None
for r in rows[1:]:
    d = dict(zip(h, r))
    if kern != d.get("Kernel Name"):
        kern = d.get("Kernel Name")
        print("##", kern[:120])
    if d.get("Metric Name") in KEYS:
        print(f"  {d['Metric Name']:<40} {d['Metric Value']:>16} {d['Metric Unit']}")
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rr = list(csv.reader(io.StringIO(raw)))
if len(rr) > 2:
    hh, units, vals = rr[0], rr[1], rr[2]
    for k in ("dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_sectors_op_atom.sum", "lts__t_sectors_op_red.sum",
              "sm__cycles_active.avg", "smsp__issue_active.avg.pct_of_peak_sustained_active",
              "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
              "gpu__time_duration.sum", "lts__t_sector_hit_rate.pct"):
        if k in hh:
            i = hh.index(k)
            print(f"  {k:<55} {vals[i]:>16} {units[i]}")
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
res, hdr, cur = [], None, None
for r in csv.reader(io.StringIO(src)):
    if r and r[0] == "File Path":
        cur = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        hdr = r
        continue
    if hdr and len(r) == len(hdr) and r[0].isdigit():
        d = dict(zip(hdr, r))
        try:
            res.append((int(d["Instructions Executed"] or 0), int(d["Warp Stall Sampling (All Samples)"] or 0), cur,
                        int(r[0]), r[1][:80]))
        except ValueError:
            pass
if res:
    ti = sum(x[0] for x in res) or 1
    ts = sum(x[1] for x in res) or 1
    print(f"  source: {ti} warp-instructions, {ts} stall samples")
    for x in sorted(res, key=lambda x: -x[1])[:ntop]:
        print(f"  {x[0] / ti * 100:5.1f}% inst {x[1] / ts * 100:5.1f}% stall  {x[2]}:{x[3]}  {x[4]}")
