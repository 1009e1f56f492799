"""Summarise the ncu launch lists of tools/profile_suite.sh: per (workload, model, kernel)
the summed time, DRAM bytes and GB/s (% of the measured HBM peak), L2 atomic + reduction
sectors per second, and time-weighted issue-slot / warp occupancy."""
import collections
import csv
import glob
import json
import os
import sys

d = sys.argv[1]
root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
try:
    hbm = json.load(open(os.path.join(root, "MEASURED_PEAKS.json"))).get("hbm_gbs", 6548.5)
except Exception:
    hbm = 6548.5
print(f"HBM peak (MEASURED_PEAKS.json): {hbm:.1f} GB/s")
for f in sorted(glob.glob(os.path.join(d, "*.csv"))):
    lines = open(f).read().splitlines()
    try:
        i = [k for k, l in enumerate(lines) if l.startswith('"ID"')][0]
    except IndexError:
        print(f"## {os.path.basename(f)}: no launches")
        continue
    rows = list(csv.reader(lines[i:]))
    h = rows[0]
    per = collections.defaultdict(dict)
    for r in rows[1:]:
        x = dict(zip(h, r))
        try:
            per[(x["ID"], x["Kernel Name"])][x["Metric Name"]] = float(x["Metric Value"].replace(",", ""))
        except ValueError:
            pass
    agg = collections.OrderedDict()
    for (_, name), m in per.items():
        short = name.split("(")[0].replace("void ", "").replace("vp::", "")[:48]
        a = agg.setdefault(short, collections.Counter())
        t = m.get("gpu__time_duration.sum", 0.0)
        a["n"] += 1
        a["ns"] += t
        a["bytes"] += m.get("dram__bytes_read.sum", 0.0) + m.get("dram__bytes_write.sum", 0.0)
        a["atom"] += m.get("lts__t_sectors_op_atom.sum", 0.0)
        a["red"] += m.get("lts__t_sectors_op_red.sum", 0.0)
        a["issue_w"] += t * m.get("smsp__issue_active.avg.pct_of_peak_sustained_active", 0.0)
        a["warps_w"] += t * m.get("sm__warps_active.avg.pct_of_peak_sustained_active", 0.0)
    print(f"## {os.path.basename(f)[:-4]}")
    print(f"  {'kernel':48s} {'n':>4s} {'ms':>8s} {'MB':>8s} {'GB/s':>7s} {'%HBM':>5s} {'atom+red/s':>10s} {'issue%':>6s} {'warps%':>6s}")
    for k, a in agg.items():
        if a["ns"] < 2000:
            continue
        s = a["ns"] / 1e9
        gbs = a["bytes"] / a["ns"] if a["ns"] else 0.0
        print(f"  {k:48s} {int(a['n']):4d} {a['ns'] / 1e6:8.3f} {a['bytes'] / 1e6:8.1f} {gbs:7.0f} {100 * gbs / hbm:5.1f} "
              f"{(a['atom'] + a['red']) / s:10.3e} {a['issue_w'] / a['ns']:6.1f} {a['warps_w'] / a['ns']:6.1f}")
