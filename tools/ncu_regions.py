"""Dev tool: instruction / stall shares of an ncu report aggregated over line ranges.
usage: ncu_regions.py REP file.cu:a-b=name ..."""
import collections
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
regions = []
for arg in sys.argv[2:]:
    loc, name = arg.split("=")
    f, r = loc.split(":")
    a, b = map(int, r.split("-"))
    regions.append((f, a, b, name))
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"], capture_output=True,
                     text=True).stdout
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
            res.append((int(d["Instructions Executed"] or 0), int(d["Warp Stall Sampling (All Samples)"] or 0), cur, int(r[0])))
        except ValueError:
            pass
ti = sum(x[0] for x in res) or 1
ts = sum(x[1] for x in res) or 1
agg = collections.Counter()
st = collections.Counter()
for n, s, f, ln in res:
    name = f
    for (rf, a, b, nm) in regions:
        if rf == f and a <= ln <= b:
            name = nm
            break
    agg[name] += n
    st[name] += s
for k, v in agg.most_common():
    print(f"{k:28s} inst {100 * v / ti:5.1f}%  stall {100 * st[k] / ts:5.1f}%")
