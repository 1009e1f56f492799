"""Dev: print gpurun_out/ab.txt (tools/gpu_ab.sh) compactly."""
import json
import sys
for l in open(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/ab.txt"):
    if l.startswith("=="):
        print(l.strip())
        continue
    try:
        d = json.loads(l)
        print(" ", d["cfg"], round(d["ms"], 3), d["kernel_ms"])
    except Exception:
        print(" ", l.strip()[:200])
