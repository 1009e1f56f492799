"""Dev tool: single runs of the CFD / pyramid / facedet pipelines for ncu and timing.

  python tools/ncu_wl.py cfd kbk|mega|tuned [--outer N] [--runs R]
  python tools/ncu_wl.py pyr kbk|mega [--imgs N]
Prints device ms per run and the per-kernel ms (stats)."""
import argparse, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_micro_zhengozsyc17_b200 import inputs, vp
from paper_conf_micro_zhengozsyc17_b200 import workloads as W

ap = argparse.ArgumentParser()
ap.add_argument("wl")
ap.add_argument("model")
ap.add_argument("--outer", type=int, default=1)
ap.add_argument("--imgs", type=int, default=32)
ap.add_argument("--runs", type=int, default=1)
ap.add_argument("--timers", action="store_true")
a = ap.parse_args()
kw = dict(flags=vp.FLAG_TIMERS) if a.timers else {}
if a.wl == "cfd":
    p = W.CfdPipeline(inputs.cfd_scene(G=4096, n_outer=a.outer), **kw)
elif a.wl == "pyr":
    p = W.PyramidPipeline(inputs.pyramid_images(a.imgs, 4096), **kw) if hasattr(W, "PyramidPipeline") else None
else:
    raise SystemExit("wl")
model = {"kbk": vp.KBK, "mega": vp.MEGAKERNEL, "coarse": vp.COARSE, "fine": vp.FINE}.get(a.model)
if model is not None:
    p.configure(model)
else:
    p.p.autotune(time_budget_s=8.0, sm_granularity=8)
for r in range(a.runs):
    st = p.run()
torch.cuda.synchronize()
print(a.wl, a.model, "ms", round(st["device_ms"], 3), "deq", st["dequeued"][:4], "kernels", st.get("kernels"))
if a.timers:
    print("exec ms", [round(x / 1e6, 2) for x in st["stage_exec_ns"][:4]], "flush ms", [round(x / 1e6, 2) for x in st["stage_flush_ns"][:4]],
          "idle ms", [round(x / 1e6, 2) for x in st["kernel_idle_ns"][:4]])
