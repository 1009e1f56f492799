"""Single runs of every workload pipeline for ncu launch lists and per-config captures.

  python tools/ncu_wl.py WL MODEL [--outer N] [--imgs N] [--runs R] [--timers]
    WL    : reyes1x | face8 | pyr | cfd | raster | raster_near | ldpc | qb4 | qb16 | qb272
    MODEL : kbk | mega | coarse | fine | tuned
Prints device ms per run and the per-kernel ms (stats).  Under ncu the kernels of one
run are serialised, so multi-group plans fall back to a megakernel rerun: profile the
per-stage kernels with `kbk` and the persistent path with `mega`."""
import argparse
import os
import sys

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
    p = W.PyramidPipeline(inputs.pyramid_images(a.imgs, 4096), **kw)
elif a.wl == "reyes1x":
    p = W.ReyesPipeline(inputs.reyes_config1(n_frames=256), **kw)
elif a.wl == "face8":
    p = W.FaceDetPipeline(inputs.face_scene(n_frames=8), **kw)
elif a.wl == "raster":
    p = W.RasterPipeline(inputs.raster_scene(), **kw)
elif a.wl == "raster_near":
    p = W.RasterPipeline(inputs.raster_near_scene(n=1 << 20, W=1920, H=1080, area_range=(0.5, 512.0)), **kw)
elif a.wl == "ldpc":
    p = W.LdpcPipeline(inputs.ldpc_scene(), **kw)
elif a.wl.startswith("qb"):
    ib = int(a.wl[2:])
    p = W.QBenchPipeline(1 << 20 if ib < 272 else 1 << 18, ib, 1, 99, **kw)  # chains (fan-out 1)
else:
    raise SystemExit(f"unknown workload {a.wl}")
model = {"kbk": vp.KBK, "mega": vp.MEGAKERNEL, "coarse": vp.COARSE, "fine": vp.FINE}.get(a.model)
if model is not None:
    p.configure(model)
else:
    p.p.autotune(time_budget_s=8.0, sm_granularity=8)
for r in range(a.runs):
    st = p.run()
    if isinstance(st, tuple):
        st = st[1]
torch.cuda.synchronize()
print(a.wl, a.model, "ms", round(st["device_ms"], 3), "deq", st["dequeued"][:6], "kernels", st.get("kernels"))
if a.timers:
    print("exec ms", [round(x / 1e6, 2) for x in st["stage_exec_ns"][:6]], "flush ms",
          [round(x / 1e6, 2) for x in st["stage_flush_ns"][:6]], "idle ms", [round(x / 1e6, 2) for x in st["kernel_idle_ns"][:4]])
