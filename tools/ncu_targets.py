"""Dev tool: single-kernel launches of the hot path for `ncu` (which serialises kernels,
so co-running persistent groups cannot be captured together).

  mega      : the whole Reyes pipeline as one megakernel (config 5 shape, --frames)
  rtc_dice  : the [Dice,Shade] RTC kernel alone: every seed patch is inserted into the
              Dice queue, the [Bound,Split] group is an (idle) KBK group
  kbk       : one launch per stage per wave
  raster_{mega,kbk}, raster_near_{mega,kbk} : config 4 / the near-clip raster workload
  bs_mega   : the block-local [Bound,Split] megakernel alone (Dice items left in a full ring)
  bs_online : the tuned hybrid ([Bound,Split] block-local recursion on 60 SMs | [Dice,Shade]
              RTC on 88) with online retirement: under ncu's serialisation the [Bound,Split]
              grid runs alone, parks every Dice item in a full-size ring and retires, then
              the RTC grid drains them -- so the first vp_kernel launch is the Bound/Split
              kernel exactly as the bench runs it
  rtc_leaf  : the [Dice,Shade] RTC kernel alone on representative leaf patches
              (tools/reyes_leaves.py: numpy approximation of the Bound/Split recursion)
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch

from paper_conf_micro_zhengozsyc17_b200 import inputs, vp
from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline

ap = argparse.ArgumentParser()
ap.add_argument("target")
ap.add_argument("--frames", type=int, default=64)
ap.add_argument("--runs", type=int, default=2)
ap.add_argument("--l2", action="store_true", help="VP_FLAG_L2_PERSIST")
args = ap.parse_args()

nsm, _ = vp.device_info(0)
if args.target.startswith("raster"):
    from paper_conf_micro_zhengozsyc17_b200.workloads import RasterPipeline
    scene = (inputs.raster_near_scene(n=1 << 20, W=1920, H=1080, area_range=(0.5, 512.0))
             if args.target.startswith("raster_near") else inputs.raster_scene())
    rp = RasterPipeline(scene)
elif args.target == "bs_mega":
    scene = inputs.reyes_config5(n_frames=args.frames)
    rp = ReyesPipeline(scene, flags=vp.FLAG_FULL_RINGS)
elif args.target == "bs_online":
    scene = inputs.reyes_config5(n_frames=args.frames)
    rp = ReyesPipeline(scene, flags=vp.FLAG_FULL_RINGS | vp.FLAG_ONLINE, queue_caps=[1 << 20, 1 << 16, 1 << 21, 1 << 12])
else:
    scene = inputs.reyes_config5(n_frames=args.frames)
    rp = ReyesPipeline(scene, flags=vp.FLAG_L2_PERSIST if args.l2 else 0)
if args.target in ("raster_mega", "raster_near_mega"):
    rp.configure(vp.MEGAKERNEL)
elif args.target in ("raster_kbk", "raster_near_kbk"):
    rp.configure(vp.KBK)
elif args.target == "mega":
    rp.configure(vp.MEGAKERNEL)
elif args.target == "kbk":
    rp.configure(vp.KBK)
elif args.target == "bs_mega":
    # the block-local [Bound, Split] kernel alone (its Dice items wait in a full-size ring
    # for the KBK [Dice, Shade] waves that run after it under ncu's serialisation)
    rp.configure(vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_MEGA, 0, nsm - 8), (2, 3, vp.GROUP_KBK, nsm - 8, nsm)], nsm))
elif args.target == "bs_online":
    rp.configure(vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_MEGA, 0, 60), (2, 3, vp.GROUP_RTC, 60, nsm)], nsm))
elif args.target == "rtc_dice":
    rp.p.insert(0, rp.seeds_dev, n=0, replace=True)
    rp.p.insert(2, rp.seeds_dev, n=scene.seeds.size)
    rp.configure(vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_KBK, 0, 8), (2, 3, vp.GROUP_RTC, 8, nsm)], nsm))
elif args.target == "rtc_leaf":
    import numpy as np
    sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
    import reyes_leaves
    lv = np.ascontiguousarray(inputs.gpu_patch_items(reyes_leaves.leaves(scene, args.frames)))  # 208-B items
    leaves_dev = torch.from_numpy(lv.view(np.uint8).reshape(-1)).cuda()
    rp.p.insert(0, rp.seeds_dev, n=0, replace=True)
    rp.p.insert(2, leaves_dev, n=lv.size)
    rp.configure(vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_KBK, 0, 8), (2, 3, vp.GROUP_RTC, 8, nsm)], nsm))
else:
    raise SystemExit(f"unknown target {args.target}")
for _ in range(args.runs):
    st = rp.run()
torch.cuda.synchronize()
print(args.target, st["device_ms"], st["dequeued"][:4], st["kernels"])
