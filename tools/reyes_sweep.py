"""Dev tool: time the Reyes batch under several execution models / SM splits with the
in-kernel timers on, print a per-stage breakdown (exec / publish / idle)."""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np
import torch

from paper_conf_micro_zhengozsyc17_b200 import inputs, vp
from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline

ap = argparse.ArgumentParser()
ap.add_argument("--frames", type=int, default=512)
ap.add_argument("--reps", type=int, default=3)
ap.add_argument("--configs", default="mega,kbk,h37,h50,h74,h100,fine_h")
ap.add_argument("--batch", type=int, default=0)
ap.add_argument("--bats", default="", help="per-stage batch sets for hybrid configs, e.g. 32,16,8,4;32,16,64,4")
ap.add_argument("--no-timers", action="store_true")
ap.add_argument("--online", action="store_true", help="VP_FLAG_ONLINE (retire + refill)")
ap.add_argument("--l2", action="store_true", help="VP_FLAG_L2_PERSIST (persisting window over the sequence words)")
args = ap.parse_args()

scene = inputs.reyes_config5(n_frames=args.frames)
nsm, _ = vp.device_info(0)


def cfgs(name):
    if name == "mega":
        return vp.MEGAKERNEL, None
    if name == "kbk":
        return vp.KBK, None
    if name == "coarse":
        return vp.COARSE, None
    if name == "fine":
        return vp.FINE, None
    if name.startswith("h"):
        s, _, bat = name[1:].partition("b")
        s = int(s)
        batch = [int(x) for x in bat.split("_")] if bat else None
        return vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_MEGA, 0, s), (2, 3, vp.GROUP_RTC, s, nsm)], nsm, batch=batch)
    if name.startswith("s") and len(name) == 3:  # both groups on every SM: quotas [Bound,Split] / [Dice,Shade]
        q0, q1 = int(name[1]), int(name[2])
        return vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_MEGA, 0, nsm), (2, 3, vp.GROUP_RTC, 0, nsm)], nsm,
                                          blocks_per_sm=[q0, 0, q1, 0])
    if name[0] in "xe" and name[1].isdigit():
        # x{s}: [Bound,Split] on SMs [0, s/2) and [nsm/2, nsm/2 + s/2) (both halves of the
        # SM-id range); e{s}: on s evenly spaced SMs; [Dice,Shade] on the rest
        s = int(name[1:])
        if name[0] == "x":
            bs = set(range(s // 2)) | set(range(nsm // 2, nsm // 2 + s - s // 2))
        else:
            bs = {(k * nsm) // s for k in range(s)}
        b = vp.make_binding([(0, 1, vp.GROUP_MEGA, 0, 0), (2, 3, vp.GROUP_RTC, 0, 0)], nsm)
        for sm in range(nsm):
            g = 0 if sm in bs else 1
            b.group_sm_mask[g][sm >> 5] |= 1 << (sm & 31)
        return vp.HYBRID, b
    if name.startswith("fine_h"):
        return vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_FINE, 0, 40), (2, 3, vp.GROUP_RTC, 40, nsm)], nsm)
    raise ValueError(name)


for timers in ((False,) if args.no_timers else (False, True)):
    rp = ReyesPipeline(scene, flags=(vp.FLAG_TIMERS if timers else 0) | (vp.FLAG_ONLINE if args.online else 0)
                       | (vp.FLAG_L2_PERSIST if args.l2 else 0))
    for name in args.configs.split(","):
        model, b = cfgs(name)
        try:
            rp.configure(model, b, args.batch)
        except vp.VPError as e:
            print(name, "configure failed", e)
            continue
        rp.run()
        times = []
        for _ in range(args.reps):
            st = rp.run()
            times.append(st["device_ms"])
        rec = {"cfg": name, "timers": timers, "ms": min(times), "ms_all": [round(t, 3) for t in times],
               "deq": st["dequeued"][:4], "kernels": st["kernels"], "kernel_ms": [round(x, 3) for x in st["kernel_ms"]],
               "admitted": st["admitted"], "kbk_launches": st["kbk_launches"]}
        if timers:
            rec["exec_ms_blocksum"] = [round(x / 1e6, 2) for x in st["stage_exec_ns"][:4]]
            rec["flush_ms_blocksum"] = [round(x / 1e6, 2) for x in st["stage_flush_ns"][:4]]
            rec["idle_ms_blocksum"] = [round(x / 1e6, 2) for x in st["kernel_idle_ns"]]
        print(json.dumps(rec), flush=True)
