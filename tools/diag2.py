"""Dev tool: parity + timing of one hybrid split in a fresh pipeline (and after a re-configure)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
from paper_conf_micro_zhengozsyc17_b200 import inputs, vp
from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline
frames = int(sys.argv[2]) if len(sys.argv) > 2 else 64
scene = inputs.reyes_config5(n_frames=frames)
nsm, _ = vp.device_info(0)
ref = None
for order in sys.argv[1].split(";"):
    rp = ReyesPipeline(scene, flags=vp.FLAG_TIMERS | vp.FLAG_QUEUE_DEPTH, watchdog_ms=20000)
    for name in order.split(","):
        if name == "mega":
            rp.configure(vp.MEGAKERNEL)
        else:
            s = int(name[1:])
            rp.configure(vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_MEGA, 0, s), (2, 3, vp.GROUP_RTC, s, nsm)], nsm))
        rc, st, msg = rp.p.run_status()
        key, _ = rp.keys()
        if ref is None:
            ref = key.copy()
        print(json.dumps({"order": order, "cfg": name, "rc": rc, "ms": round(st["device_ms"], 3),
                          "same_as_first": bool(np.array_equal(key, ref)), "deq": st["dequeued"][:4],
                          "maxdepth": st["max_depth"][:4],
                          "exec": [round(x / 1e6, 1) for x in st["stage_exec_ns"][:4]]}), flush=True)
