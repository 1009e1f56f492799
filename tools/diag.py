"""Dev tool: one Reyes config with timers + queue-depth tracking."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_micro_zhengozsyc17_b200 import inputs, vp
from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline
frames = int(sys.argv[2]) if len(sys.argv) > 2 else 512
scene = inputs.reyes_config5(n_frames=frames)
nsm, _ = vp.device_info(0)
rp = ReyesPipeline(scene, flags=vp.FLAG_TIMERS | vp.FLAG_QUEUE_DEPTH, watchdog_ms=20000)
for name in sys.argv[1].split(","):
    s = int(name[1:])
    rp.configure(vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_MEGA, 0, s), (2, 3, vp.GROUP_RTC, s, nsm)], nsm))
    for r in range(2):
        rc, st, msg = rp.p.run_status()
        print(json.dumps({"cfg": name, "rc": rc, "msg": msg, "ms": st["device_ms"], "deq": st["dequeued"][:4],
                          "maxdepth": st["max_depth"][:4], "admitted": st["admitted"],
                          "exec": [round(x / 1e6, 1) for x in st["stage_exec_ns"][:4]],
                          "flush": [round(x / 1e6, 1) for x in st["stage_flush_ns"][:4]],
                          "idle": [round(x / 1e6, 1) for x in st["kernel_idle_ns"]]}), flush=True)
