"""Dev tool: Reyes config 1 x R replicas under each model (which one overflows?)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_micro_zhengozsyc17_b200 import inputs, vp
from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline
R = int(sys.argv[1]) if len(sys.argv) > 1 else 256
rp = ReyesPipeline(inputs.reyes_config1(n_frames=R), watchdog_ms=5000)
nsm, _ = vp.device_info(0)
for name, model, b in (("kbk", vp.KBK, None), ("kbk_graph", vp.KBK_GRAPH, None), ("mega", vp.MEGAKERNEL, None),
                       ("h60", vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_MEGA, 0, 60), (2, 3, vp.GROUP_RTC, 60, nsm)], nsm))):
    rp.configure(model, b)
    rc, st, msg = rp.p.run_status()
    print(json.dumps({"m": name, "rc": rc, "msg": msg, "ms": st["device_ms"], "deq": st["dequeued"][:4],
                      "ring_count": st["ring_count"][:4], "cap": vp.config_to_string(rp.p.get_config())[:60]}), flush=True)
    if rc:
        rp = ReyesPipeline(inputs.reyes_config1(n_frames=R), watchdog_ms=5000)
