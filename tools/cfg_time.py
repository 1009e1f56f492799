"""Dev tool: time a Reyes config-5 run under a stored config string (from bench.py's
JSON line) next to the equivalent reyes_sweep-style binding, to compare like with like."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_micro_zhengozsyc17_b200 import inputs, vp
from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline
cfg = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])["config_string"]
rp = ReyesPipeline(inputs.reyes_config5(n_frames=512))
nsm, _ = vp.device_info(0)
c = vp.config_from_string(cfg)
for name, apply in (("stored", lambda: rp.p.configure_config(c)),
                    ("sweep44", lambda: rp.configure(vp.HYBRID, vp.make_binding(
                        [(0, 1, vp.GROUP_MEGA, 0, 44), (2, 3, vp.GROUP_RTC, 44, nsm)], nsm, batch=[32, 16, 8, 4]))),
                    ("stored", lambda: rp.p.configure_config(c))):
    apply()
    rp.run()
    ts = [rp.run() for _ in range(3)]
    print(name, [round(t["device_ms"], 3) for t in ts], ts[-1]["kernels"], [round(x, 3) for x in ts[-1]["kernel_ms"]],
          vp.config_to_string(rp.p.get_config())[:200], flush=True)
