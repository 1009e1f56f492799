"""Dev tool: time the LDPC decoder (100 frames x 100 iterations) under a few models."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_micro_zhengozsyc17_b200 import inputs, vp
from paper_conf_micro_zhengozsyc17_b200.workloads import LdpcPipeline
ls = inputs.ldpc_scene()
lp = LdpcPipeline(ls)
nsm, _ = vp.device_info(0)
for name, m, b in (("mega", vp.MEGAKERNEL, None), ("kbk", vp.KBK, None), ("kbk_graph", vp.KBK_GRAPH, None),
                   ("fine", vp.FINE, None)):
    lp.configure(m, b)
    lp.run()
    ts = [lp.run()["device_ms"] for _ in range(3)]
    print(json.dumps({"m": name, "ms": min(ts)}), flush=True)
best, rep = lp.p.autotune(time_budget_s=10, sm_granularity=4, batch_choices=(1, 2))
lp.run()
print(json.dumps({"m": "tuned", "ms": min(lp.run()["device_ms"] for _ in range(3)), "cfg": vp.config_to_string(best)[:100]}))
