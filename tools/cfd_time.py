"""Dev tool: time CFD config 3 (4096^2, 10 outer iterations) under a few models."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_micro_zhengozsyc17_b200 import inputs, vp
from paper_conf_micro_zhengozsyc17_b200.workloads import CfdPipeline
cs = inputs.cfd_scene(G=4096, n_outer=10)
cp = CfdPipeline(cs)
nsm, _ = vp.device_info(0)
def h3(a, b, bat):
    return vp.make_binding([(0, 0, vp.GROUP_MEGA, 0, a), (1, 2, vp.GROUP_MEGA, a, b), (3, 3, vp.GROUP_MEGA, b, nsm)], nsm, batch=bat)


for name, m, b in (("mega", vp.MEGAKERNEL, None), ("kbk", vp.KBK, None),
                   ("h3_4", vp.HYBRID, h3(8, 120, [4, 4, 2, 4])), ("h3_8", vp.HYBRID, h3(8, 120, [8, 8, 2, 8])),
                   ("h3_8b", vp.HYBRID, h3(8, 112, [8, 8, 2, 8])), ("h3_8c", vp.HYBRID, h3(4, 116, [8, 8, 2, 8])),
                   ("h3_8d", vp.HYBRID, h3(8, 128, [8, 8, 2, 8]))):
    cp.configure(m, b)
    cp.run()
    ts = [cp.run()["device_ms"] for _ in range(2)]
    print(json.dumps({"m": name, "ms": min(ts), "pct_hbm": 100 * 572 * cs.n_cells * cs.n_outer / (min(ts) / 1e3) / 1e9 / 6548.5}), flush=True)
