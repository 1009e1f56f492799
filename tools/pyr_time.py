"""Dev tool: time the config-3 pyramid (32 x 4096^2) under megakernel / tuned-like configs."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_micro_zhengozsyc17_b200 import inputs, vp
from paper_conf_micro_zhengozsyc17_b200.workloads import PyramidPipeline
rgb = inputs.pyramid_images(32, 4096)
pp = PyramidPipeline(rgb)
S = 4096
per_img = 3 * S * S + (3 * S * S + S * S) + sum(((S >> l) ** 2) * 5 for l in range(1, 13))
for name, m in (("mega", vp.MEGAKERNEL), ("kbk", vp.KBK), ("kbk_graph", vp.KBK_GRAPH)):
    pp.configure(m)
    pp.run()
    ts = [pp.run()["device_ms"] for _ in range(3)]
    print(json.dumps({"m": name, "ms": min(ts), "pct_hbm": 100 * 32 * per_img / (min(ts) / 1e3) / 1e9 / 6548.5}), flush=True)
