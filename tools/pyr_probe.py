import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_micro_zhengozsyc17_b200 import inputs, vp
from paper_conf_micro_zhengozsyc17_b200.workloads import PyramidPipeline
rgb = inputs.pyramid_images(1, int(sys.argv[2]) if len(sys.argv) > 2 else 128)
pp = PyramidPipeline(rgb, watchdog_ms=5000)
pp.configure({"kbk": vp.KBK, "mega": vp.MEGAKERNEL}[sys.argv[1]])
print(pp.p.run_status()[:2])
