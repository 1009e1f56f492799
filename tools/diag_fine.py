import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_micro_zhengozsyc17_b200 import inputs, vp
from paper_conf_micro_zhengozsyc17_b200.workloads import RasterPipeline, ReyesPipeline
which = sys.argv[1]
if which == "raster":
    rp = RasterPipeline(inputs.raster_scene(10_000, W=320, H=180), watchdog_ms=3000, flags=vp.FLAG_TIMERS)
else:
    rp = ReyesPipeline(inputs.reyes_config1(), watchdog_ms=3000, flags=vp.FLAG_TIMERS)
rp.configure(vp.FINE)
print(rp.p.profile(4))
rc, st, msg = rp.p.run_status()
print(rc, msg)
print("kernels", st["kernels"], "admitted", st["admitted"], "fallback", st["fallback_admits"], "deq", st["dequeued"][:4])
for k in range(st["num_kernels"]):
    b = st["blocks_on_sm"][k]
    print(k, "blocks_on_sm (first 16):", b[:16], "sum", sum(b))
print("idle", st["kernel_idle_ns"])
print("tail", st["ring_tail"][:4], "head", st["ring_head"][:4], "count", st["ring_count"][:4], "seed", st["seed_head"][:4], "pending", st["pending"])
print("rounds", st["kernel_rounds"])
