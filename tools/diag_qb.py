"""Dev tool: qbench under the fine model with diagnostics (admitted blocks, SMs, rings)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_micro_zhengozsyc17_b200 import vp
from paper_conf_micro_zhengozsyc17_b200.workloads import QBenchPipeline
ib = int(sys.argv[1]) if len(sys.argv) > 1 else 272
qb = QBenchPipeline(4000, ib, 0, 0, watchdog_ms=3000)
qb.configure(vp.FINE)
rc, st, msg = qb.p.run_status()
print(json.dumps({"rc": rc, "msg": msg, "kernels": st["kernels"], "admitted": st["admitted"],
                  "sms": [sum(1 for x in b if x) for b in st["blocks_on_sm"]],
                  "blocks": [sum(b) for b in st["blocks_on_sm"]], "seed_head": st["seed_head"][:3],
                  "deq": st["dequeued"][:3], "pending": st["pending"], "fallback": st["fallback_admits"],
                  "kernel_ms": st["kernel_ms"]}))
print("b0", st["blocks_on_sm"][2][:40])
