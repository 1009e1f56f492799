"""Dev tool: LDPC under the fine model with diagnostics (quotas, admitted blocks, counts)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_micro_zhengozsyc17_b200 import inputs, vp
from paper_conf_micro_zhengozsyc17_b200.workloads import LdpcPipeline
sc = inputs.ldpc_scene(n_frames=16, n_iter=20)
lp = LdpcPipeline(sc, watchdog_ms=3000)
model = sys.argv[1] if len(sys.argv) > 1 else "fine"
lp.configure({"fine": vp.FINE, "coarse": vp.COARSE}[model])
for r in range(2):
    rc, st, msg = lp.p.run_status()
    print(json.dumps({"rc": rc, "msg": msg, "kernels": st["kernels"], "admitted": st["admitted"],
                      "sms": [sum(1 for x in b if x) for b in st["blocks_on_sm"]],
                      "blocks": [sum(b) for b in st["blocks_on_sm"]], "deq": st["dequeued"][:4],
                      "pending": st["pending"], "fallback": st["fallback_admits"],
                      "ring_count": st["ring_count"][:4], "kernel_ms": [round(x, 3) for x in st["kernel_ms"]]}))
print(json.dumps(vp.config_to_string(lp.p.get_config())))
