"""Dev tool: CFD config 3 (4096^2, 10 outer iterations) under KBK (per-stage wave times),
the megakernel and a short auto-tune; prints one JSON line."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_micro_zhengozsyc17_b200 import inputs, vp  # noqa: E402
from paper_conf_micro_zhengozsyc17_b200.workloads import CfdPipeline  # noqa: E402

cs = inputs.cfd_scene(G=4096, n_outer=10)
cp = CfdPipeline(cs)
st = torch.cuda.current_stream()


def t(reps=3):
    cp.run(st)
    return min(cp.run(st)["device_ms"] for _ in range(reps))


out = {}
cp.configure(vp.KBK)
out["kbk_ms"] = t()
cp.p.set_flags(vp.FLAG_TIMERS)
cp.run(st)
out["stage_wave_ms"] = [round(x, 3) for x in cp.run(st)["stage_wave_ms"][:4]]
cp.p.set_flags(0)
cp.configure(vp.MEGAKERNEL)
out["mega_ms"] = t()
best, _ = cp.p.autotune(time_budget_s=float(os.environ.get("VP_TUNE_S", "15")), sm_granularity=4, batch_choices=(1, 2))
out["tuned_ms"] = t()
out["tuned"] = vp.config_to_string(best).split(" mask")[0]
out["pct_hbm_tuned"] = 100 * 572 * cs.n_cells * cs.n_outer / (out["tuned_ms"] / 1e3) / 6528.4e9
print(json.dumps(out), flush=True)
