"""Dev tool: run the auto-tuner on a workload with progress printed (stderr)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_micro_zhengozsyc17_b200 import inputs, vp
from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline, RasterPipeline
w = sys.argv[1]
budget = float(sys.argv[2]) if len(sys.argv) > 2 else 10
if w == "reyes":
    rp = ReyesPipeline(inputs.reyes_config5(n_frames=int(sys.argv[3]) if len(sys.argv) > 3 else 32))
else:
    rp = RasterPipeline(inputs.raster_scene(50_000, W=640, H=360))
t = time.time()
best, rep = rp.p.autotune(time_budget_s=budget, sm_granularity=8, batch_choices=(1, 2))
print(w, "tuned in", round(time.time() - t, 1), "s: run", rep.candidates_run, "of", rep.candidates_total, "timed out",
      rep.candidates_timed_out, "best", rep.best_ms, "kbk", rep.baseline_kbk_ms, "mega", rep.baseline_mega_ms)
print(vp.config_to_string(best)[:200])
