"""Dev tool: run the auto-tuner on the Reyes config-5 batch with VP_TUNE_DEBUG on."""
import os
import sys

os.environ["VP_TUNE_DEBUG"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_micro_zhengozsyc17_b200 import inputs, vp  # noqa: E402
from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline  # noqa: E402

secs = float(sys.argv[1]) if len(sys.argv) > 1 else 30.0
rp = ReyesPipeline(inputs.reyes_config5(n_frames=512))
best, rep = rp.p.autotune(time_budget_s=secs, sm_granularity=4, batch_choices=(1, 2))
print(vp.config_to_string(best), rep)
