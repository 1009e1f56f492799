"""Dev tool: autotune Reyes (small batch) and write the best config string; or
(with --cfg FILE) apply a stored config string in a fresh process and run it once."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_micro_zhengozsyc17_b200 import inputs, vp
from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline
frames = int(os.environ.get("FRAMES", "32"))
rp = ReyesPipeline(inputs.reyes_config5(n_frames=frames), watchdog_ms=5000)
if len(sys.argv) > 2 and sys.argv[1] == "--cfg":
    s = open(sys.argv[2]).read().strip()
    print("cfg:", s, flush=True)
    rp.p.configure_config(vp.config_from_string(s))
    rc, st, msg = rp.p.run_status()
    print("rc", rc, msg, st["dequeued"][:4], flush=True)
else:
    best, rep = rp.p.autotune(time_budget_s=20.0, sm_granularity=8, batch_choices=(1, 2))
    s = vp.config_to_string(best)
    open("gpurun_out/best.cfg", "w").write(s)
    print(s, flush=True)
