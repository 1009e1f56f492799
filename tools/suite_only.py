"""Dev tool: run bench.py's secondary workload suite alone and print it."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench
from paper_conf_micro_zhengozsyc17_b200 import vp
print(json.dumps(bench.workload_suite(torch, vp, torch.cuda.current_stream(), 8.0, 6548.5)), flush=True)
