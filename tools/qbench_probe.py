import sys, os, json
sys.path.insert(0, os.getcwd())
import torch
from paper_conf_micro_zhengozsyc17_b200 import vp
from paper_conf_micro_zhengozsyc17_b200.workloads import QBenchPipeline
for ib, n in ((4, 128), (16, 128), (272, 16)):
    for bat in (0, 64, 1024):
        for timers in (0, 1):
            qb = QBenchPipeline(n, ib, 2, 16, flags=vp.FLAG_TIMERS if timers else 0)
            qb.configure(vp.MEGAKERNEL, None, bat if ib != 272 or bat <= 64 else 64)
            qb.run()
            res, st = qb.run()
            s = qb.stage
            print(json.dumps({"ib": ib, "batch": bat, "timers": timers, "ms": round(st["device_ms"], 3), "kernels": st["kernels"],
                              "exec_ms_sum": round(st["stage_exec_ns"][s] / 1e6, 2), "flush_ms_sum": round(st["stage_flush_ns"][s] / 1e6, 2),
                              "idle_ms_sum": [round(x / 1e6, 2) for x in st["kernel_idle_ns"]], "rounds": st["kernel_rounds"],
                              "admitted": st.get("admitted")}), flush=True)
            del qb
    qb = QBenchPipeline(n, ib, 2, 16)
    qb.configure(vp.KBK); qb.run(); res, st = qb.run()
    print(json.dumps({"ib": ib, "kbk_ms": round(st["device_ms"], 3), "launches": st["kbk_launches"]}), flush=True)
