"""Dev tool: queue microbenchmark under the megakernel with and without cluster work stealing
(VP_FLAG_CLUSTER_STEAL): best-of-3 device ms and items stolen."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_micro_zhengozsyc17_b200 import vp  # noqa: E402
from paper_conf_micro_zhengozsyc17_b200.workloads import QBenchPipeline  # noqa: E402

for ib in (4, 16):
    for fan, depth in ((1, 99), (2, 16)):
        n = (1 << 20 if ib < 272 else 1 << 18) if fan == 1 else (1 << 7 if ib < 272 else 1 << 4)
        for bat in (0, 64 if ib == 272 else 1024):
            rec = {"ib": ib, "fan": fan, "batch": bat}
            for steal, name in ((False, "plain"), (True, "steal")):
                try:
                    qb = QBenchPipeline(n, ib, fan, depth, steal=steal)
                except vp.VPError as ex:  # a library without the flag
                    rec[name] = str(ex)[:60]
                    continue
                qb.configure(vp.MEGAKERNEL, None, bat)
                qb.run()
                best, stolen = 1e9, 0
                for _ in range(3):
                    r, st = qb.run()
                    assert r["bad"] == 0 and st["dequeued"][0] == qb.tasks()
                    best = min(best, st["device_ms"])
                    stolen = st["stolen"][0]
                rec[name + "_ms"] = round(best, 3)
                rec[name + "_stolen"] = stolen
                del qb
            print(json.dumps(rec), flush=True)
