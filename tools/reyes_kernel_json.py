"""Dev tool: write profiles/<tag>_rtc_leaf_traffic.json and profiles/<tag>_reyes_kernels.json
(the figures bench.py's roofline.traffic / roofline.issue_bound carry) from the two ncu
captures of tools/gpu_evidence.sh and the task counts ncu_targets.py printed.

usage: python tools/reyes_kernel_json.py TAG RTC_REP RTC_LOG BS_REP BS_LOG"""
import csv
import io
import json
import subprocess
import sys

tag, rtc_rep, rtc_log, bs_rep, bs_log = sys.argv[1:6]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, u, v = rows[0], rows[1], rows[2]
    return {k: (v[i], u[i]) for i, k in enumerate(h)}


def counts(log, target):
    for line in open(log):
        if line.startswith(target + " "):
            head, _, rest = line.partition("[")
            return [int(x) for x in rest.split("]")[0].split(",")]
    raise SystemExit(f"no '{target}' line in {log}")


SCALE = {"": 1.0, "byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "%": 1.0, "inst": 1.0, "warp": 1.0,
         "register/thread": 1.0, "block": 1.0, "nsecond": 1.0, "ns": 1.0, "usecond": 1e3, "us": 1e3, "msecond": 1e6,
         "ms": 1e6, "second": 1e9, "s": 1e9, "B": 1.0, "KB": 1e3, "MB": 1e6, "GB": 1e9}


def f(d, k):
    """metric value in base units (bytes, ns, counts)"""
    val, unit = d[k]
    return float(val.replace(",", "")) * SCALE[unit]


r, b = raw(rtc_rep), raw(bs_rep)
leaves = counts(rtc_log, "rtc_leaf")[2]
bound_tasks = counts(bs_log, "bs_online")[0]
rd, wr = f(r, "dram__bytes_read.sum"), f(r, "dram__bytes_write.sum")
traffic = {"kernel": "vp_kernel<ReyesF,2,3,RTC>",
           "source": f"ncu --set full of tools/ncu_targets.py rtc_leaf --frames 64 ({tag})",
           "dram_bytes_read": rd, "dram_bytes_write": wr, "leaves": leaves, "bytes_per_leaf": (rd + wr) / leaves,
           "note": "single-kernel ncu target: the leaves are pre-seeded in HBM (in the bench step they arrive "
                   "through L2-resident rings), so this per-leaf figure is an upper bound for the co-running kernel"}
kern = {"source": f"ncu --set full, profiles/{tag}_rtc_leaf.txt and profiles/{tag}_bs_ncu_dfs.txt "
                  "(tools/ncu_targets.py rtc_leaf --frames 64 / bs_online --frames 32)",
        "fused_dice_shade": {"kernel": "vp_kernel<ReyesF,2,3,RTC>",
                             "issue_active_pct": f(r, "smsp__issue_active.avg.pct_of_peak_sustained_active"),
                             "warps_active_pct": f(r, "sm__warps_active.avg.pct_of_peak_sustained_active"),
                             "warp_instructions_per_leaf": f(r, "smsp__inst_executed.sum") / leaves,
                             "dram_bytes_per_leaf": (rd + wr) / leaves,
                             "registers": int(f(r, "launch__registers_per_thread")),
                             "duration_us_64_frames_alone": f(r, "gpu__time_duration.sum") / 1e3,
                             # the second limit: the L1/shared-memory data pipe
                             "smem_wavefronts_per_leaf": f(r, "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum") / leaves,
                             "smem_pipe_pct_of_peak": f(r, "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed"),
                             "l1tex_throughput_pct": f(r, "l1tex__throughput.avg.pct_of_peak_sustained_active")},
        "bound_split_dfs": {"kernel": "vp_kernel<ReyesF,0,1,MEGA> (depth-first, direct publish)",
                            "issue_active_pct": f(b, "smsp__issue_active.avg.pct_of_peak_sustained_active"),
                            "warps_active_pct": f(b, "sm__warps_active.avg.pct_of_peak_sustained_active"),
                            "warp_instructions_per_bound_task": f(b, "smsp__inst_executed.sum") / bound_tasks,
                            "registers": int(f(b, "launch__registers_per_thread")),
                            "blocks_per_sm": int(f(b, "launch__occupancy_limit_registers"))},
        "note": "both kernels are issue-bound (IEEE div/sqrt, integer coverage, shuffles, 128-bit CAS), and the "
                "fused Dice+Shade kernel also keeps the L1/shared-memory pipe busy (its grids live in shared memory), "
                "so the fp32 fraction understates how busy they are; issue_active is the fraction of issue slots "
                "used on the SMs the kernel ran on"}
json.dump(traffic, open(f"profiles/{tag}_rtc_leaf_traffic.json", "w"), indent=1)
json.dump(kern, open(f"profiles/{tag}_reyes_kernels.json", "w"), indent=1)
print(json.dumps(kern, indent=1))
