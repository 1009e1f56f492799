#!/usr/bin/env python
"""bench.py — VersaPipe Reyes batch (BASELINE config 5) on 1..8 B200s.

One "step" = one pass of the whole hot path (every §8(a) row: seed claim, Bound,
recursive Split, Dice, Shade with per-stage queues, the configured execution model,
the resolve sink) over this rank's shard of the 512-frame x 4096-patch batch.
Frames are sharded over ranks (no data-path collective); NCCL is used only for the
timing reduction and the post-run output gather (timed separately).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl vp|reference]
  torchrun --nproc-per-node N bench.py --gpus N ...

Prints ONE JSON line on rank 0.  --impl reference times the CPU oracle (the
reference arm for this paper-only tier) on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

TOTAL_FRAMES = 512
PATCH_SIDE = 64                      # 4096 patches per frame
MEASURED = os.path.join(ROOT, "MEASURED_PEAKS.json")

# Algorithmic fp32 operations per task (counted from the stage
# definitions, excluding per-point constant Bernstein tables and integer coverage work):
# Dice (reading R-R7, separable form): 36 u-curve points x 3 coords x (4 mul + 3 add), then
# per grid point 3 coords x 7 + M.p 24 (4 rows x (3 mul + 3 add): w = 1, R-S10, so the 4th
# product is no work and the kernel does not execute it) + screen 9 (3 div, 6 mul/add) +
# Q8 snap 2 = 5292
FLOP_DICE = 36 * 3 * 7 + 81 * (3 * 7 + 24 + 9 + 2)
FLOP_SHADE = 64 * 41                 # edges, cross, |n|, n.L, sqrt/div, shade, zq, Q8 snap = 2624
FLOP_SHADE_MP = 41                   # per micropolygon actually shaded (box holds a pixel centre)
FLOP_BOUND = 16 * (24 + 6) + 40      # 16 affine projections, sx / sy (2 div + 4), split metric = 520
FLOP_SPLIT = 3 * 4 * 12              # de Casteljau, 3 coords (w = 1) x 4 curves x 12 = 144


def env_int(k, d):
    try:
        return int(os.environ.get(k, d))
    except ValueError:
        return d


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="vp", choices=["vp", "reference"])
    ap.add_argument("--frames", type=int, default=TOTAL_FRAMES)
    ap.add_argument("--model", default="tuned",
                    help="tuned (auto-tuner) | hybrid | megakernel | kbk | kbk_graph | coarse | fine")
    ap.add_argument("--tune-seconds", type=float, default=30.0)
    ap.add_argument("--split", type=int, default=44, help="SMs for the [Bound,Split] group (hybrid)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-chunk", type=int, default=64, help="frames per chunk of the streamed e2e render")
    ap.add_argument("--no-baselines", action="store_true")
    ap.add_argument("--no-suite", action="store_true", help="skip the configs 1-4 secondary measurements")
    ap.add_argument("--no-qbench", action="store_true", help="skip the queue microbenchmark (d0)")
    ap.add_argument("--suite-tune-seconds", type=float, default=8.0)
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    return ap.parse_args()


def peaks():
    try:
        return json.load(open(MEASURED))
    except Exception:
        return {}


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""

    def __init__(self, gpu_index):
        self.p = None
        self.path = os.path.join(ROOT, "gpurun_out", f"clocks_rank{gpu_index}.csv")
        try:
            os.makedirs(os.path.dirname(self.path), exist_ok=True)
            self.f = open(self.path, "w")
            self.p = subprocess.Popen(
                ["nvidia-smi", "-i", str(gpu_index), "--query-gpu=clocks.sm,clocks.max.sm,power.draw,"
                 "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
                 "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap",
                 "--format=csv,noheader,nounits", "-lms", "20"], stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None

    def wait_ready(self, timeout_s=3.0):
        """Block until nvidia-smi has written its first sample, so the timed region that
        follows is actually sampled (the tool takes ~100 ms to start)."""
        t0 = time.time()
        while self.p and time.time() - t0 < timeout_s:
            self.f.flush()
            try:
                if os.path.getsize(self.path) > 0:
                    return
            except OSError:
                pass
            time.sleep(0.01)

    def stop(self):
        if not self.p:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        try:
            self.p.wait(timeout=5)
        except Exception:
            self.p.kill()
        self.f.close()
        rows = [r.split(",") for r in open(self.path).read().strip().splitlines() if r.count(",") >= 6]
        sm = [float(r[0]) for r in rows if r[0].strip().replace(".", "").isdigit()]
        mx = [float(r[1]) for r in rows if r[1].strip().replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4) if "Active" in r[3 + i] and "Not" not in r[3 + i]})
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(rows)}


def hybrid_binding(vp, nsm, split):
    s = split or max(8, nsm // 4)
    return vp.make_binding([(0, 1, vp.GROUP_MEGA, 0, s), (2, 3, vp.GROUP_RTC, s, nsm)], nsm)


def configure(vp, rp, model, nsm, split):
    if model == "hybrid":
        rp.configure(vp.HYBRID, hybrid_binding(vp, nsm, split))
    else:
        rp.configure({"megakernel": vp.MEGAKERNEL, "kbk": vp.KBK, "kbk_graph": vp.KBK_GRAPH, "coarse": vp.COARSE,
                      "fine": vp.FINE}[model])


def time_steps(torch, rp, steps, stream):
    """K steps bracketed by events on the launching stream; returns (ms total, last stats)."""
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    ev0.record(stream)
    st = None
    kms = []
    for _ in range(steps):
        st = rp.run(stream)
        kms.append(st["kernel_ms"])
    ev1.record(stream)
    torch.cuda.synchronize()
    return ev0.elapsed_time(ev1), st, kms


# Parity frames of the timed run: spread over the orbit; the camera is nearest (deepest
# recursion, depth-8 leaves) at f = 32 mod 64 and farthest at f = 0 mod 64.
PARITY_FRAMES = (0, 32, 75, 96, 160, 224, 288, 352, 416, 480, 511)


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def oracle_frames(frames, threads):
    """The C oracle as it stands (single-threaded per frame) on the given config-5 frames,
    one frame per host thread at a time (ctypes releases the GIL, so the threads run the
    C code in parallel).  Input generation happens before the timer starts."""
    import concurrent.futures as cf
    import oracle
    from paper_conf_micro_zhengozsyc17_b200 import inputs
    scenes = [inputs.reyes_config5(n_frames=1, n_side=PATCH_SIDE, frame0=f % TOTAL_FRAMES) for f in frames]
    t0 = time.perf_counter()
    with cf.ThreadPoolExecutor(max(1, threads)) as ex:
        res = list(ex.map(oracle.reyes_pipeline, scenes))
    return time.perf_counter() - t0, res


def cpu_oracle_sample(frames_total, seconds, must=()):
    """cpu_baseline: the oracle on a bounded sample of the same workload (about `seconds`
    of CPU time over all host cores).  The sample always contains the `must` frames (the
    parity frames), then frames spread evenly over the shard.  Returns (record, per-frame
    oracle results)."""
    import oracle
    oracle.build()
    cores = os.cpu_count() or 1
    one, _ = oracle_frames([32], 1)   # the nearest-camera frame bounds the per-frame cost
    n = int(min(frames_total, max(cores, len(must), seconds * cores / max(one, 1e-3))))
    frames = list(dict.fromkeys(must))
    for f in np.linspace(0, frames_total - 1, n).astype(int).tolist():
        if len(frames) >= n:
            break
        if f not in frames:
            frames.append(f)
    dt, res = oracle_frames(frames, cores)
    items = sum(r["n_bound"] + r["n_split"] + r["n_dice"] + r["n_shade"] for r in res)
    hist = np.sum([r["depth_hist"][:9] for r in res], axis=0).tolist()
    rec = {"value": len(frames) / dt, "unit": "frames/s", "cores": cores, "threads": cores, "kind": "oracle",
           "cpu_model": cpu_model(), "items_per_sec": items / dt, "seconds": dt, "frames": len(frames),
           "sample": f"{len(frames)} of {frames_total} config-5 frames (4096 patches each, parity frames included), "
                     f"C oracle one frame per thread on {cores} threads, input generation excluded, {dt:.1f} s",
           "leaf_depth_hist_sample": hist}
    return rec, dict(zip(frames, res))


def parity_check(snap, ref):
    """The timed configuration's outputs (snapshotted right after the timed region) vs the
    oracle, per sampled frame: depth keys and shade factors bit-exact, colours within
    north_star's 1e-4 (bit-exact expected)."""
    keys_bad, s_bad, err = 0, 0, 0.0
    for f, (k, sf, c) in snap.items():
        r = ref[f]
        keys_bad += int(np.count_nonzero(k != r["key"][0]))
        s_bad += int(np.count_nonzero(sf != r["s"][0]))
        err = max(err, float(np.max(np.abs(c - r["colour"][0]))))
    return {"pass": keys_bad == 0 and s_bad == 0 and err <= 1e-4, "frames": sorted(snap), "keys_differing": keys_bad,
            "s_differing": s_bad, "max_abs_err": err, "tolerance": 1e-4,
            "checked": "outputs of the last timed step (timed configuration) vs the CPU oracle"}


def run_reference(args, rank, world):
    """--impl reference: the CPU oracle, rank 0 only (other ranks exit without work).
    Each step renders a bounded sample of the config-5 frames; ms_per_step is that
    step's measured wall time, so steps x ms_per_step is what ran."""
    if rank != 0:
        return
    import oracle
    oracle.build()
    cores = os.cpu_count() or 1
    one, _ = oracle_frames([32], 1)
    per_step = int(max(cores, min(args.frames, args.cpu_seconds / max(args.steps, 1) * cores / max(one, 1e-3))))
    frames = np.linspace(0, args.frames - 1, per_step).astype(int).tolist()
    for _ in range(args.warmup):
        oracle_frames(frames[:cores], cores)
    secs, items = [], []
    for _ in range(args.steps):
        dt, res = oracle_frames(frames, cores)
        secs.append(dt)
        items.append(sum(r["n_bound"] + r["n_split"] + r["n_dice"] + r["n_shade"] for r in res) / dt)
    ms = 1000.0 * float(np.median(secs))
    v = per_step / (ms / 1000.0)
    sample = (f"{per_step} of {args.frames} config-5 frames per step (spread over the orbit), C oracle one frame per "
              f"thread on {cores} threads, input generation excluded")
    line = {"impl": "reference", "metric": "frames/sec", "value": v, "unit": "frames/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f32",
            "data": "synthetic", "items_per_sec": float(np.median(items)), "frames_per_step": per_step,
            "config": {"workload": "reyes_batch_config5", "frames": args.frames, "patches_per_frame": 4096,
                       "image": "256x256", "max_depth": 8, "sample_frames_per_step": per_step},
            "cpu_baseline": {"value": v, "unit": "frames/s", "cores": cores, "kind": "oracle", "sample": sample,
                             "cpu_model": cpu_model()},
            "e2e": {"value": v, "unit": "frames/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def queue_microbench(torch, vp, stream):
    """the ring queues alone.  Chains (fan-out 1) and binary trees
    (fan-out 2) of 4 / 16 / 272-B items under the megakernel and both KBK flavours; tasks/s
    and ring payload GB/s (each task reads its item and writes its children)."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import QBenchPipeline
    out = {}
    for ib in (4, 16, 272):
        for fan, depth in ((1, 99), (2, 16)):
            # chains: 2^20 (2^18) live items; trees: the last level (n * 2^16) must fit the ring
            n = (1 << 20 if ib < 272 else 1 << 18) if fan == 1 else (1 << 7 if ib < 272 else 1 << 4)
            qb = QBenchPipeline(n, ib, fan, depth)
            r = {}
            # the megakernel at the default batch and at the largest one its kernel allows (the
            # batch is one of the tuner's parameters, L41; trees publish 2 children per task,
            # and larger batches amortise the publisher warp's per-round work)
            for name, model, bat in (("megakernel", vp.MEGAKERNEL, 0), ("megakernel_max_batch", vp.MEGAKERNEL, 64 if ib == 272 else 1024),
                                     ("kbk", vp.KBK, 0), ("kbk_graph", vp.KBK_GRAPH, 0)):
                qb.configure(model, None, bat)
                qb.run(stream)
                ts = []
                for _ in range(3):
                    res, st = qb.run(stream)
                    assert res["bad"] == 0 and st["dequeued"][qb.stage] == qb.tasks()
                    ts.append(st["device_ms"])
                ms = min(ts)
                r[name] = {"ms": ms, "mtasks_per_s": qb.tasks() / ms / 1e3, "batch": bat or "default",
                           # every task reads its item once; every non-seed item was written once
                           "ring_gbs": (2 * qb.tasks() - n) * ib / ms / 1e6}
            out[f"item{ib}_fan{fan}"] = {"tasks": qb.tasks(), **r}
            del qb
    return out


def oracle_mod():
    import oracle
    oracle.build()
    return oracle


def workload_suite(torch, vp, stream, tune_s, hbm_gbs):
    """Secondary measurements: every BASELINE workload (configs 1-4) through the same
    runtime, auto-tuned, vs KBK; items/s, frames/s and % of measured HBM where the
    workload is HBM-bound."""
    from paper_conf_micro_zhengozsyc17_b200 import inputs
    from paper_conf_micro_zhengozsyc17_b200.workloads import (CfdPipeline, FaceDetPipeline, PyramidPipeline,
                                                              RasterPipeline, ReyesPipeline)  # noqa: F401

    def measure(pipe, frames, alg_bytes=None, reps=3):
        best, rep = pipe.p.autotune(time_budget_s=tune_s, sm_granularity=4, batch_choices=(1, 2))
        tuned_cfg = vp.config_to_string(best)

        def t_run():
            pipe.run(stream)
            ts = []
            st = None
            for _ in range(reps):
                st = pipe.run(stream)
                ts.append(st["device_ms"])
            return min(ts), st

        ms, st = t_run()
        pipe.configure(vp.KBK)
        kbk_ms, _ = t_run()
        # per-stage wave times in a separate timed run (the event records cost KBK time)
        pipe.p.set_flags(vp.FLAG_TIMERS)
        _, kst = t_run()
        pipe.p.set_flags(0)
        pipe.configure(vp.KBK_GRAPH)
        kbkg_ms, _ = t_run()
        pipe.configure(vp.MEGAKERNEL)
        mega_ms, _ = t_run()
        pipe.p.configure_config(best)
        pipe.run(stream)  # the outputs the parity checks read come from the tuned configuration
        items = sum(st["dequeued"][:8])
        r = {"ms": ms, "frames_per_s": frames / (ms / 1e3), "items_per_s": items / (ms / 1e3),
             "items": items, "kbk_ms": kbk_ms, "kbk_graph_ms": kbkg_ms, "megakernel_ms": mega_ms,
             "speedup_vs_kbk": kbk_ms / ms, "speedup_vs_kbk_graph": kbkg_ms / ms,
             "speedup_vs_megakernel": mega_ms / ms, "tuned": tuned_cfg.split(" mask")[0]}
        # Table 2 analog (L51): the longest stage run in isolation (its KBK waves, whole GPU)
        # vs the pipeline; the difference is queue / runtime overhead and stage imbalance
        sw = [x for x in kst["stage_wave_ms"] if x > 0]
        if sw:
            r["stage_wave_ms"] = [round(x, 4) for x in kst["stage_wave_ms"][:len(st["dequeued"])]]
            r["longest_stage_ms"] = max(sw)
            r["overhead_vs_longest_stage_pct"] = 100.0 * (ms - max(sw)) / ms
        if alg_bytes:
            gbs = alg_bytes / (ms / 1e3) / 1e9
            r.update({"alg_bytes": alg_bytes, "achieved_gbs": gbs, "pct_hbm_measured": 100 * gbs / hbm_gbs})
        return r

    out = {}
    cores = os.cpu_count() or 1
    alu_peak = None
    try:
        nsm_, _ = vp.device_info(0)
        alu_peak = nsm_ * 128 * peaks().get("sm_max_mhz", 1965.0) * 1e6 / 1e12
    except Exception:
        pass

    def guarded(name, fn):
        try:
            fn()
        except Exception as ex:  # one workload's failure must not hide the others
            out[name] = {"error": repr(ex)}

    def threads_run(fn, args, threads):
        """The C oracle (as it stands) over independent units on `threads` host threads
        (ctypes releases the GIL); inputs are built before the timer."""
        import concurrent.futures as cf
        t0 = time.perf_counter()
        with cf.ThreadPoolExecutor(max(1, threads)) as ex:
            res = list(ex.map(fn, args))
        return time.perf_counter() - t0, res

    def cpu_rec(units, unit, secs, threads, sample):
        return {"value": units / secs, "unit": unit, "cores": cores, "threads": threads, "kind": "oracle",
                "cpu_model": cpu_model(), "seconds": secs, "sample": sample}

    def hbm_roof(alg_bytes, ms):
        a = alg_bytes / (ms / 1e3) / 1e9
        return {"bound": "hbm", "achieved": a, "peak": hbm_gbs, "unit": "GB/s", "frac": a / hbm_gbs,
                "peak_source": "MEASURED_PEAKS.json hbm copy bandwidth", "alg_bytes": alg_bytes}

    def reyes_roof(deq, ms):
        fl = deq[0] * FLOP_BOUND + deq[1] * FLOP_SPLIT + deq[2] * FLOP_DICE + deq[3] * FLOP_SHADE
        a = fl / (ms / 1e3) / 1e12
        return {"bound": "alu", "achieved": a, "peak": alu_peak, "unit": "TFLOP/s", "frac": a / alu_peak,
                "peak_source": "SMs x 128 fp32 lanes x sm_max_mhz (non-FMA)",
                "note": "latency-bound at one frame: >= 10 dependent rounds of small waves"}

    def w_reyes1():
        out["reyes_config1"] = measure(ReyesPipeline(inputs.reyes_config1()), 1)

    def w_reyes1x():
        # SURVEY §8(d) throughput mode: R = 256 independent config-1 frames in one run
        rp = ReyesPipeline(inputs.reyes_config1(n_frames=256))
        r = measure(rp, 256)
        one = inputs.reyes_config1()
        n = 4 * cores
        secs, res = threads_run(oracle_mod().reyes_pipeline, [one] * n, cores)
        r["cpu_baseline"] = cpu_rec(n, "frames/s", secs, cores, f"{n} config-1 frames, one per thread")
        key, s_ = rp.keys()
        col = rp.colours()
        ref = res[0]
        fr = (0, 1, 77, 128, 255)
        bad = sum(int(np.count_nonzero(key[f] != ref["key"][0])) for f in fr)
        err = max(float(np.max(np.abs(col[f] - ref["colour"][0]))) for f in fr)
        r["parity"] = {"pass": bad == 0 and err <= 1e-4, "frames": list(fr), "keys_differing": bad, "max_abs_err": err}
        r["roofline"] = reyes_roof(rp.run(stream)["dequeued"], r["ms"])
        r["leaf_depth_hist"] = list(ref["depth_hist"][:9])
        out["reyes_config1_x256"] = r

    def w_face():
        fs = inputs.face_scene()
        fp = FaceDetPipeline(fs)
        out["facedet_config2"] = measure(fp, fs.n_frames)
        out["facedet_config2"]["windows_per_s"] = fp.results()["windows"] / (out["facedet_config2"]["ms"] / 1e3)

    def w_face8():
        import dataclasses
        fs8 = inputs.face_scene(n_frames=8)  # throughput mode, R = 8 frames
        fp8 = FaceDetPipeline(fs8)
        r = measure(fp8, fs8.n_frames)
        got = fp8.results()
        r["windows_per_s"] = got["windows"] / (r["ms"] / 1e3)
        r["survivors_per_cascade_stage"] = got["survivors"]
        subs = [dataclasses.replace(fs8, rgb=fs8.rgb[f:f + 1]) for f in range(fs8.n_frames)]
        secs, res = threads_run(lambda sc: oracle_mod().fd_pipeline(sc, det_cap=1 << 20), subs, cores)
        r["cpu_baseline"] = cpu_rec(len(subs), "frames/s", secs, min(cores, len(subs)),
                                    f"the {len(subs)} 1920x1080 frames, one per thread")
        want = sorted((f, *map(int, d[1:])) for f, rr in enumerate(res) for d in rr["det"])
        have = sorted(tuple(int(v) for v in d) for d in got["det"])
        surv = [sum(rr["survivors"][k] for rr in res) for k in range(len(res[0]["survivors"]))]
        r["parity"] = {"pass": want == have and surv == got["survivors"], "detections": len(have),
                       "survivors_equal": surv == got["survivors"]}
        # ~203 MB/frame algorithmic (frame, pyramid, LBP, 16-B window items w+r)
        r["roofline"] = hbm_roof(203e6 * fs8.n_frames, r["ms"])
        r["roofline"]["note"] = ("issue-bound (cascade evaluation, integer ALU/LSU); see profiles/r2_suite_ncu.txt "
                                 "for issue-slot use")
        out["facedet_config2_x8"] = r

    def w_pyr():
        n_img, S = 32, 4096
        rgb = inputs.pyramid_images(n_img, S)
        # Gray: RGB read; Map: RGB read + level-0 write; Resize: read + write per level; hist negligible
        per_img = 3 * S * S + (3 * S * S + S * S) + sum(((S >> l) ** 2) * 5 for l in range(1, 13))
        pp = PyramidPipeline(rgb)
        r = measure(pp, n_img, alg_bytes=n_img * per_img)
        r["roofline"] = hbm_roof(n_img * per_img, r["ms"])
        got = pp.pyramid()
        ims = [rgb[i:i + 1] for i in range(n_img)]
        secs, res = threads_run(oracle_mod().pyr_pipeline, ims, cores)
        r["cpu_baseline"] = cpu_rec(n_img, "images/s", secs, min(cores, n_img), f"all {n_img} 4096^2 images, one per thread")
        bad = sum(int(np.count_nonzero(got[i] != res[i]["pyr"][0])) for i in range(n_img))
        r["parity"] = {"pass": bad == 0, "images": n_img, "bytes_differing": bad}
        out["pyramid_config3"] = r

    def w_cfd():
        import dataclasses
        cs = inputs.cfd_scene(G=4096, n_outer=10)
        cp = CfdPipeline(cs)
        r = measure(cp, 1, alg_bytes=572 * cs.n_cells * cs.n_outer, reps=2)
        r["cell_updates_per_s"] = cs.n_cells * 3 * cs.n_outer / (r["ms"] / 1e3)
        r["roofline"] = hbm_roof(572 * cs.n_cells * cs.n_outer, r["ms"])
        r["roofline"]["note"] = ("Flux is issue-bound (~1190 thread-instructions per cell: IEEE div/sqrt, 4 faces); "
                                 "the streaming stages are HBM-bound (profiles/r2_suite_ncu.txt)")
        # oracle: one outer iteration of the full 4096^2 grid (a documented subset, single thread)
        cs1 = dataclasses.replace(cs, n_outer=1)
        t0 = time.perf_counter()
        ref = oracle_mod().cfd_pipeline(cs1)
        secs = time.perf_counter() - t0
        r["cpu_baseline"] = cpu_rec(cs.n_cells * 3, "cell-updates/s", secs, 1,
                                    "1 outer iteration (3 RK steps) of the 4096^2 grid, single-threaded C oracle")
        cp1 = CfdPipeline(cs1)
        cp1.p.configure_config(cp.p.get_config())
        cp1.run(stream)
        got = cp1.state()
        r["parity"] = {"pass": bool(np.array_equal(got, ref["vars"])), "outer_iterations": 1,
                       "max_abs_err": float(np.max(np.abs(got - ref["vars"])))}
        out["cfd_config3"] = r

    def w_ldpc():
        # the LDPC decoder (Fig. 17), 100 frames x 100 iterations (L53)
        from paper_conf_micro_zhengozsyc17_b200.workloads import LdpcPipeline
        ls = inputs.ldpc_scene()
        lp = LdpcPipeline(ls)
        r = measure(lp, ls.n_frames)
        r["decoder_iterations_per_s"] = ls.n_frames * ls.n_iter / (r["ms"] / 1e3)
        t0 = time.perf_counter()
        ref = oracle_mod().ldpc_pipeline(ls)
        secs = time.perf_counter() - t0
        r["cpu_baseline"] = cpu_rec(ls.n_frames * ls.n_iter, "decoder-iterations/s", secs, 1,
                                    "all 100 frames x 100 iterations, single-threaded C oracle")
        got = lp.results()
        r["parity"] = {"pass": bool(np.array_equal(got["post"], ref["post"]) and np.array_equal(got["errors"], ref["errors"]))}
        out["ldpc_f3"] = r

    def w_raster():
        rs = inputs.raster_scene()
        rp = RasterPipeline(rs)
        r = measure(rp, 1, alg_bytes=265_000_000)
        r["triangles_per_s"] = rs.n_tris / (r["ms"] / 1e3)
        t0 = time.perf_counter()
        ref = oracle_mod().raster_pipeline(rs)
        secs = time.perf_counter() - t0
        r["cpu_baseline"] = cpu_rec(1, "frames/s", secs, 1, "the full 1M-triangle 1920x1080 frame, single-threaded")
        key = rp.keys()
        col = rp.colours()
        r["parity"] = {"pass": bool(np.array_equal(key, ref["key"]) and np.array_equal(col, ref["colour"])),
                       "keys_differing": int(np.count_nonzero(key != ref["key"]))}
        # the L2-atomic bound of Fragment (one 64-bit RED.MIN per covered sample
        # passing the depth range) against the measured RED.MIN.U64 rate into the same
        # 16.6 MB key buffer; Vertex/Clip's HBM share is in profiles/r2_suite_ncu.txt
        try:
            peak = vp.bench_red_min_u64(rs.W * rs.H)
            a = ref["n_frag_pixels"] / (r["ms"] / 1e3)
            r["roofline"] = {"bound": "l2_atomic", "achieved": a / 1e9, "peak": peak / 1e9, "unit": "G atomics/s",
                             "frac": a / peak, "atomics": int(ref["n_frag_pixels"]),
                             "peak_source": "vp_bench_red_min_u64 (measured, same buffer size)"}
        except Exception as ex:
            r["roofline"] = {"error": repr(ex)}
        r["roofline_hbm"] = hbm_roof(265_000_000, r["ms"])
        out["raster_config4"] = r

    def w_raster_near():
        # SURVEY §8(f-4), DESIGN R-S9: config-4 triangles with per-vertex z ~ U(-0.6, 0.95),
        # so about half straddle the near plane and Clip fans out 0..2 sub-triangles
        rs = inputs.raster_near_scene(n=1 << 20, W=1920, H=1080, area_range=(0.5, 512.0))
        rp = RasterPipeline(rs)
        r = measure(rp, 1)
        r["triangles_per_s"] = rs.n_tris / (r["ms"] / 1e3)
        t0 = time.perf_counter()
        ref = oracle_mod().raster_pipeline(rs)
        secs = time.perf_counter() - t0
        r["cpu_baseline"] = cpu_rec(1, "frames/s", secs, 1, "the full 1M-triangle 1920x1080 near-clip frame, single-threaded")
        key = rp.keys()
        col = rp.colours()
        r["parity"] = {"pass": bool(np.array_equal(key, ref["key"]) and np.array_equal(col, ref["colour"])),
                       "keys_differing": int(np.count_nonzero(key != ref["key"]))}
        out["raster_near_clip"] = r

    def w_pyr_fig13():
        # PAPER.md Fig. 13 (L53-L55): the pyramid at 1..32 images under KBK, KBK with
        # streams (M25: images split over 8 streams, one host thread each), the megakernel
        # and the auto-tuned pipeline
        from paper_conf_micro_zhengozsyc17_b200.workloads import PyramidKbkStreams
        S = 4096
        rgb_all = torch.from_numpy(inputs.pyramid_images(32, S)).cuda()
        rows = []
        for n_img in (1, 2, 4, 8, 16, 32):
            rgb = rgb_all[:n_img]
            pp = PyramidPipeline(rgb, rgb_on_device=rgb)
            row = {"images": n_img}

            def t(fn, reps=3):
                fn()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                ts = []
                for _ in range(reps):
                    torch.cuda.synchronize()
                    e0.record(stream)
                    fn()
                    e1.record(stream)
                    torch.cuda.synchronize()
                    ts.append(e0.elapsed_time(e1))
                return min(ts)

            pp.configure(vp.KBK)
            row["kbk_ms"] = t(lambda: pp.run(stream))
            ks = PyramidKbkStreams(rgb, 8)
            row["kbk_streams_ms"] = t(lambda: ks.run(stream))
            row["kbk_streams"] = ks.n_streams
            del ks
            pp.configure(vp.MEGAKERNEL)
            row["megakernel_ms"] = t(lambda: pp.run(stream))
            best, _ = pp.p.autotune(time_budget_s=min(tune_s, 4.0), sm_granularity=8, batch_choices=(1, 2))
            row["versapipe_ms"] = t(lambda: pp.run(stream))
            row["versapipe_config"] = vp.config_to_string(best).split(" mask")[0]
            row["images_per_s"] = {k[:-3]: n_img / (row[k] / 1e3) for k in ("kbk_ms", "kbk_streams_ms", "megakernel_ms",
                                                                           "versapipe_ms")}
            rows.append(row)
            del pp
        out["pyramid_fig13"] = rows

    for name, fn in (("reyes_config1", w_reyes1), ("reyes_config1_x256", w_reyes1x), ("facedet_config2", w_face),
                     ("facedet_config2_x8", w_face8), ("pyramid_config3", w_pyr), ("cfd_config3", w_cfd),
                     ("ldpc_f3", w_ldpc), ("raster_config4", w_raster), ("raster_near_clip", w_raster_near),
                     ("pyramid_fig13", w_pyr_fig13)):
        guarded(name, fn)
    return out


def main():
    args = parse()
    rank, world, local = env_int("RANK", 0), env_int("WORLD_SIZE", 1), env_int("LOCAL_RANK", 0)
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    import torch
    import torch.distributed as dist
    from paper_conf_micro_zhengozsyc17_b200 import build as vpbuild
    vpbuild.build()
    from paper_conf_micro_zhengozsyc17_b200 import inputs, vp
    from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline

    # VP_BENCH_ONE_GPU=1 (dev only): every rank on cuda:0 with gloo, to exercise the N > 1
    # code path (sharding, reductions, gather) on a one-GPU box; the driver never sets it
    one_gpu = os.environ.get("VP_BENCH_ONE_GPU") == "1"
    if one_gpu:
        local = 0
    torch.cuda.set_device(local)
    if world > 1:
        if one_gpu:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    nsm, cc = vp.device_info(local)
    # ---- shard: rank r renders frames [r*F/P, (r+1)*F/P) of the orbit
    from paper_conf_micro_zhengozsyc17_b200 import shard
    f0, f1 = shard.shard_range(rank, world, args.frames)
    scene = inputs.reyes_config5(n_frames=f1 - f0, n_side=PATCH_SIDE, frame0=f0)
    rp = ReyesPipeline(scene, device=local)
    tune = None
    if args.model == "tuned":
        # the paper's offline auto-tuner (L41-L45, Fig. 10) picks {grouping, models, SM
        # split, batch} on this shard before anything is timed
        t_tune = time.perf_counter()
        best_cfg, rep = rp.p.autotune(time_budget_s=args.tune_seconds, sm_granularity=1, batch_choices=(1, 2))
        tune = {"seconds": round(time.perf_counter() - t_tune, 2), "candidates_run": rep.candidates_run,
                "candidates_total": rep.candidates_total, "timed_out": rep.candidates_timed_out,
                "best_ms": rep.best_ms, "kbk_ms": rep.baseline_kbk_ms, "megakernel_ms": rep.baseline_mega_ms,
                "config": vp.config_to_string(best_cfg)}
    else:
        configure(vp, rp, args.model, nsm, args.split)
    main_cfg = rp.p.get_config()
    stream = torch.cuda.current_stream()
    for _ in range(max(args.warmup, 3) if args.warmup >= 3 else args.warmup):
        rp.run(stream)

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    # ---- timed region: inputs resident in HBM (seeds 4096 x 208 B per frame > L2)
    barrier()
    clk = Clocks(local)
    clk.wait_ready()
    t_ms, st, kms = time_steps(torch, rp, args.steps, stream)
    barrier()
    clocks = clk.stop()
    # outputs of the last timed step, for the parity check against the oracle (the
    # baselines below re-render the same buffers)
    npf = scene.W * scene.H
    snap = {}
    for f in PARITY_FRAMES:
        if f0 <= f < f1:
            lf = f - f0
            fbf = rp.fb[lf * npf:(lf + 1) * npf].cpu().numpy()
            snap[f] = (fbf[:, :2].copy().view(np.uint64).reshape(scene.H, scene.W),
                       fbf[:, 2].copy().view(np.float32).reshape(scene.H, scene.W), rp.colour[lf].cpu().numpy())
    t_ms = shard.max_over_ranks(t_ms, "cuda")
    items_all, frames_all = shard.sum_over_ranks([sum(st["dequeued"][:4]), f1 - f0], "cuda")
    ms_per_step = t_ms / args.steps
    fps = frames_all * args.steps / (t_ms / 1e3)
    ips = items_all * args.steps / (t_ms / 1e3)

    # ---- dominant kernel (largest event time among the persistent kernels of the step)
    nk = st["num_kernels"]
    kmean = np.mean(np.array(kms), axis=0) if nk else np.array([ms_per_step])
    d = st["dequeued"]
    units = st.get("work_units", [0] * 8)
    # Shade flops are counted per micropolygon the fused chain actually shades (those whose
    # box holds a pixel centre, vp_run_stats.work_units) -- 64 per grid only if Shade ran
    # unfused and no count exists
    shade_flop = units[3] * FLOP_SHADE_MP if units[3] else d[3] * FLOP_SHADE
    stage_flop = [d[0] * FLOP_BOUND, d[1] * FLOP_SPLIT, d[2] * FLOP_DICE, shade_flop]
    # persistent groups co-run for the whole step, so the dominant kernel is the one
    # with the most algorithmic work; its time is its own CUDA-event duration
    kflop = [sum(stage_flop[s] for s in range(k[0], k[1] + 1)) for k in st["kernels"]] if nk else [0]
    dom = int(np.argmax(kflop)) if nk else 0
    lo, hi, _ = st["kernels"][dom] if nk else (0, 3, 0)
    dom_flop = sum(stage_flop[s] for s in range(lo, hi + 1))
    pk = peaks()
    sm_max = pk.get("sm_max_mhz", 1965.0)
    # fp32 non-FMA issue peak: 148 SMs x 128 lanes x 1 op/clk (FMA contraction is disabled
    # for bit-exactness), at clocks.max.sm
    alu_peak = nsm * 128 * sm_max * 1e6 / 1e12
    achieved = dom_flop / (kmean[dom] / 1e3) / 1e12
    b = main_cfg.binding
    is_rtc = bool(main_cfg.has_binding and b.group_model[b.group_of_stage[lo]] == vp.GROUP_RTC)
    # traffic: dram bytes per leaf from the committed ncu --set full capture of this kernel
    # (profiles/r1_rtc_leaf_traffic.json), times the leaves this launch processed
    traffic = None
    traffic_src = None
    for name in ("r2_rtc_leaf_traffic.json", "r1_rtc_leaf_traffic.json"):
        try:
            tr = json.load(open(os.path.join(ROOT, "profiles", name)))
            if (lo, hi) == (2, 3):
                traffic = tr["bytes_per_leaf"] * d[2]
                traffic_src = f"ncu dram__bytes_read+write per leaf (profiles/{name}) x leaves"
            break
        except Exception:
            continue
    issue = None
    try:  # issue-slot view of the same kernels (the bound that actually binds), from committed captures
        issue = json.load(open(os.path.join(ROOT, "profiles", "r2_reyes_kernels.json")))
    except Exception:
        pass
    roofline = {"bound": "alu", "achieved": achieved, "peak": alu_peak, "unit": "TFLOP/s",
                "frac": achieved / alu_peak, "traffic": traffic,
                "flop_count": {"shaded_micropolygons": int(units[3]), "dice_leaves": int(d[2]),
                               "shade_flop_per_mp": FLOP_SHADE_MP, "dice_flop_per_leaf": FLOP_DICE},
                "issue_bound": issue,
                "traffic_source": traffic_src,
                "kernel": f"vp_kernel<ReyesF,{lo},{hi},{'RTC' if is_rtc else 'MEGA'}>",
                "peak_source": "derived: SMs x 128 fp32 lanes x clocks.max.sm (MEASURED_PEAKS sm_max_mhz), non-FMA",
                "kernel_ms": float(kmean[dom]), "kernel_share_of_step": float(kmean[dom] / ms_per_step)}
    # the other persistent group(s) of the step (VERDICT r1 named the [Bound, Split] group
    # as the kernel furthest below its roofline): the same ALU view, against the fp32 peak
    # of the SMs the group is bound to
    others = []
    for i, (klo, khi, _) in enumerate(st["kernels"] if nk else []):
        if i == dom:
            continue
        g = b.group_of_stage[klo] if main_cfg.has_binding else 0
        sms = sum(bin(w).count("1") for w in b.group_sm_mask[g]) if main_cfg.has_binding else nsm
        kf = sum(stage_flop[s] for s in range(klo, khi + 1))
        ka = kf / (kmean[i] / 1e3) / 1e12
        kpeak = sms * 128 * sm_max * 1e6 / 1e12
        others.append({"kernel": f"vp_kernel<ReyesF,{klo},{khi}>", "sms": sms, "achieved": ka, "peak": kpeak,
                       "unit": "TFLOP/s", "frac": ka / kpeak if kpeak else None, "kernel_ms": float(kmean[i]),
                       "flop_per_task": {"bound": FLOP_BOUND, "split": FLOP_SPLIT}})
    roofline["other_groups"] = others
    hbm = pk.get("hbm_gbs", 6548.5)
    # HBM bytes per step that must move: seeds read + fb clear/CAS/resolve + colour write
    npix = scene.n_frames * scene.W * scene.H
    bytes_step = scene.seeds.size * inputs.GPU_PATCH_DTYPE.itemsize + npix * (16 + 16 + 16 + 16)

    # ---- baselines on the same shard: KBK (one launch per stage per wave) + megakernel
    extra = {}
    if not args.no_baselines:
        for name in ("kbk", "kbk_graph", "megakernel"):
            if name == args.model:
                continue
            configure(vp, rp, name, nsm, args.split)
            rp.run(stream)
            bt, bst, _ = time_steps(torch, rp, max(1, min(args.steps, 3)), stream)
            bt_t = torch.tensor([bt], dtype=torch.float64, device="cuda")
            if world > 1:
                dist.all_reduce(bt_t, op=dist.ReduceOp.MAX)
            extra[name] = {"ms_per_step": float(bt_t.item()) / max(1, min(args.steps, 3)),
                           "launches_per_step": int(bst["kbk_launches"])}
            if name == "kbk_graph":
                # kbk_launches = graph iterations x S wave kernels; each iteration also runs S
                # planner kernels and one loop-condition kernel
                n_st = 4  # Reyes stages
                extra[name]["launches_per_step"] = 2 * int(bst["kbk_launches"]) + int(bst["kbk_launches"]) // n_st
        rp.p.configure_config(main_cfg)

    # ---- e2e through the public API with HOST buffers: every step uploads all of its seed
    # items and camera matrices from pinned host memory and downloads every colour buffer
    # (workloads.ReyesStream: chunks of frames, copies on two copy streams overlapping the
    # runs of the previous / next chunk, same tuned configuration)
    e2e = None
    if not args.no_e2e:
        from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesStream
        rs = ReyesStream(scene, chunk=args.e2e_chunk)
        rs.configure_config(main_cfg)
        host_seeds = ReyesStream.host_seeds(scene)
        host_M = torch.from_numpy(np.ascontiguousarray(scene.M, np.float32)).pin_memory()
        host_out = torch.empty((scene.n_frames, scene.H, scene.W, 4), dtype=torch.float32).pin_memory()
        e_steps = max(1, min(args.steps, 5))
        rs.render(host_seeds, host_M, host_out, stream=stream, steps=1)
        barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        rs.render(host_seeds, host_M, host_out, stream=stream, steps=e_steps)
        e1.record(stream)
        torch.cuda.synchronize()
        et = torch.tensor([e0.elapsed_time(e1)], dtype=torch.float64, device="cuda")
        if world > 1:
            dist.all_reduce(et, op=dist.ReduceOp.MAX)
        e2e = {"value": frames_all * e_steps / (float(et.item()) / 1e3), "unit": "frames/s",
               "h2d_bytes_per_step": (int(host_seeds.numel()) + int(host_M.numel()) * 4) * world,
               "d2h_bytes_per_step": int(host_out.numel() * 4) * world, "steps": e_steps,
               "chunk_frames": args.e2e_chunk,
               "how": "workloads.ReyesStream: pinned host seeds + matrices -> device, vp_run per chunk "
                      "(vp_set_params), colours -> pinned host; copies overlap the neighbouring chunks' runs"}
        # the e2e output is the same render: spot-check it against the timed run's snapshot
        e2e["matches_timed_run"] = bool(all(np.array_equal(host_out[f - f0].numpy(), snap[f][2]) for f in snap))
        del rs

    # ---- NCCL output gather (config 5), timed separately
    gather_ms = None
    if world > 1:
        barrier()
        g0, g1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        g0.record(stream)
        out = shard.gather_frames(rp.colour, args.frames)  # NCCL over NVLink
        g1.record(stream)
        torch.cuda.synchronize()
        assert out.shape[0] == args.frames
        gather_ms = shard.max_over_ranks(g0.elapsed_time(g1), "cuda")

    suite = None
    qbench = None
    if world == 1 and not args.no_suite:
        try:
            suite = workload_suite(torch, vp, stream, args.suite_tune_seconds, pk.get("hbm_gbs", 6548.5))
        except Exception as ex:  # secondary numbers must never lose the headline line
            suite = {"error": repr(ex)}
    if world == 1 and not args.no_qbench:
        try:
            qbench = queue_microbench(torch, vp, stream)
        except Exception as ex:
            qbench = {"error": repr(ex)}

    cpu = None
    parity = {"pass": None, "checked": "only at N=1 (the oracle runs on rank 0 at N=1)"}
    if rank == 0 and world == 1:
        try:
            cpu, ref = cpu_oracle_sample(args.frames, args.cpu_seconds, must=sorted(snap))
            parity = parity_check(snap, ref)
        except Exception as ex:  # the oracle is a reported baseline only
            cpu = {"value": None, "unit": "frames/s", "cores": os.cpu_count(), "kind": "oracle",
                   "sample": f"failed: {ex}"}
            parity = {"pass": False, "error": repr(ex)}

    launches = 3 + nk + int(st["kbk_launches"])   # run-init, fb clear, resolve + kernels + waves
    line = {
        "metric": "frames/sec", "value": fps, "unit": "frames/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": {"workload": "reyes_batch_config5", "frames": args.frames, "frames_per_gpu": f1 - f0,
                   "patches_per_frame": 4096, "image": "256x256", "max_depth": 8, "model": args.model,
                   "parallelism": f"frames sharded over {world} GPU(s)",
                   "l2": "inputs larger than L2 (seeds %.0f MB/GPU, frame buffers %.0f MB/GPU)" % (
                       scene.seeds.size * inputs.GPU_PATCH_DTYPE.itemsize / 1e6, npix * 32 / 1e6)},
        "items_per_sec": ips, "items_per_step": items_all,
        "stage_counts": [int(x) for x in d[:4]],
        "roofline": roofline,
        "hbm": {"min_bytes_per_step": bytes_step * world, "achieved_gbs": bytes_step * world / (ms_per_step / 1e3) / 1e9,
                "pct_of_measured": 100.0 * bytes_step * world / (ms_per_step / 1e3) / 1e9 / hbm,
                "note": "ALU/latency-bound workload (SURVEY §8(d) d5); % HBM reported, not the bound"},
        "speedup_vs_kbk": (extra["kbk"]["ms_per_step"] / ms_per_step) if "kbk" in extra else None,
        "speedup_vs_kbk_graph": (extra["kbk_graph"]["ms_per_step"] / ms_per_step) if "kbk_graph" in extra else None,
        "baselines": extra, "e2e": e2e, "gather_ms": gather_ms, "clocks": clocks, "gpu_launches": launches * args.steps,
        "cpu_baseline": cpu, "parity": parity, "device": f"sm_{cc[0]}{cc[1]} x{nsm} SMs", "autotune": tune,
        "workloads": suite,
        "queue_microbench": qbench,
        "config_string": vp.config_to_string(main_cfg),
    }
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
