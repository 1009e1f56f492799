"""Small runs of every workload family under the megakernel and a hybrid / coarse model,
for compute-sanitizer (memcheck, racecheck, synccheck, initcheck).

  compute-sanitizer --tool memcheck python tools/sanitize_run.py [--models mega,hybrid]

Sizes are reduced (the tools slow kernels down by 10-100x); the watchdog is raised and the
co-residency check still applies to the multi-kernel plans.  Each run's outputs are
compared with the CPU oracle so a sanitizer pass is also a parity pass."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np

import oracle
from paper_conf_micro_zhengozsyc17_b200 import inputs, vp
from paper_conf_micro_zhengozsyc17_b200 import workloads as W

ap = argparse.ArgumentParser()
ap.add_argument("--models", default="mega,hybrid")
ap.add_argument("--only", default="")
args = ap.parse_args()
nsm, _ = vp.device_info(0)
h = nsm // 2
KW = dict(watchdog_ms=600000)


def conf(pipe, model, groups):
    if model == "mega":
        pipe.configure(vp.MEGAKERNEL)
    elif model == "kbk":
        pipe.configure(vp.KBK)
    else:
        pipe.configure(vp.HYBRID, vp.make_binding(groups, nsm))


def toy(model):
    s = inputs.toy_seeds(2000)
    p = W.ToyPipeline(s, **KW)
    conf(p, model, [(0, 0, vp.GROUP_MEGA, 0, 16), (1, 2, vp.GROUP_RTC, 16, nsm)])
    out, st = p.run()
    ref, deq, _ = oracle.toy_pipeline(s, inputs.TOY_THRESHOLD)
    return np.array_equal(np.sort(out), np.sort(ref)) and st["dequeued"][:3] == deq


def collatz(model):
    s = inputs.collatz_seeds(3000)
    p = W.CollatzPipeline(s, **KW)
    conf(p, model, [(0, 0, vp.GROUP_MEGA, 0, h), (1, 1, vp.GROUP_MEGA, h, nsm)])
    steps, seen, _ = p.run()
    return np.array_equal(steps, oracle.collatz_definition(s)) and np.all(seen == 1)


def reyes(model):
    sc = inputs.reyes_config1()
    p = W.ReyesPipeline(sc, **KW)
    conf(p, model, [(0, 1, vp.GROUP_MEGA, 0, h), (2, 3, vp.GROUP_RTC, h, nsm)])
    p.run()
    key, _ = p.keys()
    return np.array_equal(key, oracle.reyes_pipeline(sc)["key"])


def raster(model):
    sc = inputs.raster_scene(3000, W=160, H=96)
    p = W.RasterPipeline(sc, **KW)
    conf(p, model, [(0, 1, vp.GROUP_RTC, 0, 40), (2, 3, vp.GROUP_MEGA, 40, nsm)])
    p.run()
    return np.array_equal(p.keys(), oracle.raster_pipeline(sc)["key"])


def pyramid(model):
    rgb = inputs.pyramid_images(2, 256)
    p = W.PyramidPipeline(rgb, **KW)
    conf(p, model, [(0, 1, vp.GROUP_MEGA, 0, 40), (2, 3, vp.GROUP_MEGA, 40, nsm)])
    p.run()
    return np.array_equal(p.pyramid(), oracle.pyr_pipeline(rgb)["pyr"])


def cfd(model):
    sc = inputs.cfd_scene(G=64, n_outer=2)
    p = W.CfdPipeline(sc, **KW)
    conf(p, model, [(0, 1, vp.GROUP_MEGA, 0, 40), (2, 3, vp.GROUP_MEGA, 40, nsm)])
    p.run()
    return np.array_equal(p.state(), oracle.cfd_pipeline(sc)["vars"])


def facedet(model):
    sc = inputs.face_scene(W=240, H=136, n_planted=4)
    p = W.FaceDetPipeline(sc, **KW)
    conf(p, model, [(0, 2, vp.GROUP_MEGA, 0, 40), (3, 5, vp.GROUP_MEGA, 40, nsm)])
    p.run()
    ref = oracle.fd_pipeline(sc, det_cap=1 << 20)
    return sorted(map(tuple, p.results()["det"].tolist())) == sorted(map(tuple, ref["det"].astype(np.int64).tolist()))


def ldpc(model):
    sc = inputs.ldpc_scene(n_frames=4, n_iter=5)
    p = W.LdpcPipeline(sc, **KW)
    conf(p, model, [(0, 1, vp.GROUP_MEGA, 0, 40), (2, 3, vp.GROUP_MEGA, 40, nsm)])
    p.run()
    return np.array_equal(p.results()["post"], oracle.ldpc_pipeline(sc)["post"])


ok_all = True
def qbench(model):
    # single-stage family: "hybrid" runs it as KBK waves (one group, nothing to bind)
    ok = True
    for ib in (4, 16, 272):
        p = W.QBenchPipeline(64, ib, 2, 6, **KW)
        p.configure(vp.MEGAKERNEL if model == "mega" else vp.KBK)
        lv, ids, _, deq = oracle.qbench_pipeline(p.seeds, ib, 2)
        r, st = p.run()
        ok &= (r["leaves"], r["idsum"], r["bad"]) == (lv, ids, 0) and st["dequeued"][p.stage] == deq
    return ok


for name, fn in (("toy", toy), ("collatz", collatz), ("reyes", reyes), ("raster", raster), ("pyramid", pyramid),
                 ("cfd", cfd), ("facedet", facedet), ("ldpc", ldpc), ("qbench", qbench)):
    if args.only and name not in args.only.split(","):
        continue
    for m in args.models.split(","):
        try:
            ok = bool(fn(m))
        except Exception as ex:  # report and continue: the sanitizer log is the product here
            ok = False
            print(f"{name} {m}: EXCEPTION {ex!r}", flush=True)
        ok_all &= ok
        print(f"{name} {m}: {'ok' if ok else 'MISMATCH'}", flush=True)
print("ALL OK" if ok_all else "SOME FAILED", flush=True)
