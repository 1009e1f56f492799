"""Workload assembly through the C ABI (argument marshalling only).

Each class allocates the family's device buffers with PyTorch (plumbing), fills the
vp_*_params struct with raw device pointers, registers the family's stages in order,
inserts the seeded items (insertIntoQueue) and exposes run() and the
sink outputs.  All pipeline work happens inside libvp.so.
"""
from __future__ import annotations

import numpy as np
import torch

from . import inputs, vp


def _dev(device):
    return torch.device("cuda", device)


class ToyPipeline:
    """Fig. 9 (L37): S1 doubles until >= threshold (recursive), S2 adds 1, S3 sink."""

    def __init__(self, seeds: np.ndarray, threshold: int = inputs.TOY_THRESHOLD, device: int = 0, **kw):
        self.n = int(seeds.size)
        self.out = torch.zeros(max(self.n, 1), dtype=torch.int32, device=_dev(device))
        self.n_out = torch.zeros(1, dtype=torch.int64, device=_dev(device))
        self.prm = vp.ToyParams(threshold=threshold, out=self.out.data_ptr(), n_out=self.n_out.data_ptr())
        self.p = vp.Pipeline(device, **kw)
        for kind in (vp.TOY_S1, vp.TOY_S2, vp.TOY_S3):
            self.p.register(kind, 4, self.prm)
        self.p.insert(0, np.ascontiguousarray(seeds, np.int32))

    def configure(self, model, binding=None, batch=0):
        self.p.configure(model, binding, batch)

    def run(self, stream=None):
        st = self.p.run(stream)
        n = int(self.n_out.item())
        return self.out[:n].cpu().numpy(), st


class QBenchPipeline:
    """Queue microbenchmark: n seeds of item_bytes (4 / 16 / 272) into
    the matching self-recursive stage; each task re-enqueues `fanout` copies until depth 0."""

    SIZES = (4, 16, 272)

    def __init__(self, n: int, item_bytes: int, fanout: int, depth: int, device: int = 0, steal: bool = False, **kw):
        """steal: the cluster-work-stealing build of the 4- / 16-B stage (VP_QB_ITEM*_CS with
        VP_FLAG_CLUSTER_STEAL)."""
        self.slot = self.SIZES.index(item_bytes)  # counter slot (vp_qbench_params arrays)
        self.stage = 0                            # one single-stage family per item size
        self.n, self.item_bytes, self.fanout, self.depth = n, item_bytes, fanout, depth
        self.cnt = torch.zeros(9, dtype=torch.int64, device=_dev(device))
        ptr = self.cnt.data_ptr()
        self.prm = vp.QBenchParams(fanout=fanout, depth=depth, leaves=ptr, idsum=ptr + 24, bad=ptr + 48)
        # full rings: a breadth-first fan-out-2 tree's frontier is a whole tree level
        kw["flags"] = kw.get("flags", 0) | vp.FLAG_FULL_RINGS | (vp.FLAG_CLUSTER_STEAL if steal else 0)
        self.p = vp.Pipeline(device, **kw)
        # the ring holds a whole tree level (KBK waves) or chain frontier
        big = 1 << (21 if item_bytes == 272 else 24)
        if steal and item_bytes == 272:
            raise ValueError("no stealing build of the 272-B stage (it has no block-local queue)")
        kind = ((vp.QB_ITEM4_CS, vp.QB_ITEM16_CS) if steal else (vp.QB_ITEM4, vp.QB_ITEM16, vp.QB_ITEM272))[self.slot]
        self.p.register(kind, item_bytes, self.prm, queue_capacity=big)
        self.seeds = inputs.qbench_seeds(n, item_bytes, depth)
        self.p.insert(self.stage, self.seeds, n=n)

    def configure(self, model, binding=None, batch=0):
        self.p.configure(model, binding, batch)

    def tasks(self) -> int:
        per = 1 if self.fanout == 0 else (self.depth + 1 if self.fanout == 1 else (1 << (self.depth + 1)) - 1)
        return self.n * per

    def run(self, stream=None):
        st = self.p.run(stream)
        c = self.cnt.cpu().numpy().astype(np.uint64)
        return {"leaves": int(c[self.slot]), "idsum": int(c[3 + self.slot]), "bad": int(c[6 + self.slot])}, st


class LdpcPipeline:
    """LDPC decoder (Fig. 17, L59): Initialize -> C2V -> V2C -> ProbVar, looping back to C2V
    for n_iter iterations, one item per (frame, iteration)."""

    def __init__(self, scene: inputs.LdpcScene, device: int = 0, **kw):
        dev = _dev(device)
        self.scene = scene
        nf, E = scene.n_frames, scene.N * scene.dv
        self.cv = torch.from_numpy(np.ascontiguousarray(scene.check_vars, np.int32)).to(dev)
        self.ve = torch.from_numpy(np.ascontiguousarray(scene.var_edges, np.int32)).to(dev)
        self.llr = torch.from_numpy(np.ascontiguousarray(scene.llr, np.float32)).to(dev)
        self.v2c = torch.empty((nf, E), dtype=torch.float32, device=dev)
        self.c2v = torch.empty((nf, E), dtype=torch.float32, device=dev)
        self.post = torch.empty((nf, scene.N), dtype=torch.float32, device=dev)
        self.errors = torch.zeros((nf, scene.n_iter), dtype=torch.int32, device=dev)
        self.latch = torch.zeros((nf, 2), dtype=torch.int32, device=dev)
        self.prm = vp.LdpcParams(N=scene.N, M=scene.M, dv=scene.dv, dc=scene.dc, n_frames=nf, n_iter=scene.n_iter,
                                 alpha=scene.alpha, nc_chk=scene.nc_chk, nc_var=scene.nc_var,
                                 check_vars=self.cv.data_ptr(), var_edges=self.ve.data_ptr(),
                                 llr=self.llr.data_ptr(), v2c=self.v2c.data_ptr(), c2v=self.c2v.data_ptr(),
                                 post=self.post.data_ptr(), errors=self.errors.data_ptr(), latch=self.latch.data_ptr())
        self.p = vp.Pipeline(device, **kw)
        for kind in (vp.LDPC_INIT, vp.LDPC_C2V, vp.LDPC_V2C, vp.LDPC_PROBVAR):
            self.p.register(kind, 16, self.prm)
        seeds = np.zeros((nf, 4), np.uint32)
        seeds[:, 0] = np.arange(nf, dtype=np.uint32)
        self.p.insert(0, seeds, n=nf)

    def configure(self, model, binding=None, batch=0):
        self.p.configure(model, binding, batch)

    def run(self, stream=None):
        return self.p.run(stream)

    def results(self):
        return dict(post=self.post.cpu().numpy(), errors=self.errors.cpu().numpy())


class CollatzPipeline:
    def __init__(self, seeds: np.ndarray, max_steps: int = 1000, device: int = 0, **kw):
        n = int(seeds.size)
        self.steps = torch.zeros(n, dtype=torch.int32, device=_dev(device))
        self.seen = torch.zeros(n, dtype=torch.int32, device=_dev(device))
        self.prm = vp.CollatzParams(steps_out=self.steps.data_ptr(), seen=self.seen.data_ptr(), n_ids=n,
                                    max_steps=max_steps)
        self.p = vp.Pipeline(device, **kw)
        self.p.register(vp.COLLATZ_STEP, 16, self.prm)
        self.p.register(vp.COLLATZ_SINK, 16, self.prm)
        self.p.insert(0, np.ascontiguousarray(seeds))

    def configure(self, model, binding=None, batch=0):
        self.p.configure(model, binding, batch)

    def run(self, stream=None):
        st = self.p.run(stream)
        return self.steps.cpu().numpy().view(np.uint32), self.seen.cpu().numpy().view(np.uint32), st


class RasterPipeline:
    """Vertex -> Clip -> Raster -> Fragment (+ colour resolve) over a RasterScene (Fig. 16, L59)."""

    def __init__(self, scene: inputs.RasterScene, device: int = 0, tri_range=None, **kw):
        """tri_range = (lo, hi): seed only triangles [lo, hi) (a rank's shard);
        keys keep the global triangle ids."""
        dev = _dev(device)
        self.scene = scene
        n = scene.n_tris
        self.M = torch.from_numpy(np.ascontiguousarray(scene.M, np.float32)).to(dev)
        self.pos = torch.from_numpy(np.ascontiguousarray(scene.pos, np.float32)).to(dev)
        self.col = torch.from_numpy(np.ascontiguousarray(scene.col, np.float32)).to(dev)
        near = int(getattr(scene, "near_clip", 0))
        nsub = n * (2 if near else 1)                                                 # sub-triangles 2 tri + j
        self.setup = torch.empty((nsub, 32), dtype=torch.float32, device=dev)       # 128 B per (sub-)triangle
        self.ccol = torch.empty((nsub if near else 1, 12), dtype=torch.float32, device=dev)
        self.fb = torch.empty((scene.H, scene.W), dtype=torch.int64, device=dev)
        self.colour = torch.empty((scene.H, scene.W, 4), dtype=torch.float32, device=dev)
        self.prm = vp.RasterParams(W=scene.W, H=scene.H, n_tris=n, M=self.M.data_ptr(), pos=self.pos.data_ptr(),
                                   col=self.col.data_ptr(), setup=self.setup.data_ptr(), fb=self.fb.data_ptr(),
                                   colour=self.colour.data_ptr(), near_clip=near,
                                   ccol=self.ccol.data_ptr())
        self.p = vp.Pipeline(device, **kw)
        for kind, stride in zip((vp.RASTER_VERTEX, vp.RASTER_CLIP, vp.RASTER_RASTER, vp.RASTER_FRAGMENT), (4, 4, 4, 8)):
            self.p.register(kind, stride, self.prm)
        lo, hi = tri_range if tri_range is not None else (0, n)
        self.ids = torch.arange(lo, hi, dtype=torch.int32, device=dev)
        self.p.insert(0, self.ids, n=hi - lo)

    def configure(self, model, binding=None, batch=0):
        self.p.configure(model, binding, batch)

    def run(self, stream=None):
        return self.p.run(stream)

    def keys(self):
        return self.fb.cpu().numpy().view(np.uint64)

    def colours(self):
        return self.colour.cpu().numpy()


def pyramid_levels(S):
    L = 0
    while (S >> L) >= 1:
        L += 1
    return L


def pyramid_latches_per_img(S):
    n = 1
    for l in range(1, pyramid_levels(S)):
        t = max(1, (S >> l) // 64)
        n += t * t
    return n


class PyramidPipeline:
    """Grayscale -> HistEq (CDF, Map) -> Resize (recursive) over n_img RGB8 images (Fig. 12, L53)."""

    def __init__(self, rgb: np.ndarray, device: int = 0, rgb_on_device=None, **kw):
        dev = _dev(device)
        n, S = rgb.shape[0], rgb.shape[1]
        self.n_img, self.S = n, S
        self.total = sum((S >> l) ** 2 for l in range(pyramid_levels(S)))
        self.stride = (self.total + 127) // 128 * 128
        self.rgb = rgb_on_device if rgb_on_device is not None else torch.from_numpy(np.ascontiguousarray(rgb)).to(dev)
        self.gray = torch.empty((n, S * S), dtype=torch.uint8, device=dev)
        self.pyr = torch.empty((n, self.stride), dtype=torch.uint8, device=dev)
        self.hist = torch.empty((n, 256), dtype=torch.int32, device=dev)
        self.lut = torch.empty((n, 256), dtype=torch.uint8, device=dev)
        self.latch = torch.empty((n, pyramid_latches_per_img(S)), dtype=torch.int32, device=dev)
        self.prm = vp.PyramidParams(S=S, n_img=n, rgb=self.rgb.data_ptr(), gray=self.gray.data_ptr(),
                                    pyr=self.pyr.data_ptr(), hist=self.hist.data_ptr(), lut=self.lut.data_ptr(),
                                    latch=self.latch.data_ptr())
        self.p = vp.Pipeline(device, **kw)
        for kind in (vp.PYR_GRAY, vp.PYR_CDF, vp.PYR_MAP, vp.PYR_RESIZE):
            self.p.register(kind, 16, self.prm)
        nt = S // 64
        ii, yy, xx = np.meshgrid(np.arange(n), np.arange(nt), np.arange(nt), indexing="ij")
        seeds = np.zeros((n * nt * nt, 4), np.uint32)
        seeds[:, 0], seeds[:, 2], seeds[:, 3] = ii.ravel(), yy.ravel(), xx.ravel()
        self.p.insert(0, seeds, n=seeds.shape[0])

    def configure(self, model, binding=None, batch=0):
        self.p.configure(model, binding, batch)

    def run(self, stream=None):
        return self.p.run(stream)

    def pyramid(self):
        return self.pyr.cpu().numpy()[:, : self.total]


class CfdPipeline:
    """Copy -> StepFactor -> 3 x (Flux -> TimeStep), looped (Fig. 15, L55; Rodinia euler3d)."""

    def __init__(self, scene: inputs.CfdScene, device: int = 0, **kw):
        dev = _dev(device)
        self.scene = scene
        N = scene.n_cells
        t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).to(dev)
        self.vars0, self.area, self.nb, self.normals = t(scene.vars0), t(scene.area), t(scene.nb), t(scene.normals)
        self.vars = torch.empty((2, 5, N), dtype=torch.float32, device=dev)
        self.old = torch.empty((5, N), dtype=torch.float32, device=dev)
        self.sf = torch.empty((N,), dtype=torch.float32, device=dev)
        self.flux = torch.empty((5, N), dtype=torch.float32, device=dev)
        self.ntiles = N // scene.T
        self.latch = torch.empty((2, self.ntiles), dtype=torch.int32, device=dev)
        self.prm = vp.CfdParams(G=scene.G, T=scene.T, n_outer=scene.n_outer, vars0=self.vars0.data_ptr(),
                                vars=self.vars.data_ptr(), old=self.old.data_ptr(), sf=self.sf.data_ptr(),
                                flux=self.flux.data_ptr(), area=self.area.data_ptr(), nb=self.nb.data_ptr(),
                                normals=self.normals.data_ptr(), latch=self.latch.data_ptr())
        for i in range(5):
            self.prm.ff[i] = float(scene.ff[i])
        self.p = vp.Pipeline(device, **kw)
        for kind in (vp.CFD_COPY, vp.CFD_STEP_FACTOR, vp.CFD_FLUX, vp.CFD_TIME_STEP):
            self.p.register(kind, 16, self.prm)
        seeds = np.zeros((self.ntiles, 4), np.uint32)
        seeds[:, 0] = np.arange(self.ntiles)
        if scene.n_outer > 0:
            self.p.insert(0, seeds, n=self.ntiles)

    def configure(self, model, binding=None, batch=0):
        self.p.configure(model, binding, batch)

    def run(self, stream=None):
        return self.p.run(stream)

    def state(self):
        return self.vars[(3 * self.scene.n_outer) & 1].cpu().numpy()


def face_levels(W, H):
    out, w, h = [], W, H
    while len(out) < 8 and w >= 24 and h >= 24:
        out.append((w, h))
        w, h = 4 * w // 5, 4 * h // 5
    return out


class FaceDetPipeline:
    """Gray -> HistEq (CDF, Map) -> Resize (recursive) -> LBP -> Scan over RGB frames (Fig. 14, L55)."""

    def __init__(self, scene: inputs.FaceScene, device: int = 0, det_cap: int = 1 << 20, **kw):
        dev = _dev(device)
        self.scene = scene
        F, W, H = scene.n_frames, scene.W, scene.H
        lv = face_levels(W, H)
        per = sum(w * h for w, h in lv)
        bands = [-(-h // 32) for _, h in lv]
        self.rgb = torch.from_numpy(np.ascontiguousarray(scene.rgb)).to(dev)
        self.levels = torch.empty((F, per), dtype=torch.uint8, device=dev)
        self.lbp = torch.empty((F, per), dtype=torch.uint8, device=dev)
        self.hist = torch.empty((F, 256), dtype=torch.int32, device=dev)
        self.lut = torch.empty((F, 256), dtype=torch.uint8, device=dev)
        self.weak = torch.from_numpy(np.ascontiguousarray(scene.weak)).to(dev)
        self.det = torch.empty((det_cap, 4), dtype=torch.int32, device=dev)
        self.counters = torch.zeros(32, dtype=torch.int64, device=dev)   # [0] det_count, [1] windows, [16:32] survivors
        self.latch = torch.empty((F, 1 + 3 * sum(bands)), dtype=torch.int32, device=dev)
        base = self.counters.data_ptr()
        self.prm = vp.FaceDetParams(W=W, H=H, n_frames=F, n_stages=len(scene.n_weak),
                                    n_weak_total=int(scene.n_weak.sum()), rgb=self.rgb.data_ptr(),
                                    levels=self.levels.data_ptr(), lbp=self.lbp.data_ptr(),
                                    hist=self.hist.data_ptr(), lut=self.lut.data_ptr(), weak=self.weak.data_ptr(),
                                    det=self.det.data_ptr(), det_count=base, det_cap=det_cap,
                                    survivors=base + 16 * 8, windows=base + 8, latch=self.latch.data_ptr())
        for k, (n, t) in enumerate(zip(scene.n_weak, scene.thr)):
            self.prm.n_weak[k], self.prm.thr[k] = int(n), int(t)
        self.p = vp.Pipeline(device, **kw)
        for kind in (vp.FD_GRAY, vp.FD_CDF, vp.FD_MAP, vp.FD_RESIZE, vp.FD_LBP, vp.FD_SCAN):
            self.p.register(kind, 16, self.prm)
        seeds = np.zeros((F * bands[0], 4), np.uint32)
        seeds[:, 0] = np.repeat(np.arange(F), bands[0])
        seeds[:, 2] = np.tile(np.arange(bands[0]), F)
        self.p.insert(0, seeds, n=seeds.shape[0])

    def configure(self, model, binding=None, batch=0):
        self.p.configure(model, binding, batch)

    def run(self, stream=None):
        return self.p.run(stream)

    def results(self):
        c = self.counters.cpu().numpy()
        n = int(c[0])
        det = self.det[: min(n, self.det.shape[0])].cpu().numpy().astype(np.int64)
        return dict(det=det, n_det=n, windows=int(c[1]), survivors=[int(x) for x in c[16:16 + len(self.scene.n_weak)]])


REYES_STAGES = (vp.REYES_BOUND, vp.REYES_SPLIT, vp.REYES_DICE, vp.REYES_SHADE)
# 208-B patches (R-S10) for Bound / Split / Dice; Shade's grid item as the library defines it
REYES_STRIDES = tuple(vp.stage_kind_info(k)[0] for k in REYES_STAGES)
assert REYES_STRIDES[:3] == (inputs.GPU_PATCH_DTYPE.itemsize,) * 3


class ReyesPipeline:
    """Reyes Bound -> Split (recursive) | Dice -> Shade (Fig. 1, L3) over a ReyesScene."""

    def __init__(self, scene: inputs.ReyesScene, device: int = 0, seeds_on_device: bool = True,
                 queue_caps=None, **kw):
        dev = _dev(device)
        self.scene = scene
        self.npix = scene.n_frames * scene.W * scene.H
        self.M = torch.from_numpy(np.ascontiguousarray(scene.M, np.float32)).to(dev)
        self.albedo = torch.from_numpy(np.ascontiguousarray(scene.albedo, np.float32)).to(dev)
        self.fb = torch.empty((self.npix, 4), dtype=torch.int32, device=dev)       # {u64 key, f32 s, pad}
        self.colour = torch.empty((scene.n_frames, scene.H, scene.W, 4), dtype=torch.float32, device=dev)
        L = [float(np.float32(v)) for v in scene.light]
        self.prm = vp.ReyesParams(W=scene.W, H=scene.H, n_frames=scene.n_frames,
                                  patches_per_frame=scene.patches_per_frame, max_depth=scene.max_depth,
                                  t_dice=scene.t_dice, near_w=scene.near_w, M=self.M.data_ptr(),
                                  albedo=self.albedo.data_ptr(), fb=self.fb.data_ptr(),
                                  colour=self.colour.data_ptr())
        for i in range(4):
            self.prm.L[i] = L[i]
        self.p = vp.Pipeline(device, **kw)
        caps = queue_caps or [0, 0, 0, 0]
        for kind, stride, cap in zip(REYES_STAGES, REYES_STRIDES, caps):
            self.p.register(kind, stride, self.prm, queue_capacity=cap)
        seeds = scene.seeds if scene.seeds.dtype == inputs.GPU_PATCH_DTYPE else inputs.gpu_patch_items(scene.seeds)
        seeds = np.ascontiguousarray(seeds)
        if seeds_on_device:
            self.seeds_dev = torch.from_numpy(seeds.view(np.uint8).reshape(-1)).to(dev)
            self.p.insert(0, self.seeds_dev, n=seeds.size)
        else:
            self.p.insert(0, seeds, n=seeds.size)

    def configure(self, model, binding=None, batch=0):
        self.p.configure(model, binding, batch)

    def run(self, stream=None):
        return self.p.run(stream)

    def keys(self):
        fb = self.fb.cpu().numpy()
        key = fb[:, :2].copy().view(np.uint64).reshape(self.scene.n_frames, self.scene.H, self.scene.W)
        s = fb[:, 2].copy().view(np.float32).reshape(self.scene.n_frames, self.scene.H, self.scene.W)
        return key, s

    def colours(self):
        return self.colour.cpu().numpy()


class ReyesStream:
    """End-to-end rendering of a frame batch whose inputs and outputs live in (pinned) host
    memory: the user-facing path behind bench.py's `e2e`.

    The batch is cut into chunks of `chunk` frames rendered by two pipelines in turn.  The
    seed upload of chunk i+1 (copy stream) and the colour download of chunk i-1 (a second
    copy stream) run while chunk i renders on the compute stream; vp_set_params moves each
    pipeline to its chunk (vp_reyes_params.frame_base and the chunk's matrices), so the
    seed items keep their batch-wide frame ids.  All rendering happens in libvp.so (the
    same vp_run as a resident batch); this class only orders copies, events and runs."""

    def __init__(self, scene: inputs.ReyesScene, chunk: int, config=None, device: int = 0):
        import dataclasses
        F, ppf = scene.n_frames, scene.patches_per_frame
        if F % chunk:
            raise ValueError(f"{F} frames are not a multiple of the chunk ({chunk})")
        dev = _dev(device)
        self.scene, self.chunk, self.n_chunks, self.dev = scene, chunk, F // chunk, dev
        sub = dataclasses.replace(scene, n_frames=chunk, M=scene.M[:chunk], seeds=scene.seeds[:chunk * ppf])
        self.pipes = [ReyesPipeline(sub, device) for _ in range(2)]
        if config is not None:
            for rp in self.pipes:
                rp.p.configure_config(config)
        self.seed_bytes = chunk * ppf * inputs.GPU_PATCH_DTYPE.itemsize
        self.M_dev = torch.empty((2, F, 16), dtype=torch.float32, device=dev)  # per pass parity
        self.staging = [torch.empty(self.seed_bytes, dtype=torch.uint8, device=dev) for _ in range(2)]
        self.s_in, self.s_out = torch.cuda.Stream(dev), torch.cuda.Stream(dev)
        self.ev_in = [torch.cuda.Event() for _ in range(2)]      # chunk's seeds landed in staging[b]
        self.ev_used = [torch.cuda.Event() for _ in range(2)]    # staging[b] copied into pipeline b
        self.ev_out = [torch.cuda.Event() for _ in range(2)]     # pipeline b's colours downloaded
        self.ev_M = [torch.cuda.Event() for _ in range(2)]   # a pass's last chunk has rendered

    @staticmethod
    def host_seeds(scene: inputs.ReyesScene) -> torch.Tensor:
        """The batch's seed items as the queues carry them (208-B records), in pinned host
        memory: the `host_seeds` argument of render()."""
        return torch.from_numpy(inputs.gpu_patch_items(scene.seeds).view(np.uint8).reshape(-1).copy()).pin_memory()

    def configure(self, model, binding=None, batch=0):
        for rp in self.pipes:
            rp.configure(model, binding, batch)

    def configure_config(self, cfg):
        for rp in self.pipes:
            rp.p.configure_config(cfg)

    def _params(self, b, c, k):
        rp = self.pipes[b]
        prm = rp.prm
        prm.frame_base = c * self.chunk
        prm.M = self.M_dev[k & 1].data_ptr() + c * self.chunk * 16 * 4
        rp.p.set_params(prm)

    def render(self, host_seeds: torch.Tensor, host_M: torch.Tensor, host_out: torch.Tensor, stream=None,
               steps: int = 1):
        """`steps` passes over the batch: host_seeds (pinned uint8, every frame's 208-B seed
        items, see host_seeds()),
        host_M (pinned [F, 16] float32) -> host_out (pinned [F, H, W, 4] float32).  Copies of
        consecutive passes overlap too.  Returns the last run's stats."""
        st = stream or torch.cuda.current_stream(self.dev)
        nC = self.n_chunks
        out = host_out.view(nC, -1)
        seeds = host_seeds.view(nC, -1)
        total = steps * nC
        st_last = None

        def upload(j):
            b, c, k = j & 1, j % nC, j // nC
            with torch.cuda.stream(self.s_in):
                if c == 0:  # this pass's matrices (64 B per frame), ahead of its first chunk
                    self.s_in.wait_event(self.ev_M[k & 1])   # pass k-2 is done with this buffer
                    self.M_dev[k & 1].copy_(host_M, non_blocking=True)
                self.s_in.wait_event(self.ev_used[b])
                self.staging[b].copy_(seeds[c], non_blocking=True)
                self.ev_in[b].record(self.s_in)

        upload(0)
        for j in range(total):
            b, c, k = j & 1, j % nC, j // nC
            rp = self.pipes[b]
            if j + 1 < total:
                upload(j + 1)
            st.wait_event(self.ev_in[b])     # seeds (and matrices) of chunk c are on the device
            st.wait_event(self.ev_out[b])    # pipeline b's previous colours are downloaded
            self._params(b, c, k)
            rp.p.insert(0, self.staging[b], n=self.seed_bytes // inputs.GPU_PATCH_DTYPE.itemsize, replace=True,
                        stream=st)
            self.ev_used[b].record(st)
            st_last = rp.run(st)             # vp_run returns when the chunk is rendered
            if c == nC - 1:
                self.ev_M[k & 1].record(st)  # this pass is done with its matrices
            with torch.cuda.stream(self.s_out):
                self.s_out.wait_stream(st)
                out[c].copy_(rp.colour.view(-1), non_blocking=True)
                self.ev_out[b].record(self.s_out)
        st.wait_stream(self.s_out)           # events recorded on `st` now cover the downloads
        return st_last


class PyramidKbkStreams:
    """The paper's "KBK with Stream" baseline (Fig. 13): the images are
    split over n_streams independent KBK pipelines, each driven by its own host thread on
    its own CUDA stream, so kernels of different images overlap (the limited parallelism
    of one image's KBK waves is the problem it addresses).  Same stage kernels and wave
    loop as VP_KBK (or VP_KBK_GRAPH); no queue is shared between streams."""

    def __init__(self, rgb_dev: torch.Tensor, n_streams: int, model=None, device: int = 0):
        n = rgb_dev.shape[0]
        self.n_streams = max(1, min(n_streams, n))
        bounds = np.linspace(0, n, self.n_streams + 1).astype(int)
        self.pipes = [PyramidPipeline(rgb_dev[a:b], device=device, rgb_on_device=rgb_dev[a:b])
                      for a, b in zip(bounds[:-1], bounds[1:])]
        for pp in self.pipes:
            pp.configure(vp.KBK if model is None else model)
        self.streams = [torch.cuda.Stream(_dev(device)) for _ in self.pipes]

    def run(self, stream=None):
        """One pass over every image; the caller's stream is ordered after all of them."""
        import threading
        st = stream or torch.cuda.current_stream()
        for s in self.streams:
            s.wait_stream(st)
        errs = []

        def go(pp, s):
            try:
                pp.run(s)
            except Exception as ex:  # re-raised in the caller
                errs.append(ex)

        th = [threading.Thread(target=go, args=(pp, s)) for pp, s in zip(self.pipes, self.streams)]
        for t in th:
            t.start()
        for t in th:
            t.join()
        if errs:
            raise errs[0]
        for s in self.streams:
            st.wait_stream(s)

    def pyramid(self):
        return np.concatenate([pp.pyramid() for pp in self.pipes])
