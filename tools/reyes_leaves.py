"""Dev tool (profiling inputs only, not a parity reference): approximate the Reyes
Bound/Split recursion in numpy (float64) to obtain a representative set of diceable leaf
patches, so the [Dice, Shade] kernel can be captured alone under ncu with the same item
mix the full pipeline feeds it (ncu serialises the co-running persistent groups)."""
import numpy as np

from paper_conf_micro_zhengozsyc17_b200 import inputs


def _casteljau(P, axis):
    p = [np.take(P, i, axis=axis) for i in range(4)]
    ab, bc, cd = (p[0] + p[1]) * 0.5, (p[1] + p[2]) * 0.5, (p[2] + p[3]) * 0.5
    abc, bcd = (ab + bc) * 0.5, (bc + cd) * 0.5
    m = (abc + bcd) * 0.5
    return np.stack([p[0], ab, abc, m], axis=axis), np.stack([m, bcd, cd, p[3]], axis=axis)


def leaves(scene: inputs.ReyesScene, frames: int) -> np.ndarray:
    ppf, W, H = scene.patches_per_frame, scene.W, scene.H
    out = []
    for f in range(frames):
        M = scene.M[f].reshape(4, 4).astype(np.float64)
        P = scene.seeds["cp"][f * ppf:(f + 1) * ppf].astype(np.float64).reshape(-1, 4, 4, 4)
        pid = np.arange(ppf, dtype=np.uint32)
        depth = 0
        while len(P):
            c = P @ M.T
            w = c[..., 3]
            behind = ~(w > scene.near_w)
            nb = behind.reshape(len(P), -1).sum(1)
            with np.errstate(all="ignore"):
                sx = (c[..., 0] / w * 0.5 + 0.5) * W
                sy = (c[..., 1] / w * 0.5 + 0.5) * H
            sxf, syf = sx.reshape(len(P), -1), sy.reshape(len(P), -1)
            xmin, xmax, ymin, ymax = sxf.min(1), sxf.max(1), syf.min(1), syf.max(1)
            off = (xmax < 0) | (xmin >= W) | (ymax < 0) | (ymin >= H)
            ext = np.maximum(xmax - xmin, ymax - ymin)
            lu = (np.abs(sx[:, 3] - sx[:, 0]) + np.abs(sy[:, 3] - sy[:, 0])).max(1)
            lv = (np.abs(sx[:, :, 3] - sx[:, :, 0]) + np.abs(sy[:, :, 3] - sy[:, :, 0])).max(1)
            ou = np.abs(P[:, 3, :, :3] - P[:, 0, :, :3]).sum(-1).max(1)
            ov = np.abs(P[:, :, 3, :3] - P[:, :, 0, :3]).sum(-1).max(1)
            dice = (nb == 0) & ~off & ((ext <= scene.t_dice) | (depth >= scene.max_depth))
            split = ((nb > 0) & (nb < 16) & (depth < scene.max_depth)) | ((nb == 0) & ~off & ~dice)
            udir = np.where(nb > 0, ou >= ov, lu >= lv)
            if dice.any():
                it = np.zeros(int(dice.sum()), inputs.PATCH_DTYPE)
                it["cp"] = P[dice].reshape(-1, 16, 4).astype(np.float32)
                it["id"] = (np.uint32(f) << 12) | pid[dice]
                it["depth"] = depth
                out.append(it)
            Ps, ids, us = P[split], pid[split], udir[split]
            kids, kid_ids = [], []
            for sel, axis in ((us, 1), (~us, 2)):
                if sel.any():
                    L, R = _casteljau(Ps[sel], axis)
                    kids += [L, R]
                    kid_ids += [ids[sel], ids[sel]]
            P = np.concatenate(kids) if kids else P[:0]
            pid = np.concatenate(kid_ids) if kid_ids else pid[:0]
            depth += 1
    return np.concatenate(out)
