"""Seeded synthetic input generators shared by the CUDA path and the CPU oracle.

This module holds NO arithmetic of the method (no projection, no bound/split/dice/
shade, no queueing).  It only draws seeded random numbers and lays them out in the
byte layouts both sides consume (DESIGN.md §3 "Input recipes").  Camera matrices are
scene *inputs* (computed in float64 with trigonometry, then rounded to float32),
exactly as SURVEY §8(d) "Common protocol" prescribes: anything needing sin/cos is
computed on the host and stored as float data.

Random numbers: SplitMix64 (Steele, Lea, Flood 2014), floats from the top 24 bits:
``(x >> 40) * 2**-24``.  Seed convention: ``0x56500000 + 256*config + rep``.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np

GOLDEN = np.uint64(0x9E3779B97F4A7C15)


def seed_for(config: int, rep: int = 0) -> int:
    return 0x56500000 + 256 * config + rep


def splitmix64(seed: int, n: int) -> np.ndarray:
    """n successive SplitMix64 outputs for a generator started at ``seed``."""
    with np.errstate(over="ignore"):
        i = np.arange(1, n + 1, dtype=np.uint64)
        z = np.uint64(seed & 0xFFFFFFFFFFFFFFFF) + i * GOLDEN
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    return z


def uniform01(seed: int, n: int) -> np.ndarray:
    """float64 values in [0,1) with 24 random bits each (exactly representable in f32)."""
    return (splitmix64(seed, n) >> np.uint64(40)).astype(np.float64) * (2.0 ** -24)


# ----------------------------------------------------------------------------------------
# Toy pipeline (Fig. 9) and the Collatz queue-stress pipeline (SURVEY c-0b)
# ----------------------------------------------------------------------------------------
TOY_THRESHOLD = 1 << 20


def toy_seeds(n: int, seed: int = seed_for(0), threshold: int = TOY_THRESHOLD) -> np.ndarray:
    """int32 items in [1, threshold)."""
    x = splitmix64(seed, n)
    return (np.uint64(1) + x % np.uint64(threshold - 1)).astype(np.int32)


def qbench_seeds(n: int, item_bytes: int, depth: int, id0: int = 0) -> np.ndarray:
    """Queue-microbenchmark seeds, as a flat uint32 array of n items:
    word 0 = id | depth << 24 (ids id0.. mod 2^24), words 1.. = id * 2654435761 + k * 40503
    (mod 2^32), a payload every task copies and every leaf checks."""
    W = item_bytes // 4
    ids = (np.arange(n, dtype=np.uint64) + np.uint64(id0)) & np.uint64(0xFFFFFF)
    a = np.empty((n, W), np.uint32)
    a[:, 0] = (ids | np.uint64(depth << 24)).astype(np.uint32)
    k = np.arange(1, W, dtype=np.uint64)
    a[:, 1:] = ((ids[:, None] * np.uint64(2654435761) + k[None, :] * np.uint64(40503)) & np.uint64(0xFFFFFFFF)).astype(np.uint32)
    return a.reshape(-1)


COLLATZ_DTYPE = np.dtype([("id", "<u4"), ("steps", "<u4"), ("v", "<u8")])  # 16 B


def collatz_seeds(n: int, seed: int = seed_for(0, 1), vmax: int = 1 << 16) -> np.ndarray:
    x = splitmix64(seed, n)
    a = np.zeros(n, dtype=COLLATZ_DTYPE)
    a["id"] = np.arange(n, dtype=np.uint32)
    a["v"] = np.uint64(1) + x % np.uint64(vmax - 1)
    return a


# ----------------------------------------------------------------------------------------
# Reyes (Fig. 1; L55; BASELINE configs 1 and 5)
# ----------------------------------------------------------------------------------------
# Patch item, 272 B (Table 2): float4 cp[16] (object space, w = 1), then
# u32 id = frame << 12 | patch, u32 path, u32 dirs, u32 depth.
PATCH_DTYPE = np.dtype([("cp", "<f4", (16, 4)), ("id", "<u4"), ("path", "<u4"),
                        ("dirs", "<u4"), ("depth", "<u4")])
assert PATCH_DTYPE.itemsize == 272

# The queued patch item of the CUDA path, 208 B (reading R-S10): the same
# records with the constant w = 1 dropped and x, y, z as three 16-float planes.
GPU_PATCH_DTYPE = np.dtype([("x", "<f4", (16,)), ("y", "<f4", (16,)), ("z", "<f4", (16,)), ("id", "<u4"),
                            ("path", "<u4"), ("dirs", "<u4"), ("depth", "<u4")])
assert GPU_PATCH_DTYPE.itemsize == 208


def gpu_patch_items(items: np.ndarray) -> np.ndarray:
    """PATCH_DTYPE records -> GPU_PATCH_DTYPE (a repack: no arithmetic).  Every control
    point must be affine (w == 1), which the generators guarantee."""
    if items.size and not np.all(items["cp"][..., 3] == np.float32(1.0)):
        raise ValueError("the queued Reyes patch item carries affine control points (w == 1)")
    out = np.zeros(items.shape, GPU_PATCH_DTYPE)
    for c, name in enumerate("xyz"):
        out[name] = items["cp"][..., c]
    for name in ("id", "path", "dirs", "depth"):
        out[name] = items[name]
    return out


@dataclass
class ReyesScene:
    """Everything a Reyes run reads besides the seed patches."""
    W: int
    H: int
    n_frames: int
    patches_per_frame: int
    M: np.ndarray            # [n_frames, 16] float32, row-major clip = M . p
    albedo: np.ndarray       # [patches_per_frame, 4] float32 (rgb, 0)
    light: np.ndarray        # [4] float32 unit vector (x, y, z, 0)
    seeds: np.ndarray        # PATCH_DTYPE [n_frames * patches_per_frame], frame-major
    max_depth: int = 8
    t_dice: float = 8.0
    near_w: float = 1e-3
    extra: dict = field(default_factory=dict)


def look_at_perspective(eye, target=(0.0, 0.0, 0.0), up=(0.0, 0.0, 1.0), fovy_deg=50.0,
                        aspect=1.0, near=0.1, far=100.0) -> np.ndarray:
    """float64 4x4 view-projection, D3D-style depth (z/w in [0,1] between near and far)."""
    eye = np.asarray(eye, np.float64)
    f = np.asarray(target, np.float64) - eye
    f /= np.linalg.norm(f)
    r = np.cross(f, np.asarray(up, np.float64))
    r /= np.linalg.norm(r)
    u = np.cross(r, f)
    V = np.eye(4)
    V[0, :3], V[1, :3], V[2, :3] = r, u, f
    V[:3, 3] = -V[:3, :3] @ eye
    t = 1.0 / math.tan(math.radians(fovy_deg) / 2)
    P = np.zeros((4, 4))
    P[0, 0] = t / aspect
    P[1, 1] = t
    P[2, 2] = far / (far - near)
    P[2, 3] = -near * far / (far - near)
    P[3, 2] = 1.0
    return P @ V


def heightfield_lattice(n_patch_side: int, seed: int, z_amp: float) -> np.ndarray:
    """(3n+1)^2 control lattice over [-1,1]^2, z ~ U(-z_amp, z_amp). float32 [(3n+1),(3n+1),4]."""
    m = 3 * n_patch_side + 1
    g = np.zeros((m, m, 4), np.float32)
    coords = -1.0 + 2.0 * np.arange(m) / (m - 1)
    g[:, :, 0] = coords[:, None]
    g[:, :, 1] = coords[None, :]
    g[:, :, 2] = (-z_amp + 2 * z_amp * uniform01(seed, m * m)).reshape(m, m)
    g[:, :, 3] = 1.0
    return g


def lattice_patches(lat: np.ndarray, n_patch_side: int) -> np.ndarray:
    """16 control points per patch: P[a][b] = lattice[3pi+a][3pj+b] (a = u index, b = v)."""
    n = n_patch_side * n_patch_side
    cps = np.zeros((n, 16, 4), np.float32)
    for pi in range(n_patch_side):
        for pj in range(n_patch_side):
            cps[pi * n_patch_side + pj] = lat[3 * pi:3 * pi + 4, 3 * pj:3 * pj + 4].reshape(16, 4)
    return cps


def make_patch_items(cps: np.ndarray, n_frames: int) -> np.ndarray:
    n = cps.shape[0]
    items = np.zeros(n_frames * n, PATCH_DTYPE)
    for f in range(n_frames):
        sl = slice(f * n, (f + 1) * n)
        items["cp"][sl] = cps
        items["id"][sl] = (np.uint32(f) << np.uint32(12)) | np.arange(n, dtype=np.uint32)
    return items


def default_light() -> np.ndarray:
    L = np.array([0.3, -0.5, 0.8])
    L /= np.linalg.norm(L)
    return np.array([L[0], L[1], L[2], 0.0], np.float32)


def reyes_config1(seed: int = seed_for(1), W: int = 256, H: int = 256, n_side: int = 4,
                  max_depth: int = 8, n_frames: int = 1) -> ReyesScene:
    """BASELINE config 1: 16 bicubic Bezier patches, 256x256, max split depth 8.

    4x4 patches tile a height field over [-1,1]^2 (13x13 lattice, z ~ U(-0.25,0.25));
    camera eye (0,-1.6,1.2) -> origin, up +z, fovy 50 deg, near 0.1.
    n_frames > 1: the same frame replicated (SURVEY §8(d) throughput mode, R frames in
    flight in one run).
    """
    lat = heightfield_lattice(n_side, seed, 0.25)
    cps = lattice_patches(lat, n_side)
    M = look_at_perspective((0.0, -1.6, 1.2), aspect=W / H).astype(np.float32).reshape(1, 16)
    M = np.repeat(M, n_frames, axis=0)
    alb = np.zeros((n_side * n_side, 4), np.float32)
    alb[:, :3] = uniform01(seed + 1, n_side * n_side * 3).reshape(-1, 3)
    return ReyesScene(W=W, H=H, n_frames=n_frames, patches_per_frame=n_side * n_side, M=M, albedo=alb,
                      light=default_light(), seeds=make_patch_items(cps, n_frames), max_depth=max_depth)


def reyes_frame_camera(f: int, n_frames_orbit: int = 512, W: int = 256, H: int = 256) -> np.ndarray:
    """Per-frame orbit camera of config 5: angle 2*pi*f/512, distance 1.3+1.2*(1+cos(2*pi*f/64))/2."""
    th = 2 * math.pi * f / n_frames_orbit
    d = 1.3 + 1.2 * (1 + math.cos(2 * math.pi * f / 64)) / 2
    eye = (0.8 * d * math.sin(th), -0.8 * d * math.cos(th), 0.6 * d)
    return look_at_perspective(eye, aspect=W / H).astype(np.float32).reshape(16)


def reyes_config5(n_frames: int = 512, n_side: int = 64, frame0: int = 0, seed: int = seed_for(5),
                  W: int = 256, H: int = 256, z_amp: float = 0.05, max_depth: int = 8) -> ReyesScene:
    """BASELINE config 5: a batch of frames x 4096 patches (64x64 patch height field,
    193x193 lattice) with a per-frame orbit camera.  ``frame0`` selects a shard
    [frame0, frame0 + n_frames) of the 512-frame orbit (multi-GPU sharding)."""
    lat = heightfield_lattice(n_side, seed, z_amp)
    cps = lattice_patches(lat, n_side)
    M = np.stack([reyes_frame_camera(frame0 + f, 512, W, H) for f in range(n_frames)])
    alb = np.zeros((n_side * n_side, 4), np.float32)
    alb[:, :3] = uniform01(seed + 1, n_side * n_side * 3).reshape(-1, 3)
    items = make_patch_items(cps, n_frames)
    # ids carry the LOCAL frame index (frame buffers are per shard)
    return ReyesScene(W=W, H=H, n_frames=n_frames, patches_per_frame=n_side * n_side, M=M,
                      albedo=alb, light=default_light(), seeds=items, max_depth=max_depth,
                      extra={"frame0": frame0})


@dataclass
class RasterScene:
    """BASELINE config 4 inputs: triangles in pixel space."""
    W: int
    H: int
    M: np.ndarray      # [16] float32 pixel -> NDC, w = 1
    pos: np.ndarray    # [n, 3, 4] float32 (x_px, y_px, z, 1)
    col: np.ndarray    # [n, 3, 4] float32 (r, g, b, 0)
    near_clip: int = 0  # 1: clip against z = 0 (Clip fan-out 0..2, keys carry 2 tri + j; R-S9)

    @property
    def n_tris(self):
        return self.pos.shape[0]


def pixel_to_ndc(W: int, H: int) -> np.ndarray:
    M = np.zeros((4, 4))
    M[0, 0], M[0, 3] = 2.0 / W, -1.0
    M[1, 1], M[1, 3] = 2.0 / H, -1.0
    M[2, 2] = 1.0
    M[3, 3] = 1.0
    return M.astype(np.float32).reshape(16)


def raster_scene(n: int = 1 << 20, W: int = 1920, H: int = 1080, seed: int = seed_for(4),
                 area_range=(0.5, 512.0), aspect_range=(0.25, 4.0)) -> RasterScene:
    """Synthetic triangles: centres U(screen), area log-uniform on
    [0.5, 512] px^2, aspect log-uniform on [1/4, 4], random rotation, z ~ U(0.05, 0.95)
    per vertex, colours U[0,1)^3.  Shape: base b, height h (b*h/2 = area, b/h = aspect),
    vertices (-b/2, -h/3), (b/2, -h/3), (0, 2h/3) about the centre, then rotated."""
    u = uniform01(seed, n * 17).reshape(n, 17)
    cx, cy = u[:, 0] * W, u[:, 1] * H
    la, lb = math.log(area_range[0]), math.log(area_range[1])
    area = np.exp(la + u[:, 2] * (lb - la))
    sa, sb = math.log(aspect_range[0]), math.log(aspect_range[1])
    aspect = np.exp(sa + u[:, 3] * (sb - sa))
    th = 2 * math.pi * u[:, 4]
    b = np.sqrt(2 * area * aspect)
    h = 2 * area / b
    lx = np.stack([-b / 2, b / 2, np.zeros(n)], 1)
    ly = np.stack([-h / 3, -h / 3, 2 * h / 3], 1)
    c, s = np.cos(th)[:, None], np.sin(th)[:, None]
    pos = np.zeros((n, 3, 4), np.float32)
    pos[:, :, 0] = cx[:, None] + c * lx - s * ly
    pos[:, :, 1] = cy[:, None] + s * lx + c * ly
    pos[:, :, 2] = 0.05 + 0.9 * u[:, 5:8]
    pos[:, :, 3] = 1.0
    col = np.zeros((n, 3, 4), np.float32)
    col[:, :, :3] = u[:, 8:17].reshape(n, 3, 3)
    return RasterScene(W=W, H=H, M=pixel_to_ndc(W, H), pos=pos, col=col)


def raster_near_scene(n: int = 4096, W: int = 256, H: int = 192, seed: int = seed_for(4) + 17,
                      z_range=(-0.6, 0.95), area_range=(4.0, 2048.0), perspective: bool = False) -> RasterScene:
    """Near-plane clipping workload (DESIGN R-S9): the config-4 recipe with
    per-vertex z ~ U(z_range), so about half the triangles straddle z = 0 (one or two
    vertices behind the near plane) and a few lie wholly behind it; near_clip = 1.
    perspective: w = z + 0.5 (rows 0, 1 as pixel_to_ndc, row 3 = (0, 0, 1, 0.5)), so
    vertices with z <= -0.5 have w <= 0 -- the default mode culls their triangles whole,
    the clip keeps the part in front (w = 0.5 on the plane)."""
    sc = raster_scene(n=n, W=W, H=H, seed=seed, area_range=area_range)
    u = uniform01(seed ^ 0x5A5A, n * 3).reshape(n, 3)
    sc.pos[:, :, 2] = (z_range[0] + (z_range[1] - z_range[0]) * u).astype(np.float32)
    sc.near_clip = 1
    if perspective:
        M = sc.M.reshape(4, 4).copy()
        M[3] = (0.0, 0.0, 1.0, 0.5)
        sc.M = M.reshape(16)
    return sc


def raster_quad_mesh(W: int, H: int, cell: int = 8, z: float = 0.5) -> RasterScene:
    """Watertightness pin: a full-screen grid of cell x cell squares, each split into two
    triangles along a diagonal (alternating), all at depth z."""
    tris = []
    for y in range(0, H, cell):
        for x in range(0, W, cell):
            a, b_, c_, d = (x, y), (x + cell, y), (x + cell, y + cell), (x, y + cell)
            if ((x // cell) + (y // cell)) % 2 == 0:
                tris += [(a, b_, c_), (a, c_, d)]
            else:
                tris += [(a, b_, d), (b_, c_, d)]
    n = len(tris)
    pos = np.zeros((n, 3, 4), np.float32)
    for i, t in enumerate(tris):
        for k, (px, py) in enumerate(t):
            pos[i, k] = (px, py, z, 1.0)
    col = np.full((n, 3, 4), 0.5, np.float32)
    col[:, :, 3] = 0
    return RasterScene(W=W, H=H, M=pixel_to_ndc(W, H), pos=pos, col=col)


@dataclass
class CfdScene:
    """BASELINE config 3 (CFD half) inputs: a structured G x G grid with
    Rodinia euler3d semantics.  All arrays SoA float32 / int32."""
    G: int
    T: int
    n_outer: int
    vars0: np.ndarray     # [5, G*G] density, momentum x, y, z, density energy
    area: np.ndarray      # [G*G]
    nb: np.ndarray        # [4, G*G] int32 neighbour or -2 (far field)
    normals: np.ndarray   # [4, 3, G*G]
    ff: np.ndarray        # [5] far-field conserved state

    @property
    def n_cells(self):
        return self.G * self.G


def cfd_far_field() -> np.ndarray:
    """Rodinia euler3d far field: rho 1.4, p 1, Mach 1.2, angle of attack 0 (float64 ->
    float32): (rho, rho*u, 0, 0, rho*|u|^2/2 + p/(gamma-1))."""
    gamma, rho, p, mach = 1.4, 1.4, 1.0, 1.2
    c = math.sqrt(gamma * p / rho)
    u = mach * c
    return np.array([rho, rho * u, 0.0, 0.0, rho * 0.5 * u * u + p / (gamma - 1)], np.float32)


def cfd_scene(G: int = 4096, n_outer: int = 10, seed: int = seed_for(3, 1), T: int = 0, bump_amp: float = 0.05,
              uniform: bool = False) -> CfdScene:
    """Grid cell (r, c) has index r*G + c; faces j = 0..3 are -x, +x, -y, +y with unit
    normals (-1,0,0), (1,0,0), (0,-1,0), (0,1,0), area 1; off-grid neighbours are far
    field.  Initial state = far field x (1 + amp * bump), bump = sum of 8 seeded
    Gaussians (float64 on the host).  Tiles are T = min(1024, G) cells of a row."""
    n = G * G
    T = T or min(1024, G)
    ff = cfd_far_field()
    r = np.repeat(np.arange(G), G)
    c = np.tile(np.arange(G), G)
    if uniform:
        scale = np.ones(n)
    else:
        u = uniform01(seed, 8 * 3).reshape(8, 3)
        bump = np.zeros(n)
        for g in range(8):
            r0, c0, s = u[g, 0] * G, u[g, 1] * G, G / 16.0 * (0.5 + u[g, 2])
            bump += np.exp(-((r - r0) ** 2 + (c - c0) ** 2) / (2 * s * s))
        scale = 1.0 + bump_amp * bump
    vars0 = (ff.astype(np.float64)[:, None] * scale[None, :]).astype(np.float32)
    nb = np.full((4, n), -2, np.int32)
    idx = np.arange(n, dtype=np.int64)
    nb[0] = np.where(c > 0, idx - 1, -2)
    nb[1] = np.where(c < G - 1, idx + 1, -2)
    nb[2] = np.where(r > 0, idx - G, -2)
    nb[3] = np.where(r < G - 1, idx + G, -2)
    normals = np.zeros((4, 3, n), np.float32)
    normals[0, 0], normals[1, 0], normals[2, 1], normals[3, 1] = -1.0, 1.0, -1.0, 1.0
    return CfdScene(G=G, T=T, n_outer=n_outer, vars0=vars0, area=np.ones(n, np.float32), nb=nb,
                    normals=normals, ff=ff)


@dataclass
class FaceScene:
    """BASELINE config 2 inputs: RGB frames and a synthetic LBP cascade."""
    W: int
    H: int
    rgb: np.ndarray          # [n_frames, H, W, 3] uint8
    n_weak: np.ndarray       # [K] int32
    thr: np.ndarray          # [K] int32
    weak: np.ndarray         # [sum n_weak, 12] int32: cx, cy, mask[8], in, out
    planted: np.ndarray      # [n_frames, n_planted, 2] level-0 (x, y) of the constant templates

    @property
    def n_frames(self):
        return self.rgb.shape[0]


def face_scene(W: int = 1920, H: int = 1080, n_frames: int = 1, seed: int = seed_for(2), n_planted: int = 24,
               K: int = 12) -> FaceScene:
    """Frames: 8x8 constant blocks U(0,255) + per-pixel noise in [-8, 8] (clamped), plus
    n_planted noise-free constant 24x24 templates (their interior LBP code is 255).
    Cascade: K stages, stage k has 2+k weak classifiers with cells
    U([1,22]^2), 256-bit masks with bit probability 1/2 and the template code (255) forced
    on, leaves +/-1000, threshold 1000 * (2*ceil(0.6 n_k) - n_k)."""
    nb_w, nb_h = (W + 7) // 8, (H + 7) // 8
    rgb = np.zeros((n_frames, H, W, 3), np.uint8)
    planted = np.zeros((n_frames, n_planted, 2), np.int32)
    for f in range(n_frames):
        s = seed + 1000 * f
        blocks = (splitmix64(s, nb_h * nb_w * 3) % np.uint64(256)).astype(np.int32).reshape(nb_h, nb_w, 3)
        img = np.repeat(np.repeat(blocks, 8, 0), 8, 1)[:H, :W]
        noise = (splitmix64(s + 1, H * W * 3) % np.uint64(17)).astype(np.int32).reshape(H, W, 3) - 8
        img = np.clip(img + noise, 0, 255)
        pos = splitmix64(s + 2, n_planted * 2).reshape(n_planted, 2)
        for t in range(n_planted):
            x = int(pos[t, 0] % np.uint64(W - 24))
            y = int(pos[t, 1] % np.uint64(H - 24))
            img[y:y + 24, x:x + 24] = 200
            planted[f, t] = (x, y)
        rgb[f] = img.astype(np.uint8)
    n_weak = np.array([2 + k for k in range(K)], np.int32)
    nw = int(n_weak.sum())
    r = splitmix64(seed + 77, nw * 11).reshape(nw, 11)
    weak = np.zeros((nw, 12), np.int64)
    weak[:, 0] = 1 + (r[:, 0] % np.uint64(22)).astype(np.int64)
    weak[:, 1] = 1 + (r[:, 1] % np.uint64(22)).astype(np.int64)
    masks = r[:, 2:6]                                 # 4 x 64 random bits = 256
    for w in range(8):
        weak[:, 2 + w] = ((masks[:, w // 2] >> np.uint64(32 * (w % 2))) & np.uint64(0xFFFFFFFF)).astype(np.int64)
    weak[:, 2 + 7] |= 1 << 31                         # code 255 -> word 7, bit 31
    weak[:, 10], weak[:, 11] = 1000, -1000
    weak = weak.astype(np.uint32).view(np.int32).reshape(nw, 12)
    thr = np.array([1000 * (2 * math.ceil(0.6 * n) - n) for n in n_weak], np.int32)
    return FaceScene(W=W, H=H, rgb=rgb, n_weak=n_weak, thr=thr, weak=np.ascontiguousarray(weak), planted=planted)


def pyramid_images(n_img: int = 32, S: int = 4096, seed: int = seed_for(3)) -> np.ndarray:
    """BASELINE config 3 (pyramid half) inputs: n_img RGB8 images S x S (SURVEY §8(d)
    d3a): 8x8 constant blocks U(0,255) per channel, scaled by 3/4, plus a horizontal
    gradient 0..63.  uint8 [n_img, S, S, 3]."""
    nb = S // 8
    vals = (splitmix64(seed, n_img * nb * nb * 3) % np.uint64(256)).astype(np.int32).reshape(n_img, nb, nb, 3)
    blocks = np.repeat(np.repeat(vals, 8, axis=1), 8, axis=2)
    grad = (np.arange(S, dtype=np.int32) * 64 // S)[None, None, :, None]
    return np.minimum(255, blocks * 3 // 4 + grad).astype(np.uint8)


def reyes_planar(S_px: float, W: int = 64, H: int = 64, x0: float = 8.0, y0: float = 8.0,
                 max_depth: int = 8, albedo=(0.5, 0.25, 0.75)) -> ReyesScene:
    """Closed-form special case (SURVEY c-1 pin 4): a planar patch parallel to the image
    plane, control points on a uniform grid, orthographic M that maps object (x, y) to
    NDC so that the patch spans [x0, x0+S] x [y0, y0+S] pixels (dyadic coordinates)."""
    cps = np.zeros((1, 16, 4), np.float32)
    for a in range(4):
        for b in range(4):
            cps[0, 4 * a + b] = (a, b, 0.0, 1.0)  # x = a, y = b in [0,3]
    # object x in [0,3] -> screen x0 + S*x/3 : sx = (ndc*0.5+0.5)*W, ndc = 2*sx/W - 1
    sx_scale = S_px / 3.0
    M = np.zeros((4, 4))
    M[0, 0] = 2.0 * sx_scale / W
    M[0, 3] = 2.0 * x0 / W - 1.0
    M[1, 1] = 2.0 * sx_scale / H
    M[1, 3] = 2.0 * y0 / H - 1.0
    M[2, 3] = 0.5
    M[3, 3] = 1.0
    alb = np.zeros((1, 4), np.float32)
    alb[0, :3] = albedo
    return ReyesScene(W=W, H=H, n_frames=1, patches_per_frame=1, M=M.astype(np.float32).reshape(1, 16),
                      albedo=alb, light=np.array([0.0, 0.0, 1.0, 0.0], np.float32),
                      seeds=make_patch_items(cps, 1), max_depth=max_depth)


# ----------------------------------------------------------------------------------------
# LDPC decoder (Fig. 17, L59; 100 frames x 100 iterations, L53)
# ----------------------------------------------------------------------------------------
@dataclass
class LdpcScene:
    """A (dv, dc)-regular parity-check matrix as edge lists (check-major edge order) and
    per-frame channel LLRs of the all-zero codeword (readings R-L1..R-L6)."""
    N: int
    M: int
    dv: int
    dc: int
    check_vars: np.ndarray   # [M*dc] int32: variable node of edge e = m*dc + k
    var_edges: np.ndarray    # [N*dv] int32: the dv edges of variable n, ascending
    llr: np.ndarray          # [n_frames, N] float32
    n_iter: int = 100
    alpha: float = 0.75

    @property
    def n_frames(self) -> int:
        return self.llr.shape[0]

    # pipeline decomposition (reading R-L6): chunks of <= 256 checks / variables, <= 16 each
    @property
    def nc_chk(self) -> int:
        return min(16, (self.M + 255) // 256)

    @property
    def nc_var(self) -> int:
        return min(16, (self.N + 255) // 256)


def ldpc_regular_h(N: int, dv: int, dc: int, seed: int) -> np.ndarray:
    """Socket-permutation (configuration-model) construction of a (dv, dc)-regular H:
    check-major edge list check_vars[M*dc]; a check never holds the same variable twice
    (colliding sockets are swapped with random partners until none is left)."""
    assert (N * dv) % dc == 0
    E = N * dv
    M = E // dc
    sockets = np.repeat(np.arange(N, dtype=np.int64), dv)
    key = splitmix64(seed, E)
    cv = sockets[np.argsort(key, kind="stable")].copy()
    r = 0
    while True:
        rows = cv.reshape(M, dc)
        srt = np.sort(rows, axis=1)
        bad_rows = np.nonzero((srt[:, 1:] == srt[:, :-1]).any(axis=1))[0]
        if bad_rows.size == 0:
            break
        r += 1
        pick = splitmix64(seed + 7919 * r, 2 * bad_rows.size)
        for i, m in enumerate(bad_rows):
            a = m * dc + int(pick[2 * i] % np.uint64(dc))
            b = int(pick[2 * i + 1] % np.uint64(E))
            cv[a], cv[b] = cv[b], cv[a]
    return cv.astype(np.int32)


def ldpc_var_edges(check_vars: np.ndarray, N: int, dv: int) -> np.ndarray:
    order = np.argsort(check_vars, kind="stable")      # edges grouped by variable, ascending
    ve = order.astype(np.int32).reshape(N, dv)
    assert np.all(check_vars[ve] == np.arange(N)[:, None])
    return ve.reshape(-1)


def ldpc_scene(n_frames: int = 100, N: int = 2048, dv: int = 3, dc: int = 6, ebn0_db: float = 2.0,
               n_iter: int = 100, seed: int = seed_for(6), alpha: float = 0.75) -> LdpcScene:
    """Rate-(1 - dv/dc) regular code, BPSK over AWGN at Eb/N0 = ebn0_db, all-zero codeword:
    y = 1 + sigma*z (Box-Muller in float64 from SplitMix64), LLR = 2y/sigma^2 as float32."""
    cv = ldpc_regular_h(N, dv, dc, seed)
    ve = ldpc_var_edges(cv, N, dv)
    rate = 1.0 - dv / dc
    sigma2 = 1.0 / (2.0 * rate * 10.0 ** (ebn0_db / 10.0))
    u1 = np.maximum(uniform01(seed + 1, n_frames * N).astype(np.float64), 2.0 ** -25)
    u2 = uniform01(seed + 2, n_frames * N).astype(np.float64)
    z = np.sqrt(-2.0 * np.log(u1)) * np.cos(2.0 * np.pi * u2)
    y = 1.0 + np.sqrt(sigma2) * z
    llr = (2.0 * y / sigma2).astype(np.float32).reshape(n_frames, N)
    return LdpcScene(N=N, M=N * dv // dc, dv=dv, dc=dc, check_vars=cv, var_edges=ve, llr=llr,
                     n_iter=n_iter, alpha=alpha)
