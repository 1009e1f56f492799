"""Multi-process (gloo, world_size 2 and 3, CPU) test of the frame sharder used by
bench.py for config 5: partition, per-rank rendering (the CPU oracle stands in for the
GPU compute here), counter reduction and frame gather reproduce a single-process run."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

from paper_conf_micro_zhengozsyc17_b200 import shard


def test_shard_range_partition():
    for world in (1, 2, 3, 4, 7, 8):
        for total in (0, 1, 5, 64, 512):
            ranges = [shard.shard_range(r, world, total) for r in range(world)]
            assert ranges[0][0] == 0 and ranges[-1][1] == total
            assert all(a[1] == b[0] for a, b in zip(ranges, ranges[1:]))
            sizes = [b - a for a, b in ranges]
            assert max(sizes) - min(sizes) <= 1


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, total, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from paper_conf_micro_zhengozsyc17_b200 import inputs
        f0, f1 = shard.shard_range(rank, world, total)
        sc = inputs.reyes_config5(n_frames=f1 - f0, n_side=8, frame0=f0, W=48, H=48)
        r = oracle.reyes_pipeline(sc)
        local = torch.from_numpy(r["colour"].copy())
        full = shard.gather_frames(local, total)
        counts = shard.sum_over_ranks([r["n_bound"], r["n_split"], r["n_dice"], r["n_shade"]], "cpu")
        t = shard.max_over_ranks(float(rank + 1), "cpu")
        if rank == 0:
            q.put((full.numpy(), counts, t))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_sharded_render_equals_single_process(orc, world):
    from paper_conf_micro_zhengozsyc17_b200 import inputs
    total = 5
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, total, q)) for r in range(world)]
    for p in procs:
        p.start()
    full, counts, t = q.get(timeout=120)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    ref = orc.reyes_pipeline(inputs.reyes_config5(n_frames=total, n_side=8, W=48, H=48))
    assert np.array_equal(full, ref["colour"])
    assert counts == [ref["n_bound"], ref["n_split"], ref["n_dice"], ref["n_shade"]]
    assert t == float(world)


# ---------------------------------------------------------------- raster triangle sharding
def collapse_outside(scene, lo, hi):
    """The shard's scene: triangles outside [lo, hi) collapsed to a point (zero area, culled
    by Clip), so every surviving key keeps its global triangle id."""
    import dataclasses
    pos = scene.pos.copy()
    keep = np.zeros(scene.n_tris, bool)
    keep[lo:hi] = True
    pos[~keep, 1] = pos[~keep, 0]
    pos[~keep, 2] = pos[~keep, 0]
    return dataclasses.replace(scene, pos=pos)


def test_ordered_key_transform_preserves_uint64_order():
    rng = np.random.default_rng(5)
    u = np.concatenate([rng.integers(0, 2**64 - 1, 2000, dtype=np.uint64),
                        np.array([0, 1, 2**63 - 1, 2**63, 2**63 + 1, 2**64 - 1], np.uint64)])
    o = shard.ukey_to_ordered(torch.from_numpy(u.view(np.int64))).numpy()
    assert np.array_equal(np.argsort(o, kind="stable"), np.argsort(u, kind="stable"))
    assert np.array_equal(shard.ukey_to_ordered(torch.from_numpy(o)).numpy().view(np.uint64), u)


def _raster_scene(near):
    from paper_conf_micro_zhengozsyc17_b200 import inputs
    if near:
        return inputs.raster_near_scene(1500, W=96, H=64, area_range=(2.0, 600.0), z_range=(-0.9, 0.95), perspective=True)
    return inputs.raster_scene(n=3000, W=96, H=64)


def _raster_worker(rank, world, port, q, near=False):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from paper_conf_micro_zhengozsyc17_b200 import inputs
        sc = _raster_scene(near)
        lo, hi = shard.shard_range(rank, world, sc.n_tris)
        r = oracle.raster_definition(collapse_outside(sc, lo, hi))
        k, c = shard.raster_merge(torch.from_numpy(r["key"].view(np.int64).copy()), torch.from_numpy(r["colour"].copy()))
        if rank == 0:
            q.put((k.numpy().view(np.uint64), c.numpy()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,near", [(2, False), (3, False), (2, True)])
def test_triangle_sharded_raster_equals_single_frame(orc, world, near):
    """each rank rasterises a shard of the triangles (the CPU oracle stands
    in for the GPU here); one MIN all-reduce of the z-keys plus the winner's colour
    reproduces the single-process frame bit for bit."""
    from paper_conf_micro_zhengozsyc17_b200 import inputs
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_raster_worker, args=(r, world, port, q, near)) for r in range(world)]
    for p in procs:
        p.start()
    k, c = q.get(timeout=120)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    ref = orc.raster_definition(_raster_scene(near))
    assert np.array_equal(k, ref["key"]) and np.array_equal(c, ref["colour"])
