"""Multi-GPU sharding: frames of the Reyes batch (BASELINE config 5) and
triangles of one raster frame (one exchange step, a MIN of z-keys).

Frames are independent, so rank r of P renders frames [r*F/P, (r+1)*F/P) with a complete
pipeline of its own and no inter-GPU traffic during the run.  The only exchange steps
are after the run: a max-over-ranks time, a sum of per-stage counters, and the gather of
the frame buffers (all_gather).  Backend-agnostic: NCCL over NVLink on the GPU box, gloo
on CPU in the tests.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def shard_range(rank: int, world: int, total: int) -> tuple[int, int]:
    """Contiguous, balanced, covering partition of [0, total)."""
    if not (0 <= rank < world) or total < 0:
        raise ValueError((rank, world, total))
    return rank * total // world, (rank + 1) * total // world


def max_over_ranks(value: float, device) -> float:
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    if dist.is_initialized() and dist.get_world_size() > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def sum_over_ranks(values, device) -> list[float]:
    t = torch.tensor([float(v) for v in values], dtype=torch.float64, device=device)
    if dist.is_initialized() and dist.get_world_size() > 1:
        dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return [float(x) for x in t.tolist()]


def gather_frames(local: torch.Tensor, total: int) -> torch.Tensor:
    """Gather per-rank frame blocks [n_r, ...] (n_r from shard_range) into [total, ...]
    on every rank.  Uses all_gather_into_tensor when shards are equal, else padded
    all_gather."""
    if not (dist.is_initialized() and dist.get_world_size() > 1):
        return local
    world, rank = dist.get_world_size(), dist.get_rank()
    sizes = [shard_range(r, world, total)[1] - shard_range(r, world, total)[0] for r in range(world)]
    assert local.shape[0] == sizes[rank], (local.shape, sizes, rank)
    tail = tuple(local.shape[1:])
    if len(set(sizes)) == 1 and dist.get_backend() == "nccl":
        out = torch.empty((total,) + tail, dtype=local.dtype, device=local.device)
        dist.all_gather_into_tensor(out, local.contiguous())
        return out
    m = max(sizes)
    pad = torch.zeros((m,) + tail, dtype=local.dtype, device=local.device)
    pad[: local.shape[0]] = local
    parts = [torch.empty_like(pad) for _ in range(world)]
    dist.all_gather(parts, pad)
    return torch.cat([parts[r][: sizes[r]] for r in range(world)], 0)


_SIGN = -(1 << 63)  # int64 bit pattern 0x8000000000000000


def ukey_to_ordered(keys: torch.Tensor) -> torch.Tensor:
    """uint64 z-keys stored in an int64 tensor -> int64 values with the same order under
    signed comparison (flip the top bit), so MIN reductions (which are signed) work."""
    return keys ^ _SIGN


def raster_merge(keys: torch.Tensor, colour: torch.Tensor):
    """Triangle-sharded rasterisation: every rank rendered the triangles
    of its shard_range into keys [H, W] (uint64 bits in int64: zkey << 32 | global tri id,
    UINT64_MAX = empty) and colour [H, W, 4].  One exchange step: all_reduce(MIN) of the
    order-preserving keys, then the colour of the winning triangle -- held by exactly one
    rank, because triangle ids are unique across shards -- by an all_reduce(SUM) of the
    colours masked to the pixels each rank won (exact: one addend per pixel is nonzero).
    Returns (keys, colour) of the whole frame on every rank."""
    k = ukey_to_ordered(keys.clone())
    if dist.is_initialized() and dist.get_world_size() > 1:
        dist.all_reduce(k, op=dist.ReduceOp.MIN)
    won = ukey_to_ordered(keys) == k
    c = torch.where(won.unsqueeze(-1), colour, torch.zeros_like(colour))
    if dist.is_initialized() and dist.get_world_size() > 1:
        dist.all_reduce(c, op=dist.ReduceOp.SUM)
    return ukey_to_ordered(k), c
