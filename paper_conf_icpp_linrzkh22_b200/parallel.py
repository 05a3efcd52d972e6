"""Stimulus sharding over GPUs of one box (one process per GPU, torch.distributed).

Stimuli are independent (groups carry no dependency,
P:L946-948), so the batch is split into contiguous blocks, one per rank, and
each rank simulates its block on its own GPU with no communication. NCCL is
used only after the run: max-reduction of the elapsed time and gathers of
per-stimulus results (digests, final registers) to rank 0.

The compute step is injected (``simulate(ir, s0, n) -> dict``) so the same
host logic runs on GPUs (the CUDA Simulator) or, in CPU tests, on the gloo
backend with the oracle standing in for the GPU.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np


def shard_range(n_total: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous block [s0, s0 + n) of rank `rank` (sizes differ by <= 1)."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad world/rank")
    base, extra = divmod(n_total, world)
    s0 = rank * base + min(rank, extra)
    return s0, base + (1 if rank < extra else 0)


@dataclass
class ShardResult:
    elapsed_max: float
    digest: np.ndarray | None     # [N_total][T] on rank 0 (gathered), else None
    regs: np.ndarray | None       # [N_total][RW] on rank 0 (gathered), else None


def _gather_rows(dist, local: np.ndarray, n_total: int, world: int, rank: int, device):
    """Gather [n_r][...] row blocks of every rank into [n_total][...] on all ranks
    (all_gather of equal-size padded blocks; NCCL needs equal sizes)."""
    import torch
    width = int(np.prod(local.shape[1:])) if local.ndim > 1 else 1
    rows = -(-n_total // world)
    buf = np.zeros((rows, width), dtype=np.int64)
    flat = local.reshape(local.shape[0], -1).astype(np.int64, copy=False) if local.size else buf[:0]
    buf[:flat.shape[0]] = flat
    t = torch.from_numpy(buf).to(device)
    parts = [torch.empty_like(t) for _ in range(world)]
    dist.all_gather(parts, t)
    out = []
    for r in range(world):
        s0, n = shard_range(n_total, world, r)
        out.append(parts[r][:n].cpu().numpy())
    return np.concatenate(out, axis=0).reshape((n_total,) + local.shape[1:])


def run_sharded(simulate, n_total: int, device="cpu", gather_digest=True, gather_regs=True) -> ShardResult:
    """Run `simulate(s0, n) -> {"digest": [n][T] u64, "regs": [n][RW] u32, "elapsed": s}`
    on this rank's shard, then reduce/gather (after the timed work)."""
    import torch
    import torch.distributed as dist
    world, rank = dist.get_world_size(), dist.get_rank()
    s0, n = shard_range(n_total, world, rank)
    res = simulate(s0, n)
    el = torch.tensor([float(res["elapsed"])], dtype=torch.float64, device=device)
    dist.all_reduce(el, op=dist.ReduceOp.MAX)
    dig = regs = None
    if gather_digest and res.get("digest") is not None:
        d = res["digest"].view(np.int64)
        dig = _gather_rows(dist, d, n_total, world, rank, device).view(np.uint64)
    if gather_regs and res.get("regs") is not None:
        r = res["regs"].astype(np.int64)
        regs = _gather_rows(dist, r, n_total, world, rank, device).astype(np.uint32)
    return ShardResult(float(el.item()), dig if rank == 0 else None, regs if rank == 0 else None)
