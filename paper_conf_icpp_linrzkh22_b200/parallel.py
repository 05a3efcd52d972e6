"""Stimulus sharding over the GPUs of one box (one process per GPU, torch.distributed).

Stimuli are independent (stimulus groups carry no
dependency), so a batch of ``n_total`` stimuli is split into
contiguous blocks, one per rank, and each rank simulates its block on its own
GPU with no communication during the run. The collectives run
only after the timed work:

1. ``all_reduce(MAX)`` of the elapsed device time (throughput = N·T / max);
2. a rank-0 ``gather`` of per-stimulus results — normally the N x 8-byte
   register digests (``rtlsim_reg_digest``), never the registers themselves
   (config 5's registers are ~116 GB per rank);
3. toggle coverage (N5): ``all_gather`` of every rank's [RW] u32 bitmap and a
   local bitwise OR (NCCL has no OR reduction; MAX on packed words would be
   wrong).

The compute step is injected (``simulate(s0, n) -> dict``) so exactly this
host logic runs on GPUs under NCCL (bench.py) and, in the CPU tests, under
gloo with the oracle standing in for the GPU.
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
    elapsed_max: float                 # max over ranks of the shard's elapsed time
    reg_digest: np.ndarray | None      # [n_total] u64 on rank 0 (gathered), else None
    coverage: np.ndarray | None        # [RW] u32, OR over all ranks (every rank)
    local: dict                        # this rank's own simulate() result


def gather_rows(dist, local: np.ndarray, n_total: int, device) -> np.ndarray | None:
    """Gather every rank's [n_r][...] block into [n_total][...] on rank 0
    (None elsewhere). Blocks are padded to one size (collectives need equal
    sizes); the payload travels as int64 words."""
    import torch
    world, rank = dist.get_world_size(), dist.get_rank()
    tail = local.shape[1:]
    row_bytes = local.dtype.itemsize * int(np.prod(tail, dtype=np.int64))
    raw = np.ascontiguousarray(local).view(np.uint8).reshape(local.shape[0], row_bytes)
    width8 = max(1, -(-raw.shape[1] // 8))
    rows = -(-n_total // world)
    buf = np.zeros((rows, width8 * 8), np.uint8)
    buf[:raw.shape[0], :raw.shape[1]] = raw
    t = torch.from_numpy(buf.view(np.int64)).to(device)
    parts = [torch.empty_like(t) for _ in range(world)] if rank == 0 else None
    dist.gather(t, parts, dst=0)
    if rank != 0:
        return None
    out = []
    for r in range(world):
        _, n = shard_range(n_total, world, r)
        out.append(parts[r][:n].cpu().numpy().view(np.uint8)[:, :raw.shape[1]])
    flat = np.concatenate(out, axis=0)
    return flat.view(local.dtype).reshape((n_total,) + tail)


def or_all(dist, bitmap: np.ndarray, device) -> np.ndarray:
    """Bitwise OR of an equal-size u32 bitmap over all ranks (all_gather + OR)."""
    import torch
    world = dist.get_world_size()
    t = torch.from_numpy(np.ascontiguousarray(bitmap, np.uint32).view(np.int32)).to(device)
    parts = [torch.empty_like(t) for _ in range(world)]
    dist.all_gather(parts, t)
    acc = np.zeros_like(bitmap, dtype=np.uint32)
    for p in parts:
        acc |= p.cpu().numpy().view(np.uint32)
    return acc


def run_sharded(simulate, n_total: int, device="cpu") -> ShardResult:
    """Run ``simulate(s0, n) -> {"elapsed": s, "reg_digest": [n] u64 | None,
    "coverage": [RW] u32 | None, ...}`` on this rank's shard, then reduce /
    gather (after the timed work, which ``simulate`` brackets itself)."""
    import torch
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()):   # one process: no collective
        res = simulate(0, n_total)
        dig = None if res.get("reg_digest") is None else np.asarray(res["reg_digest"], np.uint64)
        return ShardResult(float(res["elapsed"]), dig, res.get("coverage"), res)
    world, rank = dist.get_world_size(), dist.get_rank()
    s0, n = shard_range(n_total, world, rank)
    res = simulate(s0, n)
    el = torch.tensor([float(res["elapsed"])], dtype=torch.float64, device=device)
    dist.all_reduce(el, op=dist.ReduceOp.MAX)
    dig = cov = None
    if res.get("reg_digest") is not None:
        dig = gather_rows(dist, np.asarray(res["reg_digest"], np.uint64), n_total, device)
    if res.get("coverage") is not None:
        cov = or_all(dist, res["coverage"], device)
    return ShardResult(float(el.item()), dig, cov, res)
