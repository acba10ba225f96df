"""Multi-GPU host logic: every GPU holds a full replica of the net
and serves its own contiguous shard of whole queries; "there is no communication between
GPUs", so the only collectives are the one-time weight-arena broadcast
(C1), the max-over-ranks timing reduction of the harness and an optional output gather (C2).

torch.distributed is plumbing here (NCCL on B200s, gloo in the CPU tests); nothing in this
module computes any part of the forward pass.
"""
from __future__ import annotations

from typing import Tuple

import torch
import torch.distributed as dist


def query_shard(n_queries: int, rows_per_query: int, world: int, rank: int) -> Tuple[int, int]:
    """Contiguous, balanced split of n_queries whole queries over `world` ranks (strong
    scaling); returns (first_row, n_rows) of rank's shard.  Queries are never split across
    ranks (a query's rows are one service request, Table 3)."""
    if world <= 0 or not 0 <= rank < world:
        raise ValueError("bad world/rank")
    base, extra = divmod(n_queries, world)
    q0 = rank * base + min(rank, extra)
    nq = base + (1 if rank < extra else 0)
    return q0 * rows_per_query, nq * rows_per_query


def weak_shard(rows_per_rank: int, rank: int) -> Tuple[int, int]:
    """Weak scaling: every rank serves its own fixed batch; rank r's rows are the r-th block
    of the global query stream."""
    return rank * rows_per_rank, rows_per_rank


class _CudaArray:
    """__cuda_array_interface__ view of a raw device allocation (the library's weight arena)."""

    def __init__(self, ptr: int, nbytes: int):
        self.__cuda_array_interface__ = {"shape": (nbytes,), "typestr": "|u1", "data": (ptr, False), "version": 3}


def arena_tensor(net) -> torch.Tensor:
    """A zero-copy uint8 torch view of a loaded DjinnNet's weight arena (device memory)."""
    ptr, nbytes = net.arena()
    return torch.as_tensor(_CudaArray(ptr, nbytes), device=f"cuda:{net.device}")


def broadcast_buffer(buf: torch.Tensor, src: int = 0) -> torch.Tensor:
    """C1: one-time broadcast of a packed weight arena (or any byte buffer) from `src`."""
    if dist.is_initialized() and dist.get_world_size() > 1:
        dist.broadcast(buf, src=src)
    return buf


def max_over_ranks(value: float, device=None) -> float:
    """The harness's step time is the MAX over ranks (never a wall-clock of one rank)."""
    if not (dist.is_initialized() and dist.get_world_size() > 1):
        return float(value)
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def gather_rows(local: torch.Tensor, dst: int = 0):
    """C2 (optional): gather every rank's output rows to `dst` (list of tensors on dst)."""
    if not (dist.is_initialized() and dist.get_world_size() > 1):
        return [local]
    world = dist.get_world_size()
    sizes = torch.tensor([local.shape[0]], device=local.device)
    all_sizes = [torch.zeros_like(sizes) for _ in range(world)]
    dist.all_gather(all_sizes, sizes)
    n_max = int(max(s.item() for s in all_sizes))
    pad = torch.zeros((n_max,) + tuple(local.shape[1:]), dtype=local.dtype, device=local.device)
    pad[: local.shape[0]] = local
    out = [torch.zeros_like(pad) for _ in range(world)] if dist.get_rank() == dst else None
    dist.gather(pad, out, dst=dst)
    if out is None:
        return None
    return [o[: int(s.item())] for o, s in zip(out, all_sizes)]
