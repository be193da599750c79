"""Row-sharded multi-GPU A-ABFT; one process per GPU, torch.distributed.

Rank r owns rows [r*M/G, (r+1)*M/G) of A (a multiple of BS); B is replicated.  Every BS x BS
block's encode, bound, check and correction is rank-local (the partitioned encoding of P:L91
makes blocks independent).  The single exchange is the fault-counter reduction after
aabft_correct: SUM over the int64 counters and MAX over max |d|/eps, so every rank learns
whether any block anywhere was corrected or is uncorrectable.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def shard_rows(M: int, world: int, rank: int, bs: int) -> tuple[int, int]:
    """(first row, number of rows) of this rank's slab; slabs are BS-aligned and cover M."""
    if M % bs:
        raise ValueError("M must be a multiple of bs")
    nblk = M // bs
    lo = nblk * rank // world
    hi = nblk * (rank + 1) // world
    return lo * bs, (hi - lo) * bs


def reduce_counts(counts: torch.Tensor, group=None) -> torch.Tensor:
    """In-place all-reduce of an aabft_counts buffer (int64[9]: n[8] + max_ratio bits)."""
    if counts.dtype != torch.int64 or counts.numel() != 9:
        raise ValueError("counts must be the int64[9] aabft_counts buffer")
    dist.all_reduce(counts[:8], op=dist.ReduceOp.SUM, group=group)
    dist.all_reduce(counts[8:9].view(torch.float64), op=dist.ReduceOp.MAX, group=group)
    return counts


def broadcast_operand(B: torch.Tensor, src: int = 0, group=None) -> torch.Tensor:
    dist.broadcast(B, src=src, group=group)
    return B


def protected_matmul(A_local, B, *, bs: int = 64, p: int = 2, omega: float = 3.0, t: int = 0,
                     fma_model: int = 1, correct: bool = True, faults=None, group=None,
                     plan=None):
    """Protected C_local = A_local @ B on this rank, then the NCCL counter all-reduce.

    Returns (result, global_counts_dict).  ``plan`` (api.ProtectedGemm) may be passed to reuse
    buffers across calls."""
    from . import api
    M, K = A_local.shape
    N = B.shape[1]
    if plan is None:
        plan = api.ProtectedGemm(M, N, K, dtype=A_local.dtype, bs=bs, p=p, omega=omega, t=t,
                                 fma_model=fma_model, device=A_local.device)
    res = plan.run(A_local, B, faults=faults, correct=correct)
    if dist.is_available() and dist.is_initialized():
        reduce_counts(plan.counts, group)
    return res, api.counts_dict(plan.counts)
