"""Row-sharded multi-GPU A-ABFT; one process per GPU, torch.distributed.

Rank r owns rows [r*M/G, (r+1)*M/G) of A (a multiple of BS); B is replicated (one broadcast,
outside the step).  Every BS x BS block's encode, bound, check and correction is rank-local
(the partitioned encoding of P:L91 makes blocks independent).  Two exchanges:

* the encoding of B (Alg 1 steps 1c/1d) is sharded by BS-aligned column ranges:
  rank r encodes its columns of B -- the checksum columns Bcs[:, J] and the top-p of its data
  and checksum columns, in the sm_100a encode kernel -- and one all-gather gives every rank
  the full Bcs and top-p tables of B (ShardedProtectedGemm), instead of every rank re-reading
  all of B;
* after the check (which corrects in the same kernel), the fault counters: SUM over the int64 counters and MAX over
  max |d|/eps, so every rank learns whether any block anywhere was corrected or is
  uncorrectable.
Collectives are NCCL over NVLink on the GPU box; the gloo backend (CPU staging) lets the same
code run with several ranks on one GPU or on CPU tests.
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
    c = counts.cpu() if (counts.is_cuda and dist.get_backend(group) == "gloo") else counts
    dist.all_reduce(c[:8], op=dist.ReduceOp.SUM, group=group)
    dist.all_reduce(c[8:9].view(torch.float64), op=dist.ReduceOp.MAX, group=group)
    if c is not counts:
        counts.copy_(c)
    return counts


def broadcast_operand(B: torch.Tensor, src: int = 0, group=None) -> torch.Tensor:
    dist.broadcast(B, src=src, group=group)
    return B


def shard_cols(N: int, world: int, rank: int, bs: int) -> tuple[int, int]:
    """(first column, number of columns) of this rank's BS-aligned column range of B."""
    return shard_rows(N, world, rank, bs)


def _backend(group=None) -> str:
    return dist.get_backend(group)


def _all_gather_padded(x: torch.Tensor, rows_max: int, group=None) -> list[torch.Tensor]:
    """All-gather of a (rows, ...) tensor whose row count differs between ranks: padded to
    rows_max, gathered into one buffer, returned as per-rank views of the valid rows.  NCCL
    works on the device buffers; gloo stages through the host (plumbing only)."""
    world = dist.get_world_size(group)
    pad = torch.zeros((rows_max,) + tuple(x.shape[1:]), dtype=x.dtype, device=x.device)
    pad[: x.shape[0]] = x
    n = torch.tensor([x.shape[0]], dtype=torch.int64, device=x.device)
    stage = _backend(group) == "gloo" and x.is_cuda
    dev = torch.device("cpu") if stage else x.device
    out = torch.empty((world * rows_max,) + tuple(x.shape[1:]), dtype=x.dtype, device=dev)
    ns = torch.empty(world, dtype=torch.int64, device=dev)
    dist.all_gather_into_tensor(out, pad.to(dev), group=group)
    dist.all_gather_into_tensor(ns, n.to(dev), group=group)
    out = out.to(x.device).view((world, rows_max) + tuple(x.shape[1:]))
    ns = ns.cpu()
    return [out[r, : int(ns[r])] for r in range(world)]


class ShardedProtectedGemm:
    """One rank of the row-sharded protected GEMM with the sharded B encoding.

    ``run(A_local, B)``: encode this rank's A rows (sm_100a kernel) and this rank's column range
    of B (checksum columns + top-p of its data / checksum columns), all-gather the B encoding,
    then the augmented GEMM, check and correction of the local rows, and the counter
    all-reduce.  ``B`` is the full (replicated) K x N operand."""

    def __init__(self, M_local: int, N: int, K: int, *, world: int, rank: int, group=None,
                 dtype=torch.float64, bs: int = 64, p: int = 2, omega: float = 3.0, t: int = 0,
                 fma_model: int = 1, device=None, fused: bool = True):
        from . import api
        self.world, self.rank, self.group = world, rank, group
        self.N, self.K, self.bs, self.p = N, K, bs, p
        self.plan = api.ProtectedGemm(M_local, N, K, dtype=dtype, bs=bs, p=p, omega=omega, t=t,
                                      fma_model=fma_model, device=device, fused=fused)
        self.c0, self.nc = shard_cols(N, world, rank, bs)
        self.ncmax = max(shard_cols(N, world, r, bs)[1] for r in range(world))
        # encode-only plan for this rank's columns of B (M = bs is a placeholder; A unused)
        self.bplan = api.ProtectedGemm(bs, max(self.nc, bs), K, dtype=dtype, bs=bs, p=p,
                                       omega=omega, t=t, fma_model=fma_model, device=device,
                                       fused=False) if self.nc > 0 else None
        self.timings = {}

    def encode(self, A_local, B, stream=None):
        """Step 1 with the B half sharded: local encode, then one all-gather."""
        pl, bs = self.plan, self.bs
        pl.encode(A_local, None, stream)
        nJ = self.nc // bs
        if self.nc > 0:
            self.bplan.encode(None, B[:, self.c0:self.c0 + self.nc], stream)
            bcs = self.bplan.Bcs[:, :nJ].t()                         # (nJ, K): checksum columns
            tv = self.bplan.topB_val[: self.nc + nJ]
            ti = self.bplan.topB_idx[: self.nc + nJ]
        else:
            bcs = torch.empty(0, self.K, dtype=pl.dtype, device=pl.device)
            tv = torch.empty(0, self.p, dtype=torch.float64, device=pl.device)
            ti = torch.empty(0, self.p, dtype=torch.int32, device=pl.device)
        nJmax = self.ncmax // bs
        # one gather per table (Bcs columns, top-p values, top-p indices) -- each padded
        gb = _all_gather_padded(bcs.contiguous(), nJmax, self.group)
        gv = _all_gather_padded(tv.contiguous(), self.ncmax + nJmax, self.group)
        gi = _all_gather_padded(ti.contiguous(), self.ncmax + nJmax, self.group)
        N = self.N
        for r in range(self.world):
            c0, nc = shard_cols(N, self.world, r, bs)
            J0, nj = c0 // bs, nc // bs
            if nc == 0:
                continue
            pl._Bcs[:, J0:J0 + nj] = gb[r].t()
            pl.topB_val[c0:c0 + nc] = gv[r][:nc]
            pl.topB_idx[c0:c0 + nc] = gi[r][:nc]
            pl.topB_val[N + J0:N + J0 + nj] = gv[r][nc:nc + nj]
            pl.topB_idx[N + J0:N + J0 + nj] = gi[r][nc:nc + nj]

    def run(self, A_local, B, *, faults=None, correct: bool = True, stream=None):
        pl = self.plan
        pl._check_operand(A_local, pl.M, pl.K, "A")
        pl._check_operand(B, pl.K, pl.N, "B")
        from . import api
        fbuf = faults if isinstance(faults, torch.Tensor) else api.make_faults(faults, pl.device)
        nf = 0 if fbuf is None else fbuf.numel() // 48
        self.encode(A_local, B, stream)
        pl.gemm(A_local, B, fbuf, nf, stream)
        pl.check(stream, correct=correct)  # correction inside the check kernel
        reduce_counts(pl.counts, self.group)
        return pl.result()


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
