"""Host-side multi-GPU logic on CPU with the gloo backend, world size 2 (no GPU needed).

The CUDA path itself is single-GPU here; what is tested is the sharding arithmetic and the
fault-counter exchange (SUM of int64 counters, MAX of max |d|/eps) -- SURVEY §8(e)."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_dsn_braunhw14_b200.distributed import reduce_counts, shard_rows


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        c = torch.zeros(9, dtype=torch.int64)
        # rank-local counters as aabft_check/aabft_correct would leave them
        c[:8] = torch.tensor([64, 63 - rank, rank, 1 - rank, 0, 8000 + rank, 3, 2 * rank + 2])
        c[8:9].view(torch.float64)[0] = [0.25, 7.5][rank]
        reduce_counts(c)
        q.put((rank, c[:8].tolist(), float(c[8:9].view(torch.float64)[0])))
        # padded all-gather of unequal per-rank row counts (the sharded B encoding's exchange)
        from paper_conf_dsn_braunhw14_b200.distributed import _all_gather_padded
        x = torch.arange(3 * (rank + 1) * 2, dtype=torch.float64).reshape(3 * (rank + 1), 2) + 100 * rank
        parts = _all_gather_padded(x, 6)
        q.put(("G", rank, [p.tolist() for p in parts]))
        # B replication: broadcast from rank 0
        B = torch.arange(6, dtype=torch.float64) if rank == 0 else torch.zeros(6, dtype=torch.float64)
        dist.broadcast(B, src=0)
        q.put(("B", rank, B.tolist()))
    finally:
        dist.destroy_process_group()


def test_counts_allreduce_gloo_world2():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = [q.get(timeout=120) for _ in range(6)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    counts = [o for o in out if o[0] not in ("B", "G")]
    bs = [o for o in out if o[0] == "B"]
    for _, rank, parts in [o for o in out if o[0] == "G"]:
        for r, part in enumerate(parts):
            exp = torch.arange(3 * (r + 1) * 2, dtype=torch.float64).reshape(3 * (r + 1), 2) + 100 * r
            assert part == exp.tolist()
    assert len(counts) == 2
    for rank, n, mr in counts:
        assert n == [128, 63 + 62, 1, 1, 0, 16001, 6, 6]
        assert mr == 7.5
    for _, rank, b in bs:
        assert b == [0, 1, 2, 3, 4, 5]


@pytest.mark.parametrize("M,world,bs", [(4096, 8, 64), (16384, 8, 64), (1024, 3, 64), (256, 2, 32)])
def test_shard_rows_cover_and_align(M, world, bs):
    seen = []
    for r in range(world):
        r0, n = shard_rows(M, world, r, bs)
        assert r0 % bs == 0 and n % bs == 0
        seen.append((r0, n))
    assert seen[0][0] == 0
    for (a0, an), (b0, _) in zip(seen, seen[1:]):
        assert a0 + an == b0
    assert seen[-1][0] + seen[-1][1] == M
    assert max(n for _, n in seen) - min(n for _, n in seen) <= bs


def test_shard_rows_rejects_unpadded():
    with pytest.raises(ValueError):
        shard_rows(100, 2, 0, 64)
