"""The row-sharded distributed path at world size 2 on ONE GPU (gloo backend, both ranks on
cuda:0; the round's GPU box has one B200): ShardedProtectedGemm encodes each rank's rows of A
and column range of B in the sm_100a kernels, all-gathers the B encoding, runs the GEMM, check
and correction of the local rows and all-reduces the fault counters.  Checked
against the CPU oracle on the full problem: the gathered Bcs and top-p tables of B bit for bit,
C within 1e-13 of |A||B|, one fault per rank located and corrected, global counters."""
import os
import socket

import numpy as np
import pytest

import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


M, N, K, BS, P = 512, 448, 300, 64, 2
FAULTS = {0: dict(row=70, col=100, site=2, add=3.0),      # rank-local row coordinates
          1: dict(row=5, col=400, site=0, xor_mask=1 << 62)}


def _worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_dsn_braunhw14_b200 import api
        from paper_conf_dsn_braunhw14_b200.distributed import ShardedProtectedGemm, shard_rows
        r0, m = shard_rows(M, world, rank, BS)
        A = torch.from_numpy(synth.generate("uniform", m, K, seed=3, matrix_id=0, row0=r0,
                                            full_cols=K)).cuda()
        B = torch.from_numpy(synth.generate("uniform", K, N, seed=3, matrix_id=1)).cuda()
        sp = ShardedProtectedGemm(m, N, K, world=world, rank=rank, bs=BS, p=P, device="cuda:0")
        res = sp.run(A, B, faults=[FAULTS[rank]])
        torch.cuda.synchronize()
        pl = sp.plan
        q.put((rank, r0, res.C.cpu().numpy(), pl.Bcs.cpu().numpy(), pl.topB_val.cpu().numpy(),
               pl.topB_idx.cpu().numpy(), res.reports()["status"], api.counts_dict(pl.counts)))
    finally:
        dist.destroy_process_group()


def test_sharded_b_encode_world2_one_gpu(orc):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = sorted([q.get(timeout=300) for _ in range(2)], key=lambda o: o[0])
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    A = synth.generate("uniform", M, K, seed=3, matrix_id=0)
    B = synth.generate("uniform", K, N, seed=3, matrix_id=1)
    gfaults = [dict(FAULTS[r], row=FAULTS[r]["row"] + out[r][1]) for r in range(2)]
    o = orc.protected_matmul(A, B, bs=BS, p=P, faults=gfaults)
    enc = o["enc"]
    denom = np.abs(A) @ np.abs(B)
    Cg = np.concatenate([out[0][2], out[1][2]])
    assert np.max(np.abs(Cg - o["C"]) / denom) <= 1e-13
    st = np.concatenate([out[0][6], out[1][6]])
    assert np.array_equal(st, o["check"].status)
    for rank, r0, C, Bcs, tv, ti, status, cnt in out:
        assert np.array_equal(Bcs, enc["Bcs"])              # all-gathered checksum columns
        assert np.array_equal(tv, enc["topB"][0]) and np.array_equal(ti, enc["topB"][1])
        assert cnt["blocks"] == (M // BS) * (N // BS)
        assert cnt["corrected"] == 2 and cnt["checks_critical"] == 4  # global, all-reduced
        assert cnt["clean"] == cnt["blocks"] - 2
