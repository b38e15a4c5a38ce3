"""NEXT-4 through torch.distributed: one system split over 2 ranks (both on
cuda:0 here -- the box has one GPU -- with gloo carrying the 8-value maps through
host memory; on a multi-GPU box the same driver all-gathers on NCCL).  Each
rank solves its slice with dist.solve_one_system_sliced; rank 0 compares the
assembled x with the CPU oracle."""
import os

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _worker(rank, world, port, cuts, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import trigen
        from paper_conf_icpp_kimwch11_b200 import dist as tdist
        n = cuts[-1]
        arrs = trigen.generate(n, 1, "f64", 0, "dd")
        sl = [torch.from_numpy(t[cuts[rank]:cuts[rank + 1]].copy()).cuda() for t in arrs]
        x = tdist.solve_one_system_sliced(*sl)
        torch.cuda.synchronize()
        q.put((rank, x.cpu().numpy()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("cuts", [[0, 300000, 1 << 20], [0, 65536, 131072, 196608]])
def test_one_system_two_ranks(cuda_ok, cuts):
    import oracle
    import trigen
    world = len(cuts) - 1
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 31000 + (os.getpid() % 2000)
    procs = [ctx.Process(target=_worker, args=(r, world, port, cuts, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=300) for _ in range(world)], key=lambda r: r[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    x = np.concatenate([r[1] for r in res])
    n = cuts[-1]
    arrs = trigen.generate(n, 1, "f64", 0, "dd")
    xo = oracle.solve_batch(n, 1, *arrs)
    assert np.max(np.abs(x - xo) / np.abs(xo)) <= 1e-10
