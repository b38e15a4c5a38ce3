"""Row A6 / SURVEY 8(e) on the CUDA path: batch shards over 2 ranks (both on
cuda:0 -- the test box has one GPU -- with gloo carrying the edge collectives
through host memory; on the 8-GPU box the same driver runs NCCL over NVLink).
Each rank solves its systems with the CUDA Plan (C ABI, dist.cuda_solver);
rank 0 compares the gathered x with the CPU oracle element by element.
Two paths (PAPER.md P:699 / P:747: M independent systems):
  * scatter: rank 0 holds a, b, c, d -> scatter_inputs -> Plan per shard -> gather_x;
  * resident: every rank generates its own shard on its device (counter-based
    inputs, shard-invariant) -> solve_sharded -> gather_x."""
import os

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


CASES = [(16384, 37, 0, "f64"), (16384, 37, 1, "f64"), (1024, 1001, 1, "f64"), (256, 4099, 0, "f32"),
         (256, 4099, 1, "f32"), (1000, 300, 0, "f64")]


def _worker(rank, world, port, path, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        for case in CASES:
            q.put(_one(rank, world, path, *case))
    finally:
        dist.destroy_process_group()


def _one(rank, world, path, n, m, layout, dtype):
    import trigen
    import paper_conf_icpp_kimwch11_b200 as tri
    from paper_conf_icpp_kimwch11_b200 import dist as tdist
    td = tri.F64 if dtype == "f64" else tri.F32
    tdt = torch.float64 if dtype == "f64" else torch.float32
    solve_fn = tdist.cuda_solver(n, td, layout)
    q0, mr = tdist.shard_range(m, world, rank)
    if path == "scatter":
        full = None
        if rank == 0:
            full = [torch.from_numpy(t).cuda() for t in trigen.generate(n, m, dtype, layout, "dd")]
        a, b, c, d = tdist.scatter_inputs(n, m, full, layout, dtype=tdt, device=torch.device("cuda", 0))
        x = solve_fn(a, b, c, d, mr) if mr else torch.empty(0, dtype=tdt, device="cuda")
        full_x = tdist.gather_x(x, n, m, layout)
    else:
        def make_inputs(qq0, qmr):
            return [torch.from_numpy(t).cuda() for t in trigen.generate(n, qmr, dtype, layout, "dd", q0=qq0)]
        x, full_x = tdist.solve_sharded(n, m, make_inputs, solve_fn, layout=layout)
    torch.cuda.synchronize()
    return (rank, (n, m, layout, dtype), q0, mr, None if full_x is None else full_x.cpu().numpy())


@pytest.mark.parametrize("path", ["scatter", "resident"])
def test_sharded_cuda_solve(cuda_ok, path):
    import oracle
    import trigen
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 33000 + (os.getpid() % 2000) + (7 if path == "resident" else 0)
    procs = [ctx.Process(target=_worker, args=(r, world, port, path, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=600) for _ in range(world * len(CASES))]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for case in CASES:
        n, m, layout, dtype = case
        rs = sorted([r for r in res if r[1] == case], key=lambda r: r[0])
        cover = []
        for _, _, q0, mr, _ in rs:
            cover += list(range(q0, q0 + mr))
        assert cover == list(range(m)), case
        x = rs[0][4]
        assert x is not None and rs[1][4] is None
        arrs = trigen.generate(n, m, dtype, layout, "dd")
        xo = oracle.solve_batch(n, m, *arrs, layout=layout)
        err = float(np.max(np.abs(x.astype(np.float64) - xo) / np.abs(xo)))
        assert err <= (1e-10 if dtype == "f64" else 1e-4), (case, err)
