"""Multi-GPU driver for batches of independent systems (PAPER.md
P:699 Sec. III.D and P:747 Sec. IV: M independent systems).

The m systems are split into contiguous ranges, one per rank (tri_shard_range);
each rank solves its shard on its own GPU with no collective inside the solve
(the systems are independent: Eq 1 per system).  Collectives
appear only at the edges:
  * scatter_inputs: rank 0 hands each rank its a, b, c, d shard;
  * gather_x:  rank 0 collects the solution (NCCL over NVLink on the GPU box,
               gloo in the CPU tests);
  * max_over_ranks: the timing convention (job time = slowest rank).
A rank holds its shard in the same layout as the full batch with m_r columns
(CONTIGUOUS: [ql*n + i]; INTERLEAVED: [i*m_r + ql]).  The per-shard solver on
the GPU is cuda_solver (the CUDA Plan through the C ABI); with the gloo backend
(CPU tests, or several ranks sharing one GPU) the edge collectives run on host
copies of the device shards.
"""
import torch
import torch.distributed as dist

from . import CONTIGUOUS, INTERLEAVED, shard_range as _abi_shard_range


def shard_range(m, world, rank):
    """(q0, m_r): rank r owns systems [q0, q0 + m_r) (tri_shard_range)."""
    return _abi_shard_range(int(m), int(world), int(rank))


def _host_collectives(group, t):
    """gloo moves host tensors only: run its collectives on CPU copies."""
    return dist.get_backend(group) == "gloo" and t is not None and t.is_cuda


def cuda_solver(n, dtype, layout=CONTIGUOUS):
    """solve_fn for solve_sharded: the CUDA Plan (C ABI) of the rank's shard,
    created once per shard size and reused; inputs are moved to the current
    CUDA device if they are not already there."""
    from . import Plan
    plans = {}

    def solve_fn(a, b, c, d, mr):
        dev = torch.device("cuda", torch.cuda.current_device())
        a, b, c, d = (t.to(dev) for t in (a, b, c, d))
        if mr not in plans:
            plans[mr] = Plan(n, mr, dtype, layout)
        return plans[mr].solve(a, b, c, d)
    return solve_fn


def max_over_ranks(value, group=None, device=None):
    """Maximum of a python float over all ranks (all-reduce MAX)."""
    if not dist.is_available() or not dist.is_initialized():
        return float(value)
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())


def gather_x(x_local, n, m, layout=CONTIGUOUS, group=None, dst=0):
    """Assemble the full solution (n*m) on rank `dst` from every rank's shard.
    Returns the full tensor on dst, None elsewhere.  Shards are padded to
    ceil(m/G) systems for the collective and unpadded on the root."""
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    per = -(-m // world)
    q0, mr = shard_range(m, world, rank)
    dev_out = x_local.device
    if _host_collectives(group, x_local):
        x_local = x_local.cpu()
    pad = torch.zeros(n * per, dtype=x_local.dtype, device=x_local.device)
    if layout == CONTIGUOUS:
        pad[: n * mr] = x_local
    else:
        pad.view(n, per)[:, :mr] = x_local.view(n, mr)
    bufs = [torch.empty_like(pad) for _ in range(world)] if rank == dst else None
    dist.gather(pad, gather_list=bufs, dst=dst, group=group)
    if rank != dst:
        return None
    full = torch.empty(n * m, dtype=x_local.dtype, device=x_local.device)
    for r in range(world):
        rq0, rmr = shard_range(m, world, r)
        if rmr == 0:
            continue
        if layout == CONTIGUOUS:
            full[rq0 * n:(rq0 + rmr) * n] = bufs[r][: n * rmr]
        else:
            full.view(n, m)[:, rq0:rq0 + rmr] = bufs[r].view(n, per)[:, :rmr]
    return full.to(dev_out)


def scatter_inputs(n, m, full=None, layout=CONTIGUOUS, group=None, src=0, dtype=None, device=None):
    """Distribute a, b, c, d from rank `src` (dist.scatter of the
    input shards).  `full` (on src only): the 4 full n*m tensors.  Every rank
    receives its systems [q0, q0+m_r) in the same layout with m_r columns.
    Shards are padded to ceil(m/G) systems for the collective."""
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    per = -(-m // world)
    q0, mr = shard_range(m, world, rank)
    if rank == src:
        dtype, device = full[0].dtype, full[0].device
    dev_out = device
    if device is not None and _host_collectives(group, torch.empty(0, device=device)):
        device = torch.device("cpu")
        if full is not None:
            full = [t.cpu() for t in full]
    out = []
    for arr in range(4):
        recv = torch.zeros(n * per, dtype=dtype, device=device)
        send = None
        if rank == src:
            send = []
            for r in range(world):
                rq0, rmr = shard_range(m, world, r)
                buf = torch.zeros(n * per, dtype=dtype, device=device)
                if rmr:
                    if layout == CONTIGUOUS:
                        buf[: n * rmr] = full[arr][rq0 * n:(rq0 + rmr) * n]
                    else:
                        buf.view(n, per)[:, :rmr] = full[arr].view(n, m)[:, rq0:rq0 + rmr]
                send.append(buf)
        dist.scatter(recv, scatter_list=send, src=src, group=group)
        if layout == CONTIGUOUS:
            out.append(recv[: n * mr].clone().to(dev_out))
        else:
            out.append(recv.view(n, per)[:, :mr].contiguous().view(-1).to(dev_out))
    return out


def solve_sharded(n, m, make_inputs, solve_fn, layout=CONTIGUOUS, gather=True, group=None):
    """Solve this rank's shard.  make_inputs(q0, m_r) -> (a, b, c, d) for the
    global systems [q0, q0+m_r) (generated locally: shards stay resident, no
    scatter); solve_fn(a, b, c, d, m_r) -> x.  Returns (x_local, x_full or None)."""
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    q0, mr = shard_range(m, world, rank)
    if mr > 0:
        a, b, c, d = make_inputs(q0, mr)
        x = solve_fn(a, b, c, d, mr)
    else:
        x = torch.empty(0, dtype=torch.float64)
    full = gather_x(x, n, m, layout, group) if (gather and world > 1) else (x if gather else None)
    return x, full


def solve_one_system_sliced(a, b, c, d, group=None, allgather=None):
    """One system spread over the ranks: every rank holds a
    contiguous slice of its rows (a, b, c, d: this rank's slice, device tensors,
    len % 8 == 0, > 256 rows) and gets x of its slice back.  The slices exchange
    only their 8-value forward and backward maps (two all-gathers, NCCL over
    NVLink on the GPU box); all arithmetic runs in the SCAN_MC kernels
    (tri_slice_solve).  `allgather(t) -> [t_0, ..., t_{G-1}]` overrides the
    collective (tests run several slices on one device)."""
    from . import Plan, VARIANT_SCAN_MC, F64, F32, OPT_SCAN_MC_LOOKBACK
    if allgather is None:
        world = dist.get_world_size(group)
        rank = dist.get_rank(group)

        on_host = dist.get_backend(group) == "gloo"  # gloo: the 8-value maps travel through host memory

        def allgather(t):
            src = t.cpu() if on_host else t
            out = [torch.empty_like(src) for _ in range(world)]
            dist.all_gather(out, src, group=group)
            return [o.to(t.device) for o in out]
    else:
        world, rank = allgather.world, allgather.rank
    n = a.numel()
    plan = Plan(n, 1, F64 if a.dtype == torch.float64 else F32, 0)
    plan.variant = VARIANT_SCAN_MC
    plan.set_option(OPT_SCAN_MC_LOOKBACK, 0)  # the sliced phases are the three-pass form
    fmap = plan.slice_phase(0, rank, world, a, b, c, d)
    maps = torch.cat(allgather(fmap))
    bmap = plan.slice_phase(1, rank, world, a, b, c, d, maps=maps)
    bmaps = torch.cat(allgather(bmap))
    return plan.slice_phase(2, rank, world, maps=bmaps)
