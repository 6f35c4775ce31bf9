"""Multi-GPU J/K: one process per GPU, torch.distributed for the plumbing.

Each rank holds the same (deterministic) pair data, builds its shard of the canonical quartet
tasks (mako_build_jk shard = rank, nshards = world), and the partial J/K are combined with one
all-reduce (NCCL over NVLink on the box; gloo in the CPU tests of the host logic).  D is
broadcast from rank 0 first.  This is the path's only exchange step (PAPER.md:L400 one MPI rank
per GPU; the combine itself is not described by the paper -- DESIGN.md reading R10).
"""
import torch
import torch.distributed as dist


def shard_of(rank, world):
    return int(rank), int(world)


def jk_buffer(n, device, dtype=torch.float64):
    """One preallocated [2, n, n] buffer; J = buf[0] and K = buf[1] are views, so the combine below
    reduces both in one collective without a staging copy (C5: 8 GB that would otherwise be
    re-allocated every build)."""
    buf = torch.empty((2, n, n), dtype=dtype, device=device)
    return buf, buf[0], buf[1]


def combine_jk(J, K, group=None):
    """Sum the per-rank partial J and K in one collective.  When J and K are the two halves of one
    jk_buffer the all_reduce runs in place on it; otherwise they are reduced one after the other
    (no temporary)."""
    if not dist.is_initialized() or dist.get_world_size(group) == 1:
        return J, K
    base = J._base
    if (base is not None and base is K._base and base.dim() == 3 and base.shape[0] == 2 and base.is_contiguous()
            and J.data_ptr() == base.data_ptr() and K.data_ptr() == base[1].data_ptr()):
        dist.all_reduce(base, op=dist.ReduceOp.SUM, group=group)
    else:
        dist.all_reduce(J, op=dist.ReduceOp.SUM, group=group)
        dist.all_reduce(K, op=dist.ReduceOp.SUM, group=group)
    return J, K


def distributed_build_jk(pairs, D, thresh=None, J=None, K=None, group=None, build=None):
    """broadcast(D) -> local shard build -> all_reduce(J, K).  ``build`` defaults to mako.build_jk;
    tests pass a CPU stand-in to exercise the host logic under gloo."""
    if build is None:
        from .mako import build_jk as build
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    if world > 1:
        dist.broadcast(D, src=0, group=group)
    J, K = build(pairs, D, thresh=thresh, J=J, K=K, shard=rank, nshards=world)
    return combine_jk(J, K, group)
