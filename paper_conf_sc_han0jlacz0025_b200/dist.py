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


def combine_jk(J, K, group=None):
    """Sum the per-rank partial J and K in one collective (packed into one buffer)."""
    if not dist.is_initialized() or dist.get_world_size(group) == 1:
        return J, K
    buf = torch.stack([J, K])
    dist.all_reduce(buf, op=dist.ReduceOp.SUM, group=group)
    J.copy_(buf[0])
    K.copy_(buf[1])
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
