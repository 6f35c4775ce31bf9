"""Host logic of the multi-GPU path (broadcast D -> shard build -> all_reduce J, K) under gloo,
world_size 2, with the oracle's own shard split standing in for the GPU build (the GPU shard
function itself is covered by tests/test_gpu_jk.py::test_shards_sum)."""
import os

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _worker(rank, world, port, ret):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    import mako_inputs as mi
    from paper_conf_sc_han0jlacz0025_b200 import dist as mdist
    m = mi.h2o_baseline()
    sh = mi.shells_for(m, "sto-3g")
    n = sh.nbf()
    D = torch.from_numpy(mi.synthetic_density(n, 5, seed=3)) if rank == 0 else torch.zeros(n, n, dtype=torch.float64)

    def cpu_build(pairs, D, thresh=None, J=None, K=None, shard=0, nshards=1):
        j, k = oracle.jk(sh, D.numpy(), 0.0, shard, nshards)
        if J is None:
            return torch.from_numpy(j), torch.from_numpy(k)
        J.copy_(torch.from_numpy(j))
        K.copy_(torch.from_numpy(k))
        return J, K

    # separate J, K tensors (two collectives) and one preallocated [2, n, n] buffer (one in-place collective)
    J, K = mdist.distributed_build_jk(None, D, build=cpu_build)
    buf, Jv, Kv = mdist.jk_buffer(n, "cpu")
    ptr = buf.data_ptr()
    J2, K2 = mdist.distributed_build_jk(None, D, J=Jv, K=Kv, build=cpu_build)
    assert J2.data_ptr() == ptr and K2.data_ptr() == ptr + n * n * 8
    if rank == 0:
        j0, k0 = oracle.jk(sh, D.numpy(), 0.0)
        ret["err"] = float(max(np.abs(J.numpy() - j0).max(), np.abs(K.numpy() - k0).max()))
        ret["err_buf"] = float(max(np.abs(buf[0].numpy() - j0).max(), np.abs(buf[1].numpy() - k0).max()))
    dist.destroy_process_group()


def test_gloo_world2_broadcast_allreduce():
    mgr = mp.Manager()
    ret = mgr.dict()
    port = 29500 + os.getpid() % 1000
    mp.spawn(_worker, args=(2, port, ret), nprocs=2, join=True)
    assert ret["err"] < 1e-13
    assert ret["err_buf"] < 1e-13
