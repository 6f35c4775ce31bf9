"""The multi-GPU path with the real GPU build: two ranks, world_size 2, both on
cuda:0, joined by a gloo process group (collectives through the host, so neither rank's kernels wait on
the other's).  Each rank runs dist.distributed_build_jk -- broadcast(D) from rank 0, its shard of the
quartet tasks through mako_build_jk(shard = rank, nshards = 2), one all_reduce of [J; K] in the
preallocated [2, n, n] buffer -- and the combined J/K must equal the one-rank build and the oracle's.
On the 8-GPU box the same code runs over NCCL (bench.py under torchrun); only one GPU is reachable here."""
import os

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _worker(rank, world, port, ret):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    import mako_inputs as mi
    from paper_conf_sc_han0jlacz0025_b200 import Basis, Pairs, build_jk
    from paper_conf_sc_han0jlacz0025_b200 import dist as mdist
    m, b = mi.config_molecule("benzene-def2svp")
    sh = mi.shells_for(m, b)
    n = sh.nbf()
    P = Pairs(Basis(m.Z, m.xyz_bohr, sh), 1e-12)
    D0 = torch.tensor(mi.synthetic_density(n, m.nelec // 2, seed=5), device="cuda")
    D = D0.clone() if rank == 0 else torch.zeros_like(D0)
    buf, Jv, Kv = mdist.jk_buffer(n, "cuda")
    J, K = mdist.distributed_build_jk(P, D, J=Jv, K=Kv)
    torch.cuda.synchronize()
    assert J.data_ptr() == buf.data_ptr() and K.data_ptr() == buf[1].data_ptr()
    if rank == 0:
        J1, K1 = build_jk(P, D0)  # one rank, all tasks
        torch.cuda.synchronize()
        ret["d_one_rank"] = float(max((J - J1).abs().max(), (K - K1).abs().max()))
        ret["scale"] = float(max(J1.abs().max(), K1.abs().max()))
        ret["D_bcast"] = float((D - D0).abs().max())
        np.save(ret["path"] + ".J.npy", J.cpu().numpy())
        np.save(ret["path"] + ".K.npy", K.cpu().numpy())
        np.save(ret["path"] + ".D.npy", D0.cpu().numpy())
    dist.destroy_process_group()


def test_two_ranks_gloo_real_build(tmp_path):
    import oracle
    import mako_inputs as mi
    mgr = mp.Manager()
    ret = mgr.dict()
    ret["path"] = str(tmp_path / "jk")
    port = 29600 + os.getpid() % 1000
    mp.spawn(_worker, args=(2, port, ret), nprocs=2, join=True)
    assert ret["D_bcast"] == 0.0
    # shard sum vs one-rank build: same quartets, different FP64 summation order
    assert ret["d_one_rank"] <= 1e-12 * ret["scale"]
    J = np.load(ret["path"] + ".J.npy")
    K = np.load(ret["path"] + ".K.npy")
    D = np.load(ret["path"] + ".D.npy")
    m, b = mi.config_molecule("benzene-def2svp")
    sh = mi.shells_for(m, b)
    J0, K0 = oracle.jk(sh, D, 1e-12)
    assert np.abs(J - J0).max() <= 1e-8 and np.abs(K - K0).max() <= 1e-8
