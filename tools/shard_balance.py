"""Per-rank work of an N-GPU J/K build, measured on ONE GPU (row e evidence while only one GPU is reachable):
    python tools/shard_balance.py --config valinomycin-def2tzvp --nshards 8 [--shards 0,3]
Builds the pair data once, then times mako_build_jk(shard=r, nshards=N) for each r with CUDA events
(warm-up build first).  Reports per-shard seconds, max/mean (the compute-only strong-scaling
efficiency of the N-GPU job is mean/max x N-way split of the 1-GPU time) and the algorithmic FLOPs per
shard.  The NCCL broadcast(D) + all_reduce([J;K]) of the real multi-GPU step are not included."""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import mako_inputs as mi  # noqa: E402
from paper_conf_sc_han0jlacz0025_b200 import Basis, Pairs, build_jk  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="valinomycin-def2tzvp")
ap.add_argument("--nshards", type=int, default=8)
ap.add_argument("--shards", default=None, help="comma list (default: all)")
ap.add_argument("--tau", type=float, default=1e-12)
ap.add_argument("--full", action="store_true", help="also time the unsharded build")
a = ap.parse_args()
mol, basis = mi.config_molecule(a.config)
sh = mi.shells_for(mol, basis)
n = sh.nbf()
t0 = time.perf_counter()
P = Pairs(Basis(mol.Z, mol.xyz_bohr, sh), a.tau)
pair_s = time.perf_counter() - t0
D = torch.tensor(mi.synthetic_density(n, mol.nelec // 2, seed=0), device="cuda")
J, K = torch.empty_like(D), torch.empty_like(D)
shards = list(range(a.nshards)) if a.shards is None else [int(x) for x in a.shards.split(",")]
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
build_jk(P, D, J=J, K=K, shard=shards[0], nshards=a.nshards)  # warm-up (plan, code paths)
torch.cuda.synchronize()
res = []
for r in shards:
    e0.record()
    build_jk(P, D, J=J, K=K, shard=r, nshards=a.nshards)
    e1.record()
    torch.cuda.synchronize()
    f = P.flops(shard=r, nshards=a.nshards)
    res.append({"shard": r, "s": e0.elapsed_time(e1) / 1e3, "gemm_flops": f["gemm_flops"], "quartets": f["quartets"]})
    print(json.dumps(res[-1]), flush=True)
ts = [x["s"] for x in res]
out = {"config": a.config, "nbf": n, "shells": sh.nshell, "nshards": a.nshards, "pair_build_s": pair_s,
       "shard_s": ts, "max_s": max(ts), "mean_s": sum(ts) / len(ts), "max_over_mean": max(ts) / (sum(ts) / len(ts)),
       "total_flops": P.flops()["gemm_flops"]}
if a.full:
    e0.record()
    build_jk(P, D, J=J, K=K)
    e1.record()
    torch.cuda.synchronize()
    out["full_build_s"] = e0.elapsed_time(e1) / 1e3
    if len(ts) == a.nshards:
        out["compute_only_efficiency"] = out["full_build_s"] / (a.nshards * max(ts))
print(json.dumps(out), flush=True)
