"""One J/K build of a config (for ncu captures): python tools/profile_build.py [--config X] [--builds N]"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import mako_inputs as mi  # noqa: E402
from paper_conf_sc_han0jlacz0025_b200 import Basis, Pairs, build_jk  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="valinomycin-def2tzvp")
ap.add_argument("--builds", type=int, default=1)
ap.add_argument("--tau", type=float, default=1e-12)
ap.add_argument("--shard", type=int, default=0)
ap.add_argument("--nshards", type=int, default=1)
ap.add_argument("--thresh-fp64", type=float, default=None, help="reduced-precision build (mako_build_jk_mixed)")
a = ap.parse_args()
mol, basis = mi.config_molecule(a.config)
sh = mi.shells_for(mol, basis)
P = Pairs(Basis(mol.Z, mol.xyz_bohr, sh), a.tau)
D = torch.tensor(mi.synthetic_density(sh.nbf(), mol.nelec // 2, seed=0), device="cuda")
for _ in range(a.builds):
    J, K = build_jk(P, D, shard=a.shard, nshards=a.nshards, thresh_fp64=a.thresh_fp64)
torch.cuda.synchronize()
print("done", float(J.abs().sum()), float(K.abs().sum()))
