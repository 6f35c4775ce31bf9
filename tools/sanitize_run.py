"""Small J/K workloads that reach every kernel family, for compute-sanitizer:
    compute-sanitizer --tool {memcheck,synccheck,initcheck} python tools/sanitize_run.py
    compute-sanitizer --tool racecheck python tools/sanitize_run.py small   (racecheck is ~1000x slower)
benzene def2-SVP (plain, density-screened, mixed-precision tiers), a contracted s/p/d/f basis on 3 centres
(every l <= 3 class, all five families incl. the transposed ones), a 2-centre s..g basis (the l = 4
classes), mako_eri_batch (store kernels, FP64 and TF32) and an accumulate build."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import mako_inputs as mi  # noqa: E402
from paper_conf_sc_han0jlacz0025_b200 import Basis, Pairs, build_jk, eri_batch  # noqa: E402


def basis(centres, lmax, kchoice, seed):
    rng = np.random.default_rng(seed)
    xyz = rng.uniform(-1.6, 1.6, size=(centres, 3))
    at, ls, nps, ex, cf = [], [], [], [], []
    for a in range(centres):
        for l in range(lmax + 1):
            k = int(rng.choice(kchoice))
            at.append(a); ls.append(l); nps.append(k)
            ex += list(np.sort(np.exp(rng.uniform(np.log(0.15), np.log(8.0), k)))[::-1])
            cf += list(rng.uniform(0.2, 1.0, k))
    sh = mi.Shells(np.array(at, np.int32), np.array(ls, np.int32), np.array(nps, np.int32), xyz[np.array(at)],
                   np.array(ex), np.array(cf))
    return sh, np.ones(centres, np.int32), xyz


def run(sh, Z, xyz, nocc, mixed=True):
    B = Basis(Z, xyz, sh)
    P = Pairs(B, 1e-12)
    D = torch.tensor(mi.synthetic_density(sh.nbf(), nocc, seed=1), device="cuda")
    J, K = build_jk(P, D)
    build_jk(P, D, J=J, K=K, density_screen=True, thresh=1e-10)
    build_jk(P, D, J=J, K=K, accumulate=True)
    build_jk(P, D, J=J, K=K, shard=1, nshards=3)
    if mixed:
        build_jk(P, D, J=J, K=K, thresh_fp64=1e30)
    torch.cuda.synchronize()
    return B


small = len(sys.argv) > 1 and sys.argv[1] == "small"  # racecheck: the 3-centre s/p/d/f basis only
if not small:
    m, b = mi.config_molecule("benzene-def2svp")
    run(mi.shells_for(m, b), m.Z, m.xyz_bohr, m.nelec // 2)
sh, Z, xyz = basis(3 if not small else 2, 3, (1, 3), 0)
B = run(sh, Z, xyz, 10 if not small else 6)
q = [[int(a), int(b_), int(c), int(d)] for a, b_, c, d in np.random.default_rng(0).integers(0, sh.nshell, (64, 4))]
eri_batch(B, q)
eri_batch(B, q, reduced=True)
if not small:
    sh, Z, xyz = basis(2, 4, (1, 2), 3)
    run(sh, Z, xyz, 8, mixed=False)
torch.cuda.synchronize()
print("sanitize workload done")
