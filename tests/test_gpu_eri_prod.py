"""ERI-level parity (|dERI| <= 1e-10, BASELINE.json north_star) of the PRODUCTION J/K kernels.

mako_eri_batch runs the warp-per-quartet store kernel for every class; the J/K build runs four other
kernel families for the low/mid-l classes (lane-per-ket, ket-first, ket-first transposed, slot-batched;
mako_class_family).  Their ERIs are read out of mako_build_jk itself with unit densities: for
D = e_ls + e_sl (one AO pair l, s of a shell pair),
    J_{mn} = sum (mn|l's') D_l's' = 2 (mn|ls)                   (Eq. 1; J of north_star)
    K_{mk} = sum (mn|ks') D_ns'   = (ml|ks) + (ms|kl)            (K of north_star)
so one build yields the full ERI column (..|ls) through every kernel that touches the shell pair
(l, s), in both bra and ket roles.  One AO pair per shell pair of a small contracted s/p/d/f (and a
g) basis covers every class of every family; the oracle's full ERI tensor is the reference.
"""
import itertools

import numpy as np
import pytest

import oracle
import mako_inputs as mi

pytestmark = pytest.mark.gpu


def _basis(centres, lmax, kchoice, seed):
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


def _columns(sh, Z, xyz, density_screen=False):
    import torch
    from paper_conf_sc_han0jlacz0025_b200 import Basis, Pairs, build_jk
    B = Basis(Z, xyz, sh)
    P = Pairs(B, 0.0)
    n = sh.nbf()
    off = B.ao_offsets
    eri = oracle.eri_full(sh)
    D = torch.zeros((n, n), dtype=torch.float64, device="cuda")
    J = torch.empty_like(D)
    K = torch.empty_like(D)
    worst_j = worst_k = 0.0
    for x, y in itertools.combinations_with_replacement(range(sh.nshell), 2):
        lam, sig = int(off[y]), int(off[x]) + (int(off[x + 1]) - int(off[x])) // 2  # first of y, middle of x
        D.zero_()
        D[lam, sig] = 1.0
        D[sig, lam] = 1.0
        build_jk(P, D, J=J, K=K, density_screen=density_screen, thresh=1e-14 if density_screen else None)
        torch.cuda.synchronize()
        Jh, Kh = J.cpu().numpy(), K.cpu().numpy()
        f = 1.0 if lam != sig else 0.5  # D = 2 e_ll when l == s
        refJ = 2.0 * f * eri[:, :, lam, sig]
        refK = f * (eri[:, lam, :, sig] + eri[:, sig, :, lam])
        dj, dk = np.abs(Jh - refJ).max(), np.abs(Kh - refK).max()
        worst_j, worst_k = max(worst_j, dj / 2), max(worst_k, dk)
        assert dj <= 2e-10, (x, y, dj)
        assert dk <= 2e-10, (x, y, dk)
    return worst_j, worst_k


@pytest.mark.parametrize("seed", [0, 1])
def test_production_kernels_eri_columns_spdf(seed):
    """Every l <= 3 class through the production kernel of its family; K in {1, 3} primitives."""
    from paper_conf_sc_han0jlacz0025_b200.mako import class_family
    fam = class_family()
    assert {0, 1, 2, 3, 4, 5} <= set(fam[:55])  # every family appears among the l <= 3 classes
    sh, Z, xyz = _basis(3, 3, (1, 3), seed)
    wj, wk = _columns(sh, Z, xyz)
    print("spdf production kernels: max |dERI| via J %.2e, via K %.2e" % (wj, wk))


def test_production_kernels_eri_columns_density_screened():
    """The density-screened instantiations (MAKO_JK_DENSITY_SCREEN, separate template instances of every
    family): with a unit density every quartet touching the (l, s) block survives a 1e-14 threshold."""
    sh, Z, xyz = _basis(3, 3, (1, 3), 5)
    _columns(sh, Z, xyz, density_screen=True)


def test_production_kernels_eri_columns_g():
    """The 65 classes with a g shell (l = 4, row f3) through their production kernels."""
    sh, Z, xyz = _basis(2, 4, (1, 2), 3)
    wj, wk = _columns(sh, Z, xyz)
    print("spdfg production kernels: max |dERI| via J %.2e, via K %.2e" % (wj, wk))
