"""GPU parity of the ERI stages (a4-a8) against the oracle, through the C ABI (mako_boys, mako_eri_batch).
Bar (BASELINE.json north_star): |Delta ERI| <= 1e-10; Boys: |Delta F| <= 5e-15 absolute (reading R1)."""
import itertools

import numpy as np
import pytest

import oracle
import mako_inputs as mi

pytestmark = pytest.mark.gpu


def test_boys_device_vs_oracle():
    import torch
    from paper_conf_sc_han0jlacz0025_b200 import boys
    T = np.concatenate([[0.0, 1e-14, 1e-8, 1e-3], np.linspace(0.01, 45, 3001), [39.99, 40.0, 40.01, 60, 150, 1e4, 1e7]])
    # m <= 16: the g classes ((gg|gg), L = 16) run boys_eval<16> (reading R1)
    F = boys(torch.tensor(T, device="cuda"), 16).cpu().numpy()
    ref = np.array([oracle.boys(16, t) for t in T])
    err = np.abs(F - ref)
    assert err.max() <= 5e-15, (err.max(), T[np.unravel_index(err.argmax(), err.shape)[0]])
    assert (err / np.maximum(ref, 1e-300)).max() <= 2e-14


def _mixed_basis(seed, nprim_choices=(1, 3)):
    """Shells of every l <= 3 on 3 centres, random exponents (log-U[0.1,10], SURVEY S8.d microbench)."""
    rng = np.random.default_rng(seed)
    centers = rng.uniform(-2, 2, size=(3, 3))
    ls, nps, xyz, ex, cf, at = [], [], [], [], [], []
    for a in range(3):
        for l in range(4):
            k = int(rng.choice(nprim_choices))
            ls.append(l); nps.append(k); xyz.append(centers[a]); at.append(a)
            ex += list(np.exp(rng.uniform(np.log(0.1), np.log(10.0), k)))
            cf += list(rng.uniform(0.2, 1.0, k))
    sh = mi.Shells(np.array(at, np.int32), np.array(ls, np.int32), np.array(nps, np.int32), np.array(xyz),
                   np.array(ex), np.array(cf))
    return sh, np.array([1, 1, 1], np.int32), centers


def _gpu_basis(sh, Z, centers):
    from paper_conf_sc_han0jlacz0025_b200 import Basis
    return Basis(Z, centers, sh)


@pytest.mark.parametrize("seed", [0, 1])
def test_eri_batch_all_55_classes(seed):
    from paper_conf_sc_han0jlacz0025_b200 import eri_batch
    sh, Z, centers = _mixed_basis(seed)
    B = _gpu_basis(sh, Z, centers)
    rng = np.random.default_rng(100 + seed)
    by_l = {l: [i for i in range(sh.nshell) if sh.l[i] == l] for l in range(4)}
    quartets = []
    # every (la lb | lc ld) pattern in every order -> all 55 canonical classes, all swap flags
    for la, lb, lc, ld in itertools.product(range(4), repeat=4):
        quartets.append([int(rng.choice(by_l[x])) for x in (la, lb, lc, ld)])
    blocks = eri_batch(B, quartets)
    worst = 0.0
    for q, blk in zip(quartets, blocks):
        ref = oracle.eri_quartet(sh, *q)
        err = np.abs(blk.cpu().numpy() - ref).max()
        worst = max(worst, err)
        assert err <= 1e-10, (q, err)
    print("max |dERI|", worst)


def test_eri_batch_contracted_and_coincident_centres():
    """Contracted shells (K up to 6) and quartets with repeated shells / centres (the degenerate cases)."""
    from paper_conf_sc_han0jlacz0025_b200 import eri_batch
    m, b = mi.config_molecule("benzene-def2svp")
    sh = mi.shells_for(m, b)
    keep = [0, 3, 5, 6, 7, 8, 9, 36]  # C (5-prim s, 3-prim p, d) + H shells
    sub = sh.subset(keep)
    B = _gpu_basis(sub, m.Z, m.xyz_bohr)
    q = [[0, 0, 0, 0], [1, 0, 1, 0], [2, 2, 2, 2], [4, 3, 0, 7], [3, 3, 3, 3], [5, 4, 3, 2], [7, 7, 0, 0],
         [6, 6, 5, 5], [1, 2, 3, 4]]
    blocks = eri_batch(B, q)
    for qq, blk in zip(q, blocks):
        ref = oracle.eri_quartet(sub, *qq)
        assert np.abs(blk.cpu().numpy() - ref).max() <= 1e-10, qq


def test_eri_batch_empty_and_validation():
    import torch
    from paper_conf_sc_han0jlacz0025_b200 import eri_batch, MakoError
    sh, Z, centers = _mixed_basis(3)
    B = _gpu_basis(sh, Z, centers)
    assert eri_batch(B, np.zeros((0, 4), np.int32)) == []
    with pytest.raises(MakoError):
        eri_batch(B, [[0, 0, 0, 999]])
