"""GPU parity of g functions (l = 4; def2-QZVP / cc-pVQZ)
against the oracle (whose l = 4 primitives are pinned to mpmath center derivatives in
tests/test_oracle_eri.py), through the C ABI.  Bars as for l <= 3 (north_star): |dERI| <= 1e-10,
max|dJ|, max|dK| <= 1e-8, |dE_SCF| <= 1e-7 Ha; reduced tier |dERI| <= 4e-3 Q_ab Q_cd (R20)."""
import itertools

import numpy as np
import pytest

import oracle
import mako_inputs as mi

pytestmark = pytest.mark.gpu


def _basis_l4(seed, nprim_choices=(1, 2)):
    """Shells of every l <= 4 on 3 centres, random exponents (log-U[0.1,10])."""
    rng = np.random.default_rng(seed)
    centers = rng.uniform(-2, 2, size=(3, 3))
    ls, nps, xyz, ex, cf, at = [], [], [], [], [], []
    for a in range(3):
        for l in range(5):
            k = int(rng.choice(nprim_choices))
            ls.append(l); nps.append(k); xyz.append(centers[a]); at.append(a)
            ex += list(np.exp(rng.uniform(np.log(0.1), np.log(10.0), k)))
            cf += list(rng.uniform(0.2, 1.0, k))
    sh = mi.Shells(np.array(at, np.int32), np.array(ls, np.int32), np.array(nps, np.int32), np.array(xyz),
                   np.array(ex), np.array(cf))
    return sh, np.array([1, 1, 1], np.int32), centers


def _bucket(la, lb):
    la, lb = max(la, lb), min(la, lb)
    return la * (la + 1) // 2 + lb


def _cls(ls):
    X, Y = _bucket(ls[0], ls[1]), _bucket(ls[2], ls[3])
    X, Y = max(X, Y), min(X, Y)
    return X * (X + 1) // 2 + Y


def test_eri_batch_all_120_classes_fp64_and_reduced():
    from paper_conf_sc_han0jlacz0025_b200 import Basis, class_reduced, eri_batch
    sh, Z, centers = _basis_l4(11)
    B = Basis(Z, centers, sh)
    rng = np.random.default_rng(311)
    by_l = {l: [i for i in range(sh.nshell) if sh.l[i] == l] for l in range(5)}
    # every (la lb | lc ld) pattern with l <= 4 in every order: all 120 canonical classes
    quartets = [[int(rng.choice(by_l[x])) for x in ls] for ls in itertools.product(range(5), repeat=4)
                if max(ls) == 4]
    ref = [oracle.eri_quartet(sh, *q) for q in quartets]
    blocks = eri_batch(B, quartets)
    worst = 0.0
    for q, blk, r in zip(quartets, blocks, ref):
        err = np.abs(blk.cpu().numpy() - r).max()
        worst = max(worst, err)
        assert err <= 1e-10, (q, err)
    print("g classes: max |dERI| %.3e over %d quartets" % (worst, len(quartets)))
    red = class_reduced()
    blocks = eri_batch(B, quartets, reduced=True)
    Qc = {}

    def Q(a, b):
        if (a, b) not in Qc:
            Qc[(a, b)] = np.sqrt(np.abs(oracle.eri_quartet(sh, a, b, a, b)).max())
        return Qc[(a, b)]

    wr = 0.0
    for q, blk, r in zip(quartets, blocks, ref):
        err = np.abs(blk.cpu().numpy() - r).max()
        if red[_cls([sh.l[s] for s in q])]:
            b = Q(q[0], q[1]) * Q(q[2], q[3])
            wr = max(wr, err / b)
            assert err <= 4e-3 * b, (q, err, b)
        else:
            assert err <= 1e-10, (q, err)
    print("g classes, reduced tier: max |dERI|/(Q_ab Q_cd) %.3e" % wr)


def _setup(cfg, tau):
    from paper_conf_sc_han0jlacz0025_b200 import Basis, Pairs
    m, b = mi.config_molecule(cfg)
    sh = mi.shells_for(m, b)
    B = Basis(m.Z, m.xyz_bohr, sh)
    return m, sh, B, Pairs(B, tau)


def _gpu_jk(P, D, **kw):
    import torch
    from paper_conf_sc_han0jlacz0025_b200 import build_jk
    J, K = build_jk(P, torch.tensor(D, device="cuda"), **kw)
    torch.cuda.synchronize()
    return J.cpu().numpy(), K.cpu().numpy()


def test_h2o_ccpvqz_jk_and_scf_vs_oracle():
    m, sh, B, P = _setup("h2o-ccpvqz", 0.0)
    assert max(sh.l) == 4
    D = mi.synthetic_density(sh.nbf(), m.nelec // 2, seed=0)
    J0, K0 = oracle.jk(sh, D, 0.0)
    J, K = _gpu_jk(P, D)
    dj, dk = np.abs(J - J0).max(), np.abs(K - K0).max()
    print("h2o cc-pVQZ-shaped max|dJ| %.3e max|dK| %.3e" % (dj, dk))
    assert dj <= 1e-8 and dk <= 1e-8
    S, T, V = oracle.one_electron(sh, m)
    en = oracle.nuclear_repulsion(m)
    r_gpu = oracle.rhf(S, T, V, en, m.nelec // 2, lambda X: _gpu_jk(P, X))
    r_orc = oracle.rhf(S, T, V, en, m.nelec // 2, lambda X: oracle.jk(sh, X, 0.0))
    print("h2o cc-pVQZ-shaped RHF", r_gpu.energy, r_orc.energy)
    assert r_gpu.converged and abs(r_gpu.energy - r_orc.energy) <= 1e-7


def test_benzene_ccpvqz_sampled_blocks():
    """510 basis functions with g on every carbon: exact J/K blocks of sampled shell pairs (g-g, g-s,
    random) vs the oracle's definition-level blocks with the same Schwarz rule."""
    tau = 1e-12
    m, sh, B, P = _setup("benzene-ccpvqz", tau)
    D = mi.synthetic_density(sh.nbf(), m.nelec // 2, seed=0)
    J, K = _gpu_jk(P, D)
    assert np.array_equal(J, J.T) and np.array_equal(K, K.T)
    rng = np.random.default_rng(3)
    g = [i for i in range(sh.nshell) if sh.l[i] == 4]
    pairs = [(g[0], g[0]), (g[1], g[2]), (g[3], 0)] + [(int(rng.integers(sh.nshell)), int(rng.integers(sh.nshell)))]
    Jb, Kb = oracle.jk_blocks(sh, D, pairs, tau=tau, Q=oracle.schwarz(sh))
    off = B.ao_offsets
    for (x, y), jb, kb in zip(pairs, Jb, Kb):
        gj = J[off[x]:off[x + 1], off[y]:off[y + 1]]
        gk = K[off[x]:off[x + 1], off[y]:off[y + 1]]
        print("benzene cc-pVQZ block", x, y, np.abs(gj - jb).max(), np.abs(gk - kb).max())
        assert np.abs(gj - jb).max() <= 1e-8 and np.abs(gk - kb).max() <= 1e-8
