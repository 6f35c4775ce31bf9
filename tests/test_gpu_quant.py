"""GPU parity of the stage-aware reduced-precision tier (QuantMako PAPER.md §3.2
L286-L302) against the oracle, through the C ABI (mako_eri_batch_ex, mako_build_jk_mixed).

Bars:
  - reduced-tier ERIs: |d(ab|cd)| <= 4e-3 * Q_ab Q_cd per element (the per-stage budget of
    eri_quant.cuh, (2^-9 + (K1+K2) 2^-24) * sum|E~ R E~|, with sum|E~ R E~| measured at <= 4 Q_ab Q_cd
    on these inputs: DESIGN.md reading R20); classes without a reduced kernel stay at the FP64 bar
    1e-10;
  - RMSE reported per run (the quantity of PAPER.md Table 2);
  - mixed J/K: the FP64 tier is exact (thresh_fp64 -> 0 reproduces mako_build_jk); every reduced
    quartet moves a J/K element by at most 2 * 4e-3 * thresh_fp64-scale (bound checked below);
  - SCF: |E_mixed - E_FP64| <= 1e-5 Ha (north_star's reduced-precision bar).
"""
import itertools

import numpy as np
import pytest

import oracle
import mako_inputs as mi

pytestmark = pytest.mark.gpu

NAMES = ["ss", "ps", "pp", "ds", "dp", "dd", "fs", "fp", "fd", "ff", "gs", "gp", "gd", "gf", "gg"]


def _bucket(la, lb):
    la, lb = max(la, lb), min(la, lb)
    return la * (la + 1) // 2 + lb


def _cls(ls):
    X, Y = _bucket(ls[0], ls[1]), _bucket(ls[2], ls[3])
    X, Y = max(X, Y), min(X, Y)
    return X * (X + 1) // 2 + Y


def _mixed_basis(seed, nprim_choices=(1, 3)):
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


@pytest.mark.parametrize("seed", [0, 1])
def test_reduced_eri_all_55_classes(seed):
    from paper_conf_sc_han0jlacz0025_b200 import Basis, class_reduced, eri_batch
    sh, Z, centers = _mixed_basis(seed)
    B = Basis(Z, centers, sh)
    red = class_reduced()
    assert red.sum() >= 20
    rng = np.random.default_rng(200 + seed)
    by_l = {l: [i for i in range(sh.nshell) if sh.l[i] == l] for l in range(4)}
    quartets = [[int(rng.choice(by_l[x])) for x in ls] for ls in itertools.product(range(4), repeat=4)]
    blocks = eri_batch(B, quartets, reduced=True)
    Qc = {}

    def Q(a, b):  # oracle Schwarz factor of a shell pair
        if (a, b) not in Qc:
            d = oracle.eri_quartet(sh, a, b, a, b)
            Qc[(a, b)] = np.sqrt(np.abs(d).max())
        return Qc[(a, b)]

    se, n, worst = 0.0, 0, 0.0
    for q, blk in zip(quartets, blocks):
        ref = oracle.eri_quartet(sh, *q)
        err = np.abs(blk.cpu().numpy() - ref).max()
        if red[_cls([sh.l[s] for s in q])]:
            bound = Q(q[0], q[1]) * Q(q[2], q[3])
            worst = max(worst, err / bound)
            se += float(((blk.cpu().numpy() - ref) ** 2).sum()); n += ref.size
            assert err <= 4e-3 * bound, (q, err, bound)
        else:
            assert err <= 1e-10, (q, err)
    print("reduced tier: RMSE %.3e over %d ERIs, max |dERI|/(Q_ab Q_cd) %.3e" % (np.sqrt(se / n), n, worst))


def _setup(cfg, tau):
    from paper_conf_sc_han0jlacz0025_b200 import Basis, Pairs
    m, b = mi.config_molecule(cfg)
    sh = mi.shells_for(m, b)
    B = Basis(m.Z, m.xyz_bohr, sh)
    return m, sh, B, Pairs(B, tau)


def _jk(P, D, **kw):
    import torch
    from paper_conf_sc_han0jlacz0025_b200 import build_jk
    J, K = build_jk(P, torch.tensor(D, device="cuda"), **kw)
    torch.cuda.synchronize()
    return J.cpu().numpy(), K.cpu().numpy()


def _reduced_bound(sh, B, Q, D, tau, t64, cap=4e-3):
    """Per-element error bound of mako_build_jk_mixed vs the FP64 result (readings R20/R21):
    a quartet (ab|cd) runs the reduced tier iff its class has a reduced kernel and tau <= Q_ab Q_cd < T,
    T = 10^floor(log10(thresh_fp64 / max|D|)); each of its ERIs is then off by at most cap * Q_ab Q_cd
    (the ERI-level bar of test_reduced_eri_batch_error_budget, measured <= 8.6e-4).  Summed over the
    quartets contributing to each element, with |D| weights:
        |dJ_mn| <= cap sum_{cd reduced} Q_ab Q_cd sum_{l in c, s in d} |D_ls|            (m in a, n in b)
        |dK_mk| <= cap sum_{b,d: (ab|cd) reduced} Q_ab Q_cd sum_{n in b, s in d} |D_ns|   (m in a, k in c)
    over ordered shell tuples (every permutation of a canonical quartet contributes once)."""
    from paper_conf_sc_han0jlacz0025_b200.mako import class_reduced
    red = class_reduced()
    ns = sh.nshell
    off = B.ao_offsets
    l = np.asarray(sh.l)
    buck = lambda la, lb: max(la, lb) * (max(la, lb) + 1) // 2 + min(la, lb)
    bk = np.array([[buck(l[a], l[b]) for b in range(ns)] for a in range(ns)])
    X = np.maximum(bk[:, :, None, None], bk[None, None, :, :])
    Y = np.minimum(bk[:, :, None, None], bk[None, None, :, :])
    cls = X * (X + 1) // 2 + Y
    dmax = np.abs(D).max()
    T = 10.0 ** np.floor(np.log10(t64 / dmax))
    QQ = Q[:, :, None, None] * Q[None, None, :, :]
    R = red[cls] & (QQ >= tau) & (QQ < T)
    S1 = np.array([[np.abs(D[off[a]:off[a + 1], off[b]:off[b + 1]]).sum() for b in range(ns)] for a in range(ns)])
    W = np.where(R, QQ, 0.0)
    bj = cap * np.einsum("abcd,cd->ab", W, S1)
    bk_ = cap * np.einsum("abcd,bd->ac", W, S1)
    exp = lambda m: np.repeat(np.repeat(m, np.diff(off), axis=0), np.diff(off), axis=1)
    return exp(bj), exp(bk_), int(R.sum())


def test_mixed_jk_tiers_vs_oracle():
    m, sh, B, P = _setup("benzene-def2svp", 1e-12)
    D = mi.synthetic_density(sh.nbf(), m.nelec // 2, seed=7)
    Q = oracle.schwarz(sh)
    J0, K0 = oracle.jk(sh, D, 1e-12, Q=Q)
    # no reduced quartets: the FP64 tier reproduces the oracle at the FP64 bar
    J, K = _jk(P, D, thresh_fp64=1e-30)
    assert np.abs(J - J0).max() <= 1e-8 and np.abs(K - K0).max() <= 1e-8
    prev = 0.0
    for t64 in (1e-8, 1e-6, 1e-4, 1e30):
        J, K = _jk(P, D, thresh_fp64=t64)
        dj, dk = np.abs(J - J0), np.abs(K - K0)
        bj, bk, nred = _reduced_bound(sh, B, Q, D, 1e-12, t64)
        print("thresh_fp64 %.0e: %d reduced ordered quartets, max|dJ| %.3e (max bound %.3e), max|dK| %.3e "
              "(max bound %.3e), worst dJ/bound %.3f dK/bound %.3f" % (
                  t64, nred, dj.max(), bj.max(), dk.max(), bk.max(), (dj / (bj + 1e-10)).max(),
                  (dk / (bk + 1e-10)).max()))
        assert np.array_equal(J, J.T) and np.array_equal(K, K.T)
        # per element: the reduced-tier bound plus the FP64 bar for the FP64 quartets
        assert (dj <= bj + 1e-10).all() and (dk <= bk + 1e-10).all()
        assert max(dj.max(), dk.max()) >= prev * 0.1  # more reduced work -> not dramatically smaller error
        prev = max(dj.max(), dk.max())
    # fully reduced (every quartet of a reduced class): relative error at the TF32 level
    assert np.abs(J - J0).max() <= 1e-3 * np.abs(J0).max()


def _scf(mol, sh, jk_fn):
    S, T, V = oracle.one_electron(sh, mol)
    return oracle.rhf(S, T, V, oracle.nuclear_repulsion(mol), mol.nelec // 2, jk_fn)


def test_mixed_scf_energy_within_1e5():
    from paper_conf_sc_han0jlacz0025_b200 import IncrementalJK
    m, sh, B, P = _setup("benzene-def2svp", 1e-12)
    r64 = _scf(m, sh, lambda D: _jk(P, D))
    res = {}
    for t64 in (1e-6, 1e-4, 1e30):
        r = _scf(m, sh, lambda D: _jk(P, D, thresh_fp64=t64))
        res[t64] = r.energy - r64.energy
        assert r.converged
    print("benzene RHF E_fp64 %.10f, E_mixed - E_fp64:" % r64.energy, res)
    assert abs(res[1e-6]) <= 1e-5 and abs(res[1e-4]) <= 1e-5
    # convergence-aware precision schedule: reduced tier early, FP64 near convergence
    inc = IncrementalJK(P, precision_scale=1e-3)
    r = _scf(m, sh, inc)
    print("incremental mixed", r.energy - r64.energy, [(h["full"], h["thresh_fp64"]) for h in inc.history])
    assert r.converged and abs(r.energy - r64.energy) <= 1e-7
    assert any(h["thresh_fp64"] is not None for h in inc.history)
