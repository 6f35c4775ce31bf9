"""Pins for the oracle J/K digestion and RHF energies.

J_{mn} = sum_{ls} (mn|ls) D_ls, K_{ml} = sum_{ns} (mn|ls) D_ns (BASELINE.json north_star).
Pinned against: brute-force einsum on the full ERI tensor (the definition), invariants
(symmetry, tr(DJ) >= 0, tr(DK) >= 0, J = K for a single s function), the Schwarz error
bound, and textbook / published energies (tests/golden/*.txt).
"""
import os

import numpy as np
import pytest

import oracle
import mako_inputs as mi

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _golden(name):
    out = {}
    for line in open(os.path.join(GOLD, name)):
        line = line.strip()
        if not line or line.startswith("#"):
            continue
        k, v, t = line.split()
        out[k] = (float(v), float(t))
    return out


def _einsum_jk(eri, D):
    return np.einsum("ijkl,kl->ij", eri, D), np.einsum("ikjl,kl->ij", eri, D)


def test_h2_szabo_ostlund():
    g = _golden("h2_sto3g_szabo.txt")
    m = mi.h2(1.4)
    sh = mi.shells_for(m, "sto-3g")
    S, T, V = oracle.one_electron(sh, m)
    eri = oracle.eri_full(sh)
    assert abs(S[0, 1] - g["S12"][0]) < g["S12"][1]
    assert abs(eri[0, 0, 0, 0] - g["(11|11)"][0]) < g["(11|11)"][1]
    assert abs(eri[0, 0, 1, 1] - g["(11|22)"][0]) < g["(11|22)"][1]
    assert abs(eri[1, 0, 1, 0] - g["(21|21)"][0]) < g["(21|21)"][1]
    assert abs(eri[1, 0, 0, 0] - g["(21|11)"][0]) < g["(21|11)"][1]
    r = oracle.rhf(S, T, V, oracle.nuclear_repulsion(m), 1, lambda D: _einsum_jk(eri, D))
    assert r.converged and abs(r.energy - g["E_total"][0]) < g["E_total"][1]


def test_h2o_published_energies():
    g = _golden("h2o_sto3g.txt")
    m = mi.h2o_crawford()
    assert abs(oracle.nuclear_repulsion(m) - g["crawford_enuc"][0]) < g["crawford_enuc"][1]
    for mol, key in ((mi.h2o_crawford(), "crawford_E"), (mi.h2o_baseline(), "baseline_E")):
        sh = mi.shells_for(mol, "sto-3g")
        S, T, V = oracle.one_electron(sh, mol)
        r = oracle.rhf(S, T, V, oracle.nuclear_repulsion(mol), mol.nelec // 2, lambda D: oracle.jk(sh, D))
        assert r.converged and abs(r.energy - g[key][0]) < g[key][1], (key, r.energy)


def _small_dfbasis():
    mol = mi.Molecule(["O", "H", "H"], mi.h2o_baseline().xyz_bohr)
    sh = mi.shells_for(mol, "def2-tzvp")
    # keep a mixed subset with s, p, d, f (keeps the brute-force tensor small)
    keep = [0, 5, 8, 10, 11, 14, 15]
    return sh.subset(keep)


def test_jk_screened_equals_bruteforce():
    sh = _small_dfbasis()
    N = sh.nbf()
    eri = oracle.eri_full(sh)
    D = mi.synthetic_density(N, 3, seed=1)
    J0, K0 = _einsum_jk(eri, D)
    J, K = oracle.jk(sh, D, tau=0.0)
    assert np.abs(J - J0).max() < 1e-12 * max(1.0, np.abs(J0).max())
    assert np.abs(K - K0).max() < 1e-12 * max(1.0, np.abs(K0).max())
    assert np.allclose(J, J.T, atol=1e-14) and np.allclose(K, K.T, atol=1e-14)
    assert np.sum(D * J) >= 0 and np.sum(D * K) >= 0
    # shards partition the canonical quartets
    Js = sum(oracle.jk(sh, D, 0.0, s, 3)[0] for s in range(3))
    assert np.abs(Js - J).max() < 1e-12 * np.abs(J).max()
    # sampled blocks straight from the definition
    off = np.concatenate([[0], np.cumsum(2 * sh.l + 1)])
    pairs = [(0, 0), (3, 1), (2, 6), (5, 4)]
    Jb, Kb = oracle.jk_blocks(sh, D, pairs)
    for (x, y), jb, kb in zip(pairs, Jb, Kb):
        assert np.allclose(jb, J0[off[x]:off[x + 1], off[y]:off[y + 1]], atol=1e-12)
        assert np.allclose(kb, K0[off[x]:off[x + 1], off[y]:off[y + 1]], atol=1e-12)


def test_single_s_function_J_equals_K():
    sh = mi.Shells(np.zeros(1, np.int32), np.zeros(1, np.int32), np.array([3], np.int32), np.zeros((1, 3)),
                   np.array([3.0, 0.7, 0.2]), np.array([0.3, 0.5, 0.4]))
    D = np.array([[1.7]])
    J, K = oracle.jk(sh, D)
    assert J[0, 0] == K[0, 0] and J[0, 0] > 0


def test_schwarz_screening_error_bound():
    sh = _small_dfbasis()
    N = sh.nbf()
    D = mi.synthetic_density(N, 3, seed=2)
    Q = oracle.schwarz(sh)
    tau = 1e-3
    J0, K0 = oracle.jk(sh, D, 0.0)
    J1, K1 = oracle.jk(sh, D, tau)
    # each dropped canonical quartet moves any element by <= 2 * 2 * tau * max|D| * n_d^2 (8 perms, block size)
    ndrop = sum(1 for a in range(sh.nshell) for b in range(a + 1) for c in range(sh.nshell) for d in range(c + 1)
                if Q[a, b] * Q[c, d] < tau)
    bound = 4 * tau * np.abs(D).max() * 49 * max(ndrop, 1)
    assert ndrop > 0
    assert np.abs(J1 - J0).max() <= bound and np.abs(K1 - K0).max() <= bound


def test_quartet_sample_shards_sum_to_full_build():
    """orc_jk_qsample (the timing sample of bench.py's cpu_baseline / reference arm): the quartet shards
    (canonical quartet index % n == shard) partition the build exactly, for n below and above the number
    of canonical quartets."""
    import mako_inputs as mi
    m, b = mi.config_molecule("benzene-def2svp")
    sh = mi.shells_for(m, b).subset(list(range(14)))
    D = mi.synthetic_density(sh.nbf(), 6, seed=2)
    J0, K0 = oracle.jk(sh, D, 1e-12)
    for n in (5, 13, 20000):
        Js, Ks = np.zeros_like(J0), np.zeros_like(K0)
        for s in range(n if n < 100 else 0):
            j, k = oracle.jk_qsample(sh, D, 1e-12, s, n)
            Js += j
            Ks += k
        if n >= 100:  # sample a few shards only: a non-matching shard is empty, a matching one is one quartet
            nq = sh.nshell * (sh.nshell + 1) // 2
            nq = nq * (nq + 1) // 2
            empty, _ = oracle.jk_qsample(sh, D, 1e-12, nq, nq + 1)
            assert not empty.any()
            continue
        assert np.abs(Js - J0).max() <= 1e-12 * np.abs(J0).max()
        assert np.abs(Ks - K0).max() <= 1e-12 * np.abs(K0).max()
