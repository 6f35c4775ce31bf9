"""Pins of the oracle's density-weighted screening (orc_jk_dw; reading R17):
the rule written out by brute force over the full ERI tensor on a tiny basis, the tau_dw = 0 limit,
and the per-quartet error bound."""
import itertools

import numpy as np

import oracle
import mako_inputs as mi


def _weights(sh, D):
    """Q_ab Q_cd max(|D| over the six shell blocks) for every shell quartet (the rule's left side)."""
    Q = oracle.schwarz(sh)
    off = np.concatenate([[0], np.cumsum(2 * np.asarray(sh.l) + 1)])
    ns = sh.nshell
    dsh = np.array([[np.abs(D[off[x]:off[x + 1], off[y]:off[y + 1]]).max() for y in range(ns)] for x in range(ns)])
    w = np.zeros((ns,) * 4)
    for a, b, c, d in itertools.product(range(ns), repeat=4):
        w[a, b, c, d] = Q[a, b] * Q[c, d] * max(dsh[a, b], dsh[c, d], dsh[a, c], dsh[a, d], dsh[b, c], dsh[b, d])
    return w, off


def _brute_dw(sh, D, tau_dw):
    """J/K from the full ERI tensor, summing only over shell quartets kept by the rule (all 8
    permutations of a kept canonical quartet are kept: the rule is permutation invariant)."""
    eri = oracle.eri_full(sh)
    w, off = _weights(sh, D)
    ns = sh.nshell
    mask = np.zeros_like(eri, dtype=bool)
    for a, b, c, d in itertools.product(range(ns), repeat=4):
        if w[a, b, c, d] >= tau_dw:
            mask[off[a]:off[a + 1], off[b]:off[b + 1], off[c]:off[c + 1], off[d]:off[d + 1]] = True
    e = np.where(mask, eri, 0.0)
    return np.einsum("ijkl,kl->ij", e, D), np.einsum("ikjl,kl->ij", e, D), mask


def test_dw_rule_brute_force_h2o():
    mol = mi.h2o_baseline()
    sh = mi.shells_for(mol, "sto-3g")
    D = mi.synthetic_density(sh.nbf(), 5, seed=3) * 1e-4
    w, _ = _weights(sh, D)
    for tau_dw in np.quantile(w, [0.3, 0.7]):
        J0, K0, mask = _brute_dw(sh, D, tau_dw)
        assert 0 < mask.mean() < 1  # the rule drops some quartets and keeps some
        J, K = oracle.jk_dw(sh, D, 0.0, tau_dw)
        assert np.abs(J - J0).max() <= 1e-13 and np.abs(K - K0).max() <= 1e-13


def test_dw_limits_and_bound_benzene():
    m, b = mi.config_molecule("benzene-def2svp")
    sh = mi.shells_for(m, b)
    D = mi.synthetic_density(sh.nbf(), m.nelec // 2, seed=0)
    J0, K0 = oracle.jk(sh, D, 0.0)
    J1, K1 = oracle.jk_dw(sh, D, 0.0, 0.0)  # tau_dw = 0 keeps everything
    assert np.abs(J1 - J0).max() <= 1e-12 and np.abs(K1 - K0).max() <= 1e-12
    # every dropped quartet moves an element by <= 2 tau_dw; at most (number of canonical quartets)
    # quartets touch one element -> a rigorous (loose) bound, and the dropped part is not empty
    tau_dw = 1e-9
    J2, K2 = oracle.jk_dw(sh, D * 1e-3, 0.0, tau_dw)
    J3, K3 = oracle.jk(sh, D * 1e-3, 0.0)
    npair = sh.nshell * (sh.nshell + 1) // 2
    bound = 2 * tau_dw * npair * (npair + 1) / 2
    err = max(np.abs(J2 - J3).max(), np.abs(K2 - K3).max())
    assert 0 < err <= bound
