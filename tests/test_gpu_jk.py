"""GPU parity of the J/K build (the hot path) against the oracle, through the C ABI.
Bars (BASELINE.json north_star): max|dJ|, max|dK| <= 1e-8; |dE_SCF| <= 1e-7 Ha."""
import numpy as np
import pytest

import oracle
import mako_inputs as mi

pytestmark = pytest.mark.gpu


def _setup(cfg, tau):
    import torch
    from paper_conf_sc_han0jlacz0025_b200 import Basis, Pairs
    m, b = mi.config_molecule(cfg)
    sh = mi.shells_for(m, b)
    B = Basis(m.Z, m.xyz_bohr, sh)
    P = Pairs(B, tau)
    return m, sh, B, P


def _gpu_jk(P, D, thresh=None, shard=0, nshards=1):
    import torch
    from paper_conf_sc_han0jlacz0025_b200 import build_jk
    Dt = torch.tensor(D, device="cuda")
    J, K = build_jk(P, Dt, thresh=thresh, shard=shard, nshards=nshards)
    torch.cuda.synchronize()
    return J.cpu().numpy(), K.cpu().numpy()


def test_h2o_jk_vs_bruteforce():
    m, sh, B, P = _setup("h2o-sto3g", 0.0)
    D = mi.synthetic_density(sh.nbf(), 5, seed=0)
    eri = oracle.eri_full(sh)
    J0 = np.einsum("ijkl,kl->ij", eri, D)
    K0 = np.einsum("ikjl,kl->ij", eri, D)
    J, K = _gpu_jk(P, D)
    assert np.abs(J - J0).max() <= 1e-8 and np.abs(K - K0).max() <= 1e-8
    assert np.abs(J - J0).max() <= 1e-12 * np.abs(J0).max()
    assert np.array_equal(J, J.T) and np.array_equal(K, K.T)


def test_benzene_jk_vs_oracle_tau0():
    m, sh, B, P = _setup("benzene-def2svp", 0.0)
    D = mi.synthetic_density(sh.nbf(), m.nelec // 2, seed=0)
    J0, K0 = oracle.jk(sh, D, 0.0)
    J, K = _gpu_jk(P, D)
    dj, dk = np.abs(J - J0).max(), np.abs(K - K0).max()
    print("benzene max|dJ|", dj, "max|dK|", dk)
    assert dj <= 1e-8 and dk <= 1e-8


def test_benzene_screened_vs_oracle():
    tau = 1e-10
    m, sh, B, P = _setup("benzene-def2svp", tau)
    D = mi.synthetic_density(sh.nbf(), m.nelec // 2, seed=1)
    J0, K0 = oracle.jk(sh, D, tau)
    J, K = _gpu_jk(P, D)
    # same Schwarz rule on both sides; Q's differ only by rounding, so only borderline quartets can differ
    bound = 4 * tau * np.abs(D).max() * 25 * 10
    assert np.abs(J - J0).max() <= max(1e-8, bound) and np.abs(K - K0).max() <= max(1e-8, bound)


def test_shards_sum():
    m, sh, B, P = _setup("benzene-def2svp", 1e-12)
    D = mi.synthetic_density(sh.nbf(), m.nelec // 2, seed=2)
    J1, K1 = _gpu_jk(P, D)
    for n in (2, 3, 8):
        Js = np.zeros_like(J1); Ks = np.zeros_like(K1)
        for s in range(n):
            j, k = _gpu_jk(P, D, shard=s, nshards=n)
            Js += j; Ks += k
        assert np.abs(Js - J1).max() <= 1e-12 * np.abs(J1).max()
        assert np.abs(Ks - K1).max() <= 1e-12 * np.abs(K1).max()


def _rhf_energy(mol, sh, jk_fn):
    S, T, V = oracle.one_electron(sh, mol)
    return oracle.rhf(S, T, V, oracle.nuclear_repulsion(mol), mol.nelec // 2, jk_fn)


def test_scf_energies_h2o_and_benzene():
    for cfg, tau in (("h2o-sto3g", 0.0), ("benzene-def2svp", 0.0)):
        m, sh, B, P = _setup(cfg, tau)
        r_gpu = _rhf_energy(m, sh, lambda D: _gpu_jk(P, D))
        r_orc = _rhf_energy(m, sh, lambda D: oracle.jk(sh, D, 0.0))
        assert r_gpu.converged and r_orc.converged
        print(cfg, r_gpu.energy, r_orc.energy)
        assert abs(r_gpu.energy - r_orc.energy) <= 1e-7
    # published pin through the GPU J/K (tests/golden/h2o_sto3g.txt)
    from paper_conf_sc_han0jlacz0025_b200 import Basis, Pairs
    mol = mi.h2o_crawford()
    sh = mi.shells_for(mol, "sto-3g")
    P = Pairs(Basis(mol.Z, mol.xyz_bohr, sh), 0.0)
    r = _rhf_energy(mol, sh, lambda D: _gpu_jk(P, D))
    assert abs(r.energy - (-74.942079928192)) <= 1e-8


def test_gly10_sampled_blocks():
    """(Gly)10 cc-pVTZ (f functions, all 55 classes): J/K blocks of sampled shell pairs vs the oracle's
    definition-level blocks with the same Schwarz rule."""
    tau = 1e-12
    m, sh, B, P = _setup("gly10-ccpvtz", tau)
    D = mi.synthetic_density(sh.nbf(), m.nelec // 2, seed=0)
    J, K = _gpu_jk(P, D)
    rng = np.random.default_rng(0)
    fshells = [i for i in range(sh.nshell) if sh.l[i] == 3]
    pairs = [(int(rng.integers(sh.nshell)), int(rng.integers(sh.nshell))) for _ in range(3)] + \
            [(fshells[0], fshells[1]), (fshells[2], 0)]
    Q = oracle.schwarz(sh)
    Jb, Kb = oracle.jk_blocks(sh, D, pairs, tau=tau, Q=Q)
    off = B.ao_offsets
    for (x, y), jb, kb in zip(pairs, Jb, Kb):
        gj = J[off[x]:off[x + 1], off[y]:off[y + 1]]
        gk = K[off[x]:off[x + 1], off[y]:off[y + 1]]
        assert np.abs(gj - jb).max() <= 1e-8, (x, y, np.abs(gj - jb).max())
        assert np.abs(gk - kb).max() <= 1e-8, (x, y, np.abs(gk - kb).max())


def test_valinomycin_full_size_sampled_blocks():
    """The bench workload (valinomycin-sized def2-TZVP-shaped, tau = 1e-12, the same build call bench.py
    times): exact J/K blocks of sampled shell pairs vs the oracle's definition-level blocks."""
    tau = 1e-12
    m, sh, B, P = _setup("valinomycin-def2tzvp", tau)
    D = mi.synthetic_density(sh.nbf(), m.nelec // 2, seed=0)
    J, K = _gpu_jk(P, D)
    assert np.array_equal(J, J.T) and np.array_equal(K, K.T)
    rng = np.random.default_rng(7)
    # same-atom shell pairs (significant pairs, non-trivial J and K blocks), s-p and d-f
    atoms = [int(a) for a in rng.choice(np.unique(sh.atom[sh.l == 3]), 2, replace=False)]
    def on(a, l):
        return [i for i in range(sh.nshell) if sh.atom[i] == a and sh.l[i] == l][0]
    pairs = [(on(atoms[0], 0), on(atoms[0], 1)), (on(atoms[1], 2), on(atoms[1], 3))]
    Q = oracle.schwarz(sh)
    # plus 20 random blocks: 10 among the significant shell pairs (Q_ab >= 1e-4, every l combination
    # likely), 10 uniformly random (mostly distant pairs: J large, K tiny)
    sig = np.argwhere(Q >= 1e-4)
    pairs += [tuple(int(v) for v in sig[i]) for i in rng.choice(len(sig), 10, replace=False)]
    pairs += [(int(rng.integers(sh.nshell)), int(rng.integers(sh.nshell))) for _ in range(10)]
    Jb, Kb = oracle.jk_blocks(sh, D, pairs, tau=tau, Q=Q)
    off = B.ao_offsets
    worst = 0.0
    for k, ((x, y), jb, kb) in enumerate(zip(pairs, Jb, Kb)):
        gj = J[off[x]:off[x + 1], off[y]:off[y + 1]]
        gk = K[off[x]:off[x + 1], off[y]:off[y + 1]]
        err = max(np.abs(gj - jb).max(), np.abs(gk - kb).max())
        worst = max(worst, err)
        if k < 2:
            print("valinomycin block", x, y, np.abs(jb).max(), np.abs(kb).max(), err)
            assert np.abs(jb).max() > 1e-3 and np.abs(kb).max() > 1e-6
        assert np.abs(gj - jb).max() <= 1e-8 and np.abs(gk - kb).max() <= 1e-8, (x, y, err)
    print("valinomycin: %d blocks, max |dJ|,|dK| %.2e" % (len(pairs), worst))


def test_flop_accounting_library_equals_reference_arm():
    """bench.py's reference arm counts the workload's algorithmic FLOPs in Python from the oracle's Q;
    the library counts them from its own pair data: both must agree (same screening, same order)."""
    import bench
    m, sh, B, P = _setup("benzene-def2svp", 1e-12)
    lib = P.flops()
    py_flops, py_q = bench.workload_flops(sh, oracle.schwarz(sh), 1e-12)
    assert py_q == lib["quartets"]
    assert abs(py_flops - lib["gemm_flops"]) <= 1e-9 * lib["gemm_flops"]


def _contracted_basis(centers, k, seed):
    """Random centres with one s, p, d and f shell each, k primitives on every shell (the paper's E1
    setting): the d/f x d/f bras are contracted, so the chunk-outer kernels
    (jk_kernel_cb, quartet_block_cbra) run."""
    rng = np.random.default_rng(seed)
    xyz = rng.uniform(-1.5, 1.5, size=(centers, 3))
    at, ls, nps, ex, cf = [], [], [], [], []
    for a in range(centers):
        for l in range(4):
            at.append(a); ls.append(l); nps.append(k)
            ex += list(np.sort(np.exp(rng.uniform(np.log(0.2), np.log(5.0), k)))[::-1])
            cf += list(rng.uniform(0.2, 1.0, k))
    sh = mi.Shells(np.array(at, np.int32), np.array(ls, np.int32), np.array(nps, np.int32), xyz[np.array(at)],
                   np.array(ex), np.array(cf))
    return sh, np.ones(centers, np.int32), xyz


def test_contracted_df_bras_vs_oracle():
    from paper_conf_sc_han0jlacz0025_b200 import Basis, Pairs
    sh, Z, xyz = _contracted_basis(3, 3, seed=11)
    P = Pairs(Basis(Z, xyz, sh), 0.0)
    D = mi.synthetic_density(sh.nbf(), 6, seed=3)
    J0, K0 = oracle.jk(sh, D, 0.0)
    J, K = _gpu_jk(P, D)
    dj, dk = np.abs(J - J0).max(), np.abs(K - K0).max()
    print("contracted d/f max|dJ|", dj, "max|dK|", dk, "|J|", np.abs(J0).max())
    assert dj <= 1e-8 and dk <= 1e-8
