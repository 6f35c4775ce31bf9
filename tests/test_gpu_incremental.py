"""GPU parity of density-weighted screening (mako_build_jk_ex, MAKO_JK_DENSITY_SCREEN) against the
oracle's rule (orc_jk_dw), and of the incremental SCF against the
plain SCF.  Bars: max|dJ|, max|dK| <= 1e-8; |dE_SCF| <= 1e-7 Ha (north_star)."""
import json
import os

import numpy as np
import pytest

import oracle
import mako_inputs as mi

pytestmark = pytest.mark.gpu


def _setup(cfg, tau):
    from paper_conf_sc_han0jlacz0025_b200 import Basis, Pairs
    m, b = mi.config_molecule(cfg)
    sh = mi.shells_for(m, b)
    B = Basis(m.Z, m.xyz_bohr, sh)
    return m, sh, B, Pairs(B, tau)


def _gpu(P, D, thresh, dw):
    import torch
    from paper_conf_sc_han0jlacz0025_b200 import build_jk
    J, K = build_jk(P, torch.tensor(D, device="cuda"), thresh=thresh, density_screen=dw)
    torch.cuda.synchronize()
    return J.cpu().numpy(), K.cpu().numpy()


def test_density_screen_vs_oracle_rule():
    m, sh, B, P = _setup("benzene-def2svp", 1e-12)
    Q = oracle.schwarz(sh)
    for scale, tau_dw in ((1.0, 1e-9), (1e-3, 1e-9), (1e-6, 1e-10)):
        D = mi.synthetic_density(sh.nbf(), m.nelec // 2, seed=4) * scale
        J0, K0 = oracle.jk_dw(sh, D, 1e-12, tau_dw, Q=Q)
        J, K = _gpu(P, D, tau_dw, True)
        dj, dk = np.abs(J - J0).max(), np.abs(K - K0).max()
        print("density screen", scale, tau_dw, dj, dk)
        assert dj <= 1e-8 and dk <= 1e-8
        assert np.array_equal(J, J.T) and np.array_equal(K, K.T)
    # tau_dw -> 0: identical to the plain build
    D = mi.synthetic_density(sh.nbf(), m.nelec // 2, seed=5)
    J1, K1 = _gpu(P, D, 1e-12, False)
    J2, K2 = _gpu(P, D, 1e-30, True)
    assert np.abs(J1 - J2).max() <= 1e-12 * np.abs(J1).max() and np.abs(K1 - K2).max() <= 1e-12 * np.abs(K1).max()


def test_accumulate_and_density_delta():
    """MAKO_JK_ACCUMULATE + mako_density_delta (the incremental update inside the C ABI): J[D1] +
    J[D2 - D1] equals J[D2] (J, K linear in D); max|dD| is exact; a NaN in D is rejected."""
    import torch
    from paper_conf_sc_han0jlacz0025_b200 import MakoError, build_jk, density_delta
    m, sh, B, P = _setup("benzene-def2svp", 1e-12)
    n = sh.nbf()
    D1 = torch.tensor(mi.synthetic_density(n, m.nelec // 2, seed=8), device="cuda")
    D2 = torch.tensor(mi.synthetic_density(n, m.nelec // 2, seed=9), device="cuda")
    J, K = build_jk(P, D1)
    dD, dmax = density_delta(P, D2, D1)
    torch.cuda.synchronize()
    ref = (D2 - D1)
    assert torch.equal(dD, ref) and dmax == float(ref.abs().max())
    build_jk(P, dD, J=J, K=K, accumulate=True)
    J2, K2 = build_jk(P, D2)
    torch.cuda.synchronize()
    assert float((J - J2).abs().max()) <= 1e-12 * float(J2.abs().max())
    assert float((K - K2).abs().max()) <= 1e-12 * float(K2.abs().max())
    # accumulate with density screening and with the mixed build
    J3, K3 = build_jk(P, D1, density_screen=True, thresh=1e-13)
    build_jk(P, dD, J=J3, K=K3, density_screen=True, thresh=1e-13, accumulate=True)
    torch.cuda.synchronize()
    assert float((J3 - J2).abs().max()) <= 1e-8 and float((K3 - K2).abs().max()) <= 1e-8
    # non-finite densities fail loudly (NaN survives the block maxima)
    Dn = D1.clone()
    Dn[3, 5] = float("nan")
    with pytest.raises(MakoError):
        density_delta(P, Dn, D1)
    with pytest.raises(MakoError):
        build_jk(P, Dn, density_screen=True)


def _scf(mol, sh, jk_fn):
    S, T, V = oracle.one_electron(sh, mol)
    return oracle.rhf(S, T, V, oracle.nuclear_repulsion(mol), mol.nelec // 2, jk_fn)


def test_incremental_scf_energies():
    from paper_conf_sc_han0jlacz0025_b200 import Basis, IncrementalJK, Pairs
    # published pin (tests/golden/h2o_sto3g.txt) through the incremental, density-screened GPU J/K
    mol = mi.h2o_crawford()
    sh = mi.shells_for(mol, "sto-3g")
    P = Pairs(Basis(mol.Z, mol.xyz_bohr, sh), 1e-12)
    inc = IncrementalJK(P)
    r = _scf(mol, sh, inc)
    assert r.converged and abs(r.energy - (-74.942079928192)) <= 1e-8
    assert any(not h["full"] for h in inc.history)
    # benzene: incremental vs plain GPU SCF and vs the oracle SCF
    m, sh, B, P = _setup("benzene-def2svp", 1e-12)
    inc = IncrementalJK(P)
    r_inc = _scf(m, sh, inc)
    r_gpu = _scf(m, sh, lambda D: _gpu(P, D, 1e-12, False))
    r_orc = _scf(m, sh, lambda D: oracle.jk(sh, D, 1e-12))
    print("benzene", r_inc.energy, r_gpu.energy, r_orc.energy, [(h["full"], h["tau"]) for h in inc.history])
    assert r_inc.converged and abs(r_inc.energy - r_gpu.energy) <= 1e-7
    assert abs(r_inc.energy - r_orc.energy) <= 1e-7
    assert r_inc.iterations <= r_gpu.iterations + 4  # the schedule does not derail the SCF
    hist = inc.history
    assert hist[0]["full"] and not all(h["full"] for h in hist)
    assert hist[-1]["tau"] == pytest.approx(1e-12)  # tightened to tau_final near convergence


@pytest.mark.skipif(not os.environ.get("MAKO_SCF_TIMING"), reason="timing run (MAKO_SCF_TIMING=1)")
@pytest.mark.parametrize("cfg", ["benzene-def2svp", "gly10-def2svp"])
def test_scf_timing_line(cfg):
    """Measurement line of a full RHF on the GPU J/K (BASELINE configs[1] benzene def2-SVP "full SCF";
    gly10-def2svp = the polyglycine family of PAPER.md Fig. 8 for the row-f2 comparison), written to
    gpurun_out/scf_<cfg>.json in bench.py's JSON format.  Two SCF runs with the same driver:
      plain        mako_build_jk on D_n every iteration (the value / s_per_iter of the line);
      incremental  IncrementalJK: Delta D builds with density-weighted screening, accumulated in the
                   library, convergence-aware threshold (row f2).
    s/iter = mean device time of the J/K build per SCF iteration excluding the first.
    The oracle RHF (same driver, oracle J/K) gives dE and the cpu_baseline (benzene only: the oracle
    J/K of (Gly)10 takes minutes per iteration).  H, S and the SCF driver are test support (oracle/)."""
    import time
    import torch
    import bench
    from paper_conf_sc_han0jlacz0025_b200 import IncrementalJK, build_jk
    from paper_conf_sc_han0jlacz0025_b200.mako import FAMILY_KERNELS, class_family
    m, sh, B, P = _setup(cfg, 1e-12)
    n = sh.nbf()
    S, T, V = oracle.one_electron(sh, m)
    enuc = oracle.nuclear_repulsion(m)
    nocc = m.nelec // 2
    flops = P.flops()["gemm_flops"]
    cls_flops, _ = P.class_flops()
    Dd = torch.empty((n, n), dtype=torch.float64, device="cuda")
    J, K = torch.empty_like(Dd), torch.empty_like(Dd)
    ms = []
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)

    def plain(D):
        Dd.copy_(torch.from_numpy(D))
        ev0.record()
        build_jk(P, Dd, J=J, K=K)
        ev1.record()
        torch.cuda.synchronize()
        ms.append(ev0.elapsed_time(ev1))
        return J.cpu().numpy(), K.cpu().numpy()

    plain(np.zeros((n, n)))  # warm-up (plan, first launches)
    ms.clear()
    clocks = bench.ClockSampler(0)
    clocks.start()
    P.profile(True)
    t0 = time.perf_counter()
    r_plain = oracle.rhf(S, T, V, enuc, nocc, plain, e_tol=1e-10, d_tol=1e-8)
    t1 = time.perf_counter()
    cls_ms, cls_n = P.profile_read()
    P.profile(False)
    inc = IncrementalJK(P)
    r_inc = oracle.rhf(S, T, V, enuc, nocc, inc, e_tol=1e-10, d_tol=1e-8)
    t2 = time.perf_counter()
    clk = clocks.stop()
    inc_ms = [h["ms"] for h in inc.history]
    plain_s = float(np.mean(ms[1:])) * 1e-3
    inc_s = float(np.mean(inc_ms[1:])) * 1e-3
    pk = bench.peaks()
    c = int(np.argmax(cls_ms))
    ach = cls_flops[c] / (cls_ms[c] / max(cls_n[c], 1) * 1e-3) / 1e12
    X = int((np.sqrt(8 * c + 1) - 1) // 2)
    Y = c - X * (X + 1) // 2
    nm = ["ss", "ps", "pp", "ds", "dp", "dd", "fs", "fp", "fd", "ff", "gs", "gp", "gd", "gf", "gg"]
    out = {"metric": bench.METRIC, "value": flops / plain_s / 1e12, "unit": bench.UNIT, "n_gpus": 1,
           "steps": len(ms), "warmup": 1, "ms_per_step": plain_s * 1e3, "higher_is_better": True,
           "vs_baseline": None, "dtype": "f64", "data": "synthetic",
           "config": {"workload": cfg + "-rhf", "basis": mi.basis_label(mi.config_molecule(cfg)[1]), "nbf": n,
                      "shells": sh.nshell, "tau": 1e-12, "gemm_flops_per_build": flops},
           "s_per_iter": plain_s, "clocks": clk,
           "roofline": {"bound": "tensor", "achieved": ach, "peak": pk["dmma_m16n8k4_tflops"], "unit": "TFLOP/s",
                        "frac": ach / pk["dmma_m16n8k4_tflops"], "traffic": None,
                        "kernel": f"{FAMILY_KERNELS[int(class_family()[c])]} class ({nm[X]}|{nm[Y]})",
                        "share_of_step": float(cls_ms[c] / max(cls_ms.sum(), 1e-9))},
           "scf": {"plain": {"energy": r_plain.energy, "iterations": r_plain.iterations,
                             "converged": r_plain.converged, "build_s_per_iter_excl_first": plain_s,
                             "wall_s_per_iter": (t1 - t0) / r_plain.iterations},
                   "incremental": {"energy": r_inc.energy, "iterations": r_inc.iterations,
                                   "converged": r_inc.converged, "build_s_per_iter_excl_first": inc_s,
                                   "wall_s_per_iter": (t2 - t1) / r_inc.iterations,
                                   "full_builds": int(sum(h["full"] for h in inc.history)),
                                   "build_ms": inc_ms, "tau_per_build": [h["tau"] for h in inc.history]},
                   "speedup_incremental": plain_s / inc_s,
                   "dE_incremental_vs_plain": r_inc.energy - r_plain.energy,
                   "support": "H, S, guess, DIIS: oracle/ (test support); J/K: libmako"}}
    if cfg == "benzene-def2svp":
        t3 = time.perf_counter()
        r_orc = oracle.rhf(S, T, V, enuc, nocc, lambda D: oracle.jk(sh, D, 1e-12), e_tol=1e-10, d_tol=1e-8)
        t4 = time.perf_counter()
        out["scf"]["oracle"] = {"energy": r_orc.energy, "iterations": r_orc.iterations,
                                "wall_s_per_iter": (t4 - t3) / r_orc.iterations}
        out["scf"]["dE_plain_vs_oracle"] = r_plain.energy - r_orc.energy
        out["cpu_baseline"] = {"value": flops / ((t4 - t3) / r_orc.iterations) / 1e12, "unit": bench.UNIT,
                               "cores": oracle.num_threads(), "kind": "oracle",
                               "sample": "the full oracle RHF (oracle J/K every iteration), wall per iteration"}
        assert abs(r_plain.energy - r_orc.energy) <= 1e-7
    os.makedirs("gpurun_out", exist_ok=True)
    json.dump(out, open(f"gpurun_out/scf_{cfg}.json", "w"), indent=1)
    print(json.dumps({k: v for k, v in out.items() if k != "scf"}))
    assert r_plain.converged and r_inc.converged
    assert abs(r_inc.energy - r_plain.energy) <= 1e-7
