"""Plain RHF driver (numpy) -- SUPPORT for the E_SCF pins, test infrastructure only.

F = H + J - K/2 with D the total density (reading R9); core-Hamiltonian
guess, symmetric orthogonalisation, DIIS(8).  The J/K builder is a callable so the same
driver (same H, S, guess, DIIS) runs with the oracle's J/K or the GPU library's J/K and
Delta E isolates the J/K error.
"""
from dataclasses import dataclass

import numpy as np


@dataclass
class RHFResult:
    energy: float
    e_elec: float
    e_nuc: float
    D: np.ndarray
    iterations: int
    converged: bool


def rhf(S, T, V, e_nuc, nocc, jk_fn, max_iter=100, e_tol=1e-10, d_tol=1e-8, diis_n=8):
    H = T + V
    s, U = np.linalg.eigh(S)
    X = U @ np.diag(s ** -0.5) @ U.T

    def density(F):
        e, C = np.linalg.eigh(X.T @ F @ X)
        C = X @ C
        return 2.0 * C[:, :nocc] @ C[:, :nocc].T

    D = density(H)
    E_old = 0.0
    focks, errs = [], []
    converged = False
    it = 0
    for it in range(1, max_iter + 1):
        J, K = jk_fn(D)
        F = H + J - 0.5 * K
        E = 0.5 * np.sum(D * (H + F))
        err = X.T @ (F @ D @ S - S @ D @ F) @ X
        rms = np.sqrt(np.mean(err ** 2))
        if abs(E - E_old) < e_tol and rms < d_tol:
            converged = True
            break
        E_old = E
        focks.append(F); errs.append(err)
        if len(focks) > diis_n:
            focks.pop(0); errs.pop(0)
        if len(focks) >= 2:
            n = len(focks)
            Bm = -np.ones((n + 1, n + 1)); Bm[n, n] = 0.0
            for i in range(n):
                for j in range(n):
                    Bm[i, j] = np.sum(errs[i] * errs[j])
            rhs = np.zeros(n + 1); rhs[n] = -1.0
            try:
                c = np.linalg.solve(Bm, rhs)[:n]
                F = sum(ci * Fi for ci, Fi in zip(c, focks))
            except np.linalg.LinAlgError:
                pass
        D = density(F)
    return RHFResult(E + e_nuc, E, e_nuc, D, it, converged)
