"""Flatten (molecule, basis name) into the plain shell arrays both sides consume."""
from dataclasses import dataclass

import numpy as np

from .basis_data import BASIS_SETS


@dataclass
class Shells:
    atom: np.ndarray     # int32 [nshell]
    l: np.ndarray        # int32 [nshell]
    nprim: np.ndarray    # int32 [nshell]
    xyz: np.ndarray      # float64 [nshell, 3] bohr (copy of the atom position)
    exps: np.ndarray     # float64 [sum nprim]
    coefs: np.ndarray    # float64 [sum nprim]  (for normalised primitives, as tabulated)

    @property
    def nshell(self):
        return len(self.l)

    def nbf(self, pure=True):
        return int(sum((2 * l + 1) if pure else (l + 1) * (l + 2) // 2 for l in self.l))

    def subset(self, idx):
        idx = np.asarray(idx)
        poff = np.concatenate([[0], np.cumsum(self.nprim)])
        ex = np.concatenate([self.exps[poff[i]:poff[i + 1]] for i in idx])
        cf = np.concatenate([self.coefs[poff[i]:poff[i + 1]] for i in idx])
        return Shells(self.atom[idx].copy(), self.l[idx].copy(), self.nprim[idx].copy(), self.xyz[idx].copy(),
                      ex, cf)


def shells_for(mol, basis):
    data = BASIS_SETS[basis] if isinstance(basis, str) else basis
    atom, ls, npr, xyz, ex, cf = [], [], [], [], [], []
    for ia, s in enumerate(mol.symbols):
        for (l, e, c) in data[s]:
            atom.append(ia); ls.append(l); npr.append(len(e)); xyz.append(mol.xyz_bohr[ia])
            ex += list(e); cf += list(c)
    return Shells(np.array(atom, np.int32), np.array(ls, np.int32), np.array(npr, np.int32),
                  np.array(xyz, np.float64).reshape(-1, 3), np.array(ex, np.float64), np.array(cf, np.float64))
