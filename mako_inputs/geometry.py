"""Molecular geometries for the BASELINE.json configurations (all seeded / deterministic).

Recipes:
  C1 H2O STO-3G      R(OH)=0.9572 A, angle 104.52 deg  (plus Crawford's geometry for the published pin)
  C2 benzene         D6h, r(CC)=1.397 A, r(CH)=1.084 A
  C3 (Gly)10         C20H32N10O11, idealised planar extended strand, 3.6 A rise per residue
  C4 valinomycin-sized  C54H90N6O18 (168 atoms) random packing in a sphere, 0.087 atoms/A^3, dmin 1.0 A, seed 0
  C5 ubiquitin-sized    C378H629N105O118S1 (1231 atoms), same packing, seed 0
"""
import math
from dataclasses import dataclass, field

import numpy as np

ANGSTROM_TO_BOHR = 1.0 / 0.52917721092
Z_OF = {"H": 1, "C": 6, "N": 7, "O": 8, "S": 16}


@dataclass
class Molecule:
    symbols: list
    xyz_bohr: np.ndarray          # [natm, 3]
    name: str = ""

    @property
    def Z(self):
        return np.array([Z_OF[s] for s in self.symbols], dtype=np.int32)

    @property
    def natm(self):
        return len(self.symbols)

    @property
    def nelec(self):
        return int(self.Z.sum())

    def min_distance_angstrom(self):
        x = self.xyz_bohr / ANGSTROM_TO_BOHR
        d = np.sqrt(((x[:, None, :] - x[None, :, :]) ** 2).sum(-1))
        d[np.diag_indices(len(x))] = np.inf
        return float(d.min())


def _mol(symbols, xyz, unit="bohr", name=""):
    xyz = np.asarray(xyz, dtype=np.float64).reshape(-1, 3)
    if unit == "angstrom":
        xyz = xyz * ANGSTROM_TO_BOHR
    return Molecule(list(symbols), xyz, name)


def h2(R=1.4):
    return _mol(["H", "H"], [[0, 0, 0], [0, 0, R]], name="H2")


def h2o_crawford():
    """Crawford's programming-project H2O geometry (bohr); published STO-3G E = -74.942079928192."""
    return _mol(["O", "H", "H"], [[0.0, -0.143225816552, 0.0],
                                  [1.638036840407, 1.136548822547, -0.0],
                                  [-1.638036840407, 1.136548822547, -0.0]], name="H2O-crawford")


def h2o_baseline():
    """R(OH) = 0.9572 A, angle 104.52 deg (BASELINE.json configs[0])."""
    r, th = 0.9572, math.radians(104.52) / 2
    return _mol(["O", "H", "H"], [[0, 0, 0], [0, r * math.sin(th), r * math.cos(th)],
                                  [0, -r * math.sin(th), r * math.cos(th)]], unit="angstrom", name="H2O")


def benzene():
    rcc, rch = 1.397, 1.084
    sym, xyz = [], []
    for k in range(6):
        a = math.pi / 3 * k
        sym.append("C"); xyz.append([rcc * math.cos(a), rcc * math.sin(a), 0.0])
    for k in range(6):
        a = math.pi / 3 * k
        sym.append("H"); xyz.append([(rcc + rch) * math.cos(a), (rcc + rch) * math.sin(a), 0.0])
    return _mol(sym, xyz, unit="angstrom", name="benzene")


def glycine_oligomer(n=10):
    """Idealised extended (phi = psi = 180 deg) planar polyglycine, H-(Gly)n-OH, Angstrom template."""
    sym, xyz = [], []
    rise = 3.6
    for i in range(n):
        x0 = rise * i
        res = [("N", (0.00, 0.00, 0.0)), ("H", (-0.35, 0.95, 0.0)),
               ("C", (1.21, 0.80, 0.0)), ("H", (1.21, 1.45, 0.89)), ("H", (1.21, 1.45, -0.89)),
               ("C", (2.30, -0.30, 0.0)), ("O", (2.30, -1.53, 0.0))]
        for s, (x, y, z) in res:
            sym.append(s); xyz.append([x0 + x, y, z])
    sym.append("H"); xyz.append([-0.45, -0.90, 0.0])                       # N-terminal extra H
    xl = rise * (n - 1)
    sym.append("O"); xyz.append([xl + 3.60, 0.00, 0.0])                    # C-terminal OH
    sym.append("H"); xyz.append([xl + 3.95, 0.92, 0.0])
    return _mol(sym, xyz, unit="angstrom", name=f"(Gly){n}")


def _formula_symbols(formula):
    sym = []
    for el, cnt in formula:
        sym += [el] * cnt
    return sym


def random_packed(formula, density=0.087, dmin=1.0, seed=0, name=""):
    """Uniform random packing in a sphere (atoms/A^3 = density), min pair distance dmin (A), seeded."""
    sym = _formula_symbols(formula)
    n = len(sym)
    r = (3.0 * n / (4.0 * math.pi * density)) ** (1.0 / 3.0)
    rng = np.random.default_rng(seed)
    pts = np.zeros((0, 3))
    cell = dmin
    grid = {}
    while len(pts) < n:
        p = rng.uniform(-r, r, size=3)
        if p @ p > r * r:
            continue
        key = tuple((p // cell).astype(int))
        ok = True
        for dx in (-1, 0, 1):
            for dy in (-1, 0, 1):
                for dz in (-1, 0, 1):
                    for j in grid.get((key[0] + dx, key[1] + dy, key[2] + dz), ()):
                        if np.sum((pts[j] - p) ** 2) < dmin * dmin:
                            ok = False
        if ok:
            grid.setdefault(key, []).append(len(pts))
            pts = np.vstack([pts, p])
    # deterministic element placement: shuffle symbols with the same seed
    perm = rng.permutation(n)
    sym = [sym[i] for i in perm]
    return _mol(sym, pts, unit="angstrom", name=name)


VALINOMYCIN = [("C", 54), ("H", 90), ("N", 6), ("O", 18)]
UBIQUITIN = [("C", 378), ("H", 629), ("N", 105), ("O", 118), ("S", 1)]

# BASELINE.json configs (index -> (name, molecule factory, basis))
CONFIGS = {
    "h2o-sto3g": (h2o_baseline, "sto-3g"),
    "benzene-def2svp": (benzene, "def2-svp"),
    "gly10-ccpvtz": (lambda: glycine_oligomer(10), "cc-pvtz"),
    # not a BASELINE config: the SCF-timing case of the incremental builder
    "gly10-def2svp": (lambda: glycine_oligomer(10), "def2-svp"),
    # not BASELINE configs: g functions (cc-pVQZ family of PAPER.md:L392)
    "h2o-ccpvqz": (h2o_baseline, "cc-pvqz"),
    "benzene-ccpvqz": (benzene, "cc-pvqz"),
    "valinomycin-def2tzvp": (lambda: random_packed(VALINOMYCIN, name="valinomycin-sized"), "def2-tzvp"),
    "ubiquitin-def2tzvp": (lambda: random_packed(UBIQUITIN, name="ubiquitin-sized"), "def2-tzvp"),
}


def config_molecule(name):
    fac, basis = CONFIGS[name]
    return fac(), basis
