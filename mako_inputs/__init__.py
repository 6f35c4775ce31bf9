"""Seeded, synthetic inputs shared by the oracle tests and the CUDA-path tests/bench.

This module holds NO arithmetic of the method (no normalisation, no integrals, no
screening): only basis-set *data* (exponents / contraction coefficients as tabulated
or "shaped"), molecular geometries, and seeded random density matrices.  Both the
oracle (oracle/) and the product (paper_conf_sc_han0jlacz0025_b200/) consume the flat
arrays produced by :func:`shells_for` and do their own normalisation.
"""
from .basis_data import BASIS_SETS, basis_label
from .geometry import (Molecule, ANGSTROM_TO_BOHR, h2, h2o_crawford, h2o_baseline, benzene,
                       glycine_oligomer, random_packed, CONFIGS, config_molecule)
from .shells import Shells, shells_for
from .density import synthetic_density, random_quartet_pairs

__all__ = ["BASIS_SETS", "basis_label", "Molecule", "ANGSTROM_TO_BOHR", "h2", "h2o_crawford", "h2o_baseline",
           "benzene", "glycine_oligomer", "random_packed", "CONFIGS", "config_molecule", "Shells", "shells_for",
           "synthetic_density", "random_quartet_pairs"]
