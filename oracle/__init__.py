"""CPU ORACLE -- test infrastructure only.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs
may import this package.  The product package (paper_conf_sc_han0jlacz0025_b200) never
imports it.  See oracle/mako_oracle.c for the method citations.
"""
from .oracle import (build_oracle, boys, sph_coeffs, eri_quartet, eri_full, schwarz, jk, jk_qsample, jk_dw, jk_blocks,
                     one_electron, nuclear_repulsion, num_threads)
from .scf import rhf, RHFResult

__all__ = ["build_oracle", "boys", "sph_coeffs", "eri_quartet", "eri_full", "schwarz", "jk", "jk_qsample", "jk_dw", "jk_blocks",
           "one_electron", "nuclear_repulsion", "num_threads", "rhf", "RHFResult"]
