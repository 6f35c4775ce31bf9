"""Seeded synthetic density matrices and random shell data (no method arithmetic)."""
import numpy as np


def synthetic_density(nbf, nocc, seed=0):
    """D = 2 X X^T / n_occ with X ~ N(0,1) [nbf x nocc]: symmetric PSD."""
    rng = np.random.default_rng(seed)
    X = rng.standard_normal((nbf, nocc))
    return 2.0 * X @ X.T / nocc


def random_quartet_pairs(rng, n, nshell):
    return rng.integers(0, nshell, size=(n, 4)).astype(np.int32)
