"""Pins for the oracle Boys function F_m(T) (Eq. 4 seed [0]^(m) ~ F_m).

Pinned against: F_m(0) = 1/(2m+1) (closed form), F_0 = 1/2 sqrt(pi/T) erf(sqrt T) (closed form),
and mpmath's incomplete gamma at 30 digits: F_m(T) = gamma(m+1/2, 0..T) / (2 T^(m+1/2)).
"""
import mpmath as mp
import numpy as np
import pytest

import oracle

mp.mp.dps = 30


def f_ref(m, T):
    if T == 0:
        return mp.mpf(1) / (2 * m + 1)
    T = mp.mpf(T)
    return mp.gammainc(m + mp.mpf(1) / 2, 0, T) / (2 * T ** (m + mp.mpf(1) / 2))


@pytest.mark.parametrize("T", [0.0, 1e-12, 1e-6, 0.01, 0.3, 1.0, 2.5, 7.3, 12.0, 19.9, 29.999, 30.0, 30.001,
                               35.0, 50.0, 117.0, 800.0, 1e5])
def test_boys_vs_mpmath(T):
    F = oracle.boys(16, T)
    for m in range(17):
        ref = float(f_ref(m, T))
        assert abs(F[m] - ref) <= 2e-15 * abs(ref) + 1e-300, (m, T, F[m], ref)


def test_boys_zero_closed_form():
    F = oracle.boys(20, 0.0)
    assert np.allclose(F, [1.0 / (2 * m + 1) for m in range(21)], rtol=0, atol=1e-16)


def test_boys_f0_erf_closed_form():
    for T in [0.5, 3.0, 25.0, 31.0, 60.0]:
        ref = 0.5 * mp.sqrt(mp.pi / T) * mp.erf(mp.sqrt(T))
        assert abs(oracle.boys(0, T)[0] - float(ref)) < 1e-16 * 2


def test_boys_downward_identity():
    # F_m = (2T F_{m+1} + e^{-T}) / (2m+1) holds for the exact function
    for T in [0.2, 4.0, 22.0, 45.0]:
        F = oracle.boys(12, T)
        for m in range(12):
            assert abs(F[m] - (2 * T * F[m + 1] + np.exp(-T)) / (2 * m + 1)) < 4e-16 * F[m]
