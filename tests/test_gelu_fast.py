"""Pin the erf approximation the bf16 GEMM epilogue uses (common.cuh gelu_erf_fast):
Abramowitz & Stegun 7.1.26, |erf error| <= 1.5e-7, restated here in fp64 and
checked against scipy's erf; GELU = max(z,0) - 0.5|z| erfc(|z|/sqrt2) identity."""
import numpy as np
from scipy.special import erf

P, A = 0.3275911, (0.254829592, -0.284496736, 1.421413741, -1.453152027, 1.061405429)


def erfc_as(a):
    t = 1.0 / (1.0 + P * a)
    poly = sum(c * t ** (k + 1) for k, c in enumerate(A))
    return poly * np.exp(-a * a)


def test_as_7_1_26_bound():
    a = np.linspace(0, 10, 200001)
    assert np.max(np.abs((1 - erfc_as(a)) - erf(a))) <= 1.5e-7


def test_gelu_identity():
    z = np.linspace(-12, 12, 100001)
    exact = 0.5 * z * (1 + erf(z / np.sqrt(2)))
    fast = np.maximum(z, 0) - 0.5 * np.abs(z) * erfc_as(np.abs(z) / np.sqrt(2))
    assert np.max(np.abs(fast - exact)) <= 1.5e-7 * 0.5 * 12
    # bf16 output rounding is 2^-9 relative: the approximation is far below it
    big = np.abs(exact) > 1e-3
    assert np.max(np.abs(fast - exact)[big] / np.abs(exact[big])) < 2 ** -12
