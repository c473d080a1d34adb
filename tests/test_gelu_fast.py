"""Pin the erf approximation the bf16 GEMM epilogues use (common.cuh gelu2_erf_fast), restated
here in fp64 and checked against scipy's erf (reading S2: GELU is the erf form):
  * Abramowitz & Stegun 7.1.28 (the default, one MUFU op per element):
    erfc(a) = (1 + c1 a + ... + c6 a^6)^-16, |erf error| <= 3e-7;
  * Abramowitz & Stegun 7.1.26 (ARLO_GELU2_AS26 A/B variant, two MUFU ops):
    erfc(a) = (a1 t + ... + a5 t^5) exp(-a^2), t = 1 / (1 + p a), |erf error| <= 1.5e-7;
and the identity GELU(z) = max(z, 0) - 0.5 |z| erfc(|z| / sqrt 2) both kernels evaluate."""
import numpy as np
from scipy.special import erf

P, A = 0.3275911, (0.254829592, -0.284496736, 1.421413741, -1.453152027, 1.061405429)
C28 = (0.0705230784, 0.0422820123, 0.0092705272, 0.0001520143, 0.0002765672, 0.0000430638)


def erfc_as26(a):
    t = 1.0 / (1.0 + P * a)
    poly = sum(c * t ** (k + 1) for k, c in enumerate(A))
    return poly * np.exp(-a * a)


def erfc_as28(a):
    return (1.0 + sum(c * a ** (k + 1) for k, c in enumerate(C28))) ** -16


def test_as_7_1_26_bound():
    a = np.linspace(0, 10, 200001)
    assert np.max(np.abs((1 - erfc_as26(a)) - erf(a))) <= 1.5e-7


def test_as_7_1_28_bound():
    a = np.linspace(0, 10, 200001)
    assert np.max(np.abs((1 - erfc_as28(a)) - erf(a))) <= 3e-7


def test_gelu_identity():
    z = np.linspace(-12, 12, 100001)
    exact = 0.5 * z * (1 + erf(z / np.sqrt(2)))
    big = np.abs(exact) > 1e-3
    for erfc, bound, rel in ((erfc_as26, 1.5e-7, 2 ** -12), (erfc_as28, 3e-7, 2 ** -11)):
        fast = np.maximum(z, 0) - 0.5 * np.abs(z) * erfc(np.abs(z) / np.sqrt(2))
        assert np.max(np.abs(fast - exact)) <= bound * 0.5 * 12
        # bf16 output rounding is 2^-9 relative: the approximation stays well below it
        assert np.max(np.abs(fast - exact)[big] / np.abs(exact[big])) < rel


def test_as28_fp32_evaluation():
    """The kernel's fp32 evaluation order (coefficients pre-scaled by 2^(-k/2), Horner in |z|,
    rcp then four squarings) stays within 2^-11 relative of the exact GELU where |GELU| > 1e-3
    and within 1e-6 absolute everywhere."""
    z = np.linspace(-12, 12, 400001).astype(np.float32)
    az = np.abs(z)
    s = 2 ** -0.5
    p = np.float32(C28[5] * s ** 6)
    for k in range(4, -1, -1):
        p = (az * p + np.float32(C28[k] * s ** (k + 1))).astype(np.float32)
    p = (az * p + np.float32(1)).astype(np.float32)
    r = (np.float32(1) / p).astype(np.float32)
    for _ in range(4):
        r = (r * r).astype(np.float32)
    g = (np.maximum(z, 0) + (np.float32(-0.5) * az) * r).astype(np.float64)
    exact = 0.5 * z.astype(np.float64) * (1 + erf(z / np.sqrt(2)))
    assert np.max(np.abs(g - exact)) <= 1e-6
    big = np.abs(exact) > 1e-3
    assert np.max(np.abs(g - exact)[big] / np.abs(exact[big])) < 2 ** -11
