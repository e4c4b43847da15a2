"""Pins for oracle steps O2-O5 (elliptic integrals, flux Green's function, filament field,
self term) against closed forms, mpmath, quadrature and calculus identities -- never
against the oracle itself.  SURVEY.md §8(c) "What pins each part"."""
import math
import os

import mpmath
import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

MU0_2PI = 2e-7


def test_golden_closed_forms(oracle_mod):
    mpmath.mp.dps = 40
    g14 = mpmath.gamma(mpmath.mpf(1) / 4)
    K_half = g14 ** 2 / (4 * mpmath.sqrt(mpmath.pi))
    E_half = g14 ** 2 / (8 * mpmath.sqrt(mpmath.pi)) + mpmath.pi ** 1.5 / g14 ** 2
    path = os.path.join(ROOT, "tests", "golden", "elliptic_closed_forms.txt")
    rows = [l.split() for l in open(path) if l.strip() and not l.startswith("#")]
    for m, K, E in rows:
        m, K, E = float(m), float(K), float(E)
        if m == 0.5:
            assert abs(float(K_half) - K) <= 2e-16 * K
            assert abs(float(E_half) - E) <= 2e-16 * E
        Ko, Eo = oracle_mod.ellip_ke(m)
        assert abs(Ko - K) <= 4 * np.spacing(K)
        assert abs(Eo - E) <= 4 * np.spacing(E)


@pytest.mark.parametrize("m1", [1e-13, 1e-10, 1e-7, 1e-4, 0.01, 0.2, 0.5, 0.8, 0.99, 1 - 1e-6])
def test_ellip_vs_mpmath(oracle_mod, m1):
    mpmath.mp.dps = 40
    m1m = mpmath.mpf(m1)
    m = float(1 - m1m)
    K, E = oracle_mod.ellip_ke(m, m1)
    Kr = mpmath.ellipk(1 - m1m)
    Er = mpmath.ellipe(1 - m1m)
    assert abs(K - float(Kr)) <= 4e-16 * float(Kr)
    # E = RF - (m/3) RD loses ~log10(K) digits as m -> 1 (cancellation); bound by K*eps
    assert abs(E - float(Er)) <= 4e-16 * max(1.0, float(Kr))


def test_legendre_relation(oracle_mod):
    """E K' + E' K - K K' = pi/2 for all m (DLMF 19.7.1)."""
    for m in np.linspace(0.01, 0.99, 25):
        K, E = oracle_mod.ellip_ke(m, 1 - m)
        Kp, Ep = oracle_mod.ellip_ke(1 - m, m)
        assert abs(E * Kp + Ep * K - K * Kp - math.pi / 2) < 4e-15


def test_K_log_asymptote(oracle_mod):
    """K(m) = ln(4/sqrt(m1)) + O(m1 ln m1) as m1 -> 0 (DLMF 19.12.1)."""
    for m1 in [1e-8, 1e-10, 1e-12]:
        K, _ = oracle_mod.ellip_ke(1 - m1, m1)
        assert abs(K - math.log(4 / math.sqrt(m1))) < 10 * m1 * abs(math.log(m1))


def _loop_flux_quadrature(R, Z, Rs, Zs, M=4000):
    """psi = R A_phi = (mu0 R Rs/4 pi) int_0^{2pi} cos(phi) dphi / sqrt(R^2+Rs^2+dz^2-2 R Rs cos phi)
    by the trapezoidal rule (exponentially convergent for a periodic integrand)."""
    phi = 2 * np.pi * np.arange(M) / M
    dz = Z - Zs
    # |r - r'|^2 = (R-Rs)^2 + dz^2 + 4 R Rs sin^2(phi/2), written without cancellation
    f = np.cos(phi) / np.sqrt((R - Rs) ** 2 + dz * dz + 4 * R * Rs * np.sin(phi / 2) ** 2)
    return 1e-7 * R * Rs * (2 * np.pi / M) * math.fsum(f)


PAIRS = [(1.0, 0.0, 1.5, 0.3), (0.9, -1.2, 2.4, 1.1), (2.5, 1.5, 0.85, -1.55),
         (1.7, 0.01, 1.71, 0.0), (1.2, 0.5, 1.25, 0.45), (2.0, 0.0, 2.0, 0.05)]


@pytest.mark.parametrize("pair", PAIRS)
def test_green_vs_quadrature(oracle_mod, pair):
    R, Z, Rs, Zs = pair
    G = oracle_mod.green_psi(R, Z, Rs, Zs)
    near = math.hypot(R - Rs, Z - Zs) < 0.1
    q = _loop_flux_quadrature(R, Z, Rs, Zs, M=200000 if near else 4000)
    assert abs(G - q) <= 1e-13 * abs(q)


def test_green_vs_mpmath_quad(oracle_mod):
    mpmath.mp.dps = 30
    R, Z, Rs, Zs = 1.3, 0.2, 2.1, -0.4
    f = lambda p: mpmath.cos(p) / mpmath.sqrt(R * R + Rs * Rs + (Z - Zs) ** 2 - 2 * R * Rs * mpmath.cos(p))
    ref = 1e-7 * R * Rs * mpmath.quad(f, [0, mpmath.pi, 2 * mpmath.pi])
    assert abs(oracle_mod.green_psi(R, Z, Rs, Zs) - float(ref)) <= 2e-15 * abs(float(ref))


def test_green_reciprocity(oracle_mod):
    rng = np.random.default_rng(0)
    for _ in range(200):
        R, Rs = rng.uniform(0.84, 2.54, 2)
        Z, Zs = rng.uniform(-1.6, 1.6, 2)
        a = oracle_mod.green_psi(R, Z, Rs, Zs)
        b = oracle_mod.green_psi(Rs, Zs, R, Z)
        assert abs(a - b) <= 4 * np.spacing(abs(a))


def test_green_is_homogeneous_solution(oracle_mod):
    """Delta* G = 0 away from the source; second-order FD residual shrinks as h^2."""
    R, Z, Rs, Zs = 1.4, 0.3, 2.0, -0.5
    res = []
    for h in [2e-3, 1e-3]:
        g = lambda r, z: oracle_mod.green_psi(r, z, Rs, Zs)
        d2r = (g(R + h, Z) - 2 * g(R, Z) + g(R - h, Z)) / h ** 2
        d1r = (g(R + h, Z) - g(R - h, Z)) / (2 * h)
        d2z = (g(R, Z + h) - 2 * g(R, Z) + g(R, Z - h)) / h ** 2
        scale = abs(d2r) + abs(d1r / R) + abs(d2z)
        res.append(abs(d2r - d1r / R + d2z) / scale)
    assert res[0] < 1e-5 and res[1] < res[0] / 3.0


def _richardson(f, x, h):
    d = lambda h: (f(x + h) - f(x - h)) / (2 * h)
    return (4 * d(h / 2) - d(h)) / 3


@pytest.mark.parametrize("pair", PAIRS[:5])
def test_field_is_curl_of_flux(oracle_mod, pair):
    """B_R = -(1/R) dpsi/dZ, B_Z = (1/R) dpsi/dR at the field point (O5)."""
    R, Z, Rs, Zs = pair
    br, bz = oracle_mod.green_brbz(R, Z, Rs, Zs)
    h = 1e-3 * max(0.05, math.hypot(R - Rs, Z - Zs))
    dpdz = _richardson(lambda z: oracle_mod.green_psi(R, z, Rs, Zs), Z, h)
    dpdr = _richardson(lambda r: oracle_mod.green_psi(r, Z, Rs, Zs), R, h)
    scale = math.hypot(br, bz)
    assert abs(br + dpdz / R) <= 1e-9 * scale
    assert abs(bz - dpdr / R) <= 1e-9 * scale


def test_field_divergence_free(oracle_mod):
    R, Z, Rs, Zs = 1.5, 0.4, 2.2, -0.3
    h = 1e-4
    d_rbr = (oracle_mod.green_brbz(R + h, Z, Rs, Zs)[0] * (R + h)
             - oracle_mod.green_brbz(R - h, Z, Rs, Zs)[0] * (R - h)) / (2 * h)
    d_bz = (oracle_mod.green_brbz(R, Z + h, Rs, Zs)[1] - oracle_mod.green_brbz(R, Z - h, Rs, Zs)[1]) / (2 * h)
    br, bz = oracle_mod.green_brbz(R, Z, Rs, Zs)
    assert abs(d_rbr / R + d_bz) < 1e-7 * math.hypot(br, bz) / 0.1


def test_self_term_vs_cell_average(oracle_mod):
    """O4: point-to-cell average of G over a uniformly filled cell, O((d/R)^2) agreement.
    The value is 'parity unpinned' beyond this (it never reaches a result)."""
    from scipy import integrate
    R = 1.7
    errs = []
    for n in [65, 257]:
        dR, dZ = 1.7 / (n - 1), 3.2 / (n - 1)
        ref, _ = integrate.dblquad(lambda z, r: oracle_mod.green_psi(R, 0.0, r, z),
                                   R - dR / 2, R + dR / 2, -dZ / 2, dZ / 2, epsabs=0, epsrel=1e-10)
        ref /= dR * dZ
        errs.append(abs(oracle_mod.green_self(R, dR, dZ) - ref) / abs(ref))
    assert errs[0] < 1e-4 and errs[1] < errs[0] / 8
