"""Pins for the oracle's full steps_ (reading R4): the bicubic
Hermite interpolant, the Newton stationary-point search, the axis / X-point / boundary rule and
the connectivity-filtered mask.  Pinned against closed forms (quadratics are reproduced exactly;
the diverted Solov'ev's X-points are analytic), finite differences of the interpolant's own values,
scipy.ndimage.label (an independent flood fill) and the O8 rule it must reduce to for a limited
plasma.  steps_ itself is only named by the paper."""
import math

import numpy as np
import pytest

import synth


def _oracle(oracle_mod, n, steps=1):
    cfg = synth.small_config(n)
    orc = oracle_mod.Oracle.from_config(cfg)
    orc.set_steps_mode(steps)
    return cfg, orc


def _quadratic(cfg, a, b, c, d, e, f):
    """psi = a t^2 + b u^2 + c t u + d t + e u + f in index coordinates (t, u) = (i, j)."""
    t = np.arange(cfg.grid.nw, dtype=np.float64)[:, None]
    u = np.arange(cfg.grid.nh, dtype=np.float64)[None, :]
    return (a * t * t + b * u * u + c * t * u + d * t + e * u + f).reshape(-1)


def test_hermite_reproduces_quadratics(oracle_mod):
    """Central differences are exact for quadratics and the bicubic Hermite patch reproduces every
    bicubic, so value and all derivatives equal the quadratic's closed form anywhere."""
    cfg, orc = _oracle(oracle_mod, 17)
    rng = np.random.default_rng(11)
    for _ in range(5):
        a, b, c, d, e, f = rng.uniform(-1, 1, 6)
        psi = _quadratic(cfg, a, b, c, d, e, f)
        for _ in range(20):
            t, u = rng.uniform(1.0, 14.0, 2)
            got = orc.hermite_eval(psi, t, u)
            exp = [a * t * t + b * u * u + c * t * u + d * t + e * u + f,
                   2 * a * t + c * u + d, 2 * b * u + c * t + e, 2 * a, 2 * b, c]
            np.testing.assert_allclose(got, exp, rtol=0, atol=1e-12 * (1 + np.abs(exp).max()))


def test_hermite_derivatives_match_finite_differences(oracle_mod):
    """The derivative basis functions against central differences of the interpolant's values
    (pins every d/e polynomial against the value polynomials) on a non-polynomial psi."""
    cfg, orc = _oracle(oracle_mod, 33)
    psi = synth.solovev_diverted_psi(cfg.grid) + 1e-3 * synth.smooth_modes(cfg.grid, 3)
    rng = np.random.default_rng(12)
    h = 1e-4
    for _ in range(30):
        t, u = rng.uniform(2.05, 29.95, 2)
        if abs(t - round(t)) < 2 * h or abs(u - round(u)) < 2 * h:
            continue  # stay inside one cell (the second derivatives jump across cell edges)
        p = lambda dt, du: orc.hermite_eval(psi, t + dt, u + du)[0]
        d = orc.hermite_eval(psi, t, u)
        fd = [(p(h, 0) - p(-h, 0)) / (2 * h), (p(0, h) - p(0, -h)) / (2 * h),
              (p(h, 0) - 2 * p(0, 0) + p(-h, 0)) / h ** 2, (p(0, h) - 2 * p(0, 0) + p(0, -h)) / h ** 2,
              (p(h, h) - p(h, -h) - p(-h, h) + p(-h, -h)) / (4 * h * h)]
        scale = np.abs(psi).max()
        np.testing.assert_allclose(d[1:], fd, rtol=0, atol=1e-6 * scale)


def test_hermite_interpolates_and_is_c1(oracle_mod):
    """At a node: the node value and the central differences; across a cell edge: p and both
    first derivatives continuous (C1), the property that makes Newton's method well defined."""
    cfg, orc = _oracle(oracle_mod, 33)
    psi = synth.solovev_diverted_psi(cfg.grid) + 1e-3 * synth.smooth_modes(cfg.grid, 4)
    P = psi.reshape(33, 33)
    for (i, j) in [(3, 4), (10, 20), (17, 17), (29, 2 + 1)]:
        d = orc.hermite_eval(psi, float(i), float(j))
        assert d[0] == P[i, j]
        assert abs(d[1] - 0.5 * (P[i + 1, j] - P[i - 1, j])) <= 1e-15 * abs(P).max()
        assert abs(d[2] - 0.5 * (P[i, j + 1] - P[i, j - 1])) <= 1e-15 * abs(P).max()
    eps = 1e-12
    for x in [5.0, 12.0, 20.0]:
        for u in [7.3, 15.5]:
            lo, hi = orc.hermite_eval(psi, x - eps, u), orc.hermite_eval(psi, x + eps, u)
            np.testing.assert_allclose(lo[:3], hi[:3], rtol=0, atol=1e-9 * abs(P).max())


@pytest.mark.parametrize("kind", ["max", "saddle"])
def test_newton_finds_quadratic_stationary_point(oracle_mod, kind):
    """A quadratic's stationary point solves a 2x2 linear system: Newton lands on it exactly."""
    cfg, orc = _oracle(oracle_mod, 21)
    t0, u0 = 9.37, 11.61
    if kind == "max":
        a, b, c = -1.0, -0.6, 0.3
    else:
        a, b, c = -1.0, 0.7, 0.2
    # psi = a (t-t0)^2 + b (u-u0)^2 + c (t-t0)(u-u0) + 0.25
    d = -2 * a * t0 - c * u0
    e = -2 * b * u0 - c * t0
    f = a * t0 * t0 + b * u0 * u0 + c * t0 * u0 + 0.25
    psi = _quadratic(cfg, a, b, c, d, e, f)
    conv, out = orc.newton_stationary(psi, 9.0, 12.0)
    assert conv
    assert abs(out[0] - t0) < 1e-11 and abs(out[1] - u0) < 1e-11
    assert abs(out[2] - 0.25) < 1e-12
    assert (out[3] > 0) == (kind == "max")


def test_axis_and_xpoints_converge_to_analytic_double_null(oracle_mod):
    """Double-null Solov'ev (d = 0): axis at (R0, 0) with psi = 0, X-points at (R_x, +-Z_x) with
    psi_x = -scale B (R0^2 - R_x^2)^2 (closed forms, synth.diverted_xpoints).  Errors fall at least
    at second order in the grid spacing
    over the refinement (the first halving is pre-asymptotic)."""
    rx, zx, psix = synth.diverted_xpoints()
    errs = []
    for n in (33, 65, 129, 257):
        cfg, orc = _oracle(oracle_mod, n)
        psi = synth.solovev_diverted_psi(cfg.grid, d=0.0)
        cnt, pa, pb, mask, ph = orc.normalize(psi)
        info = orc.steps_info()
        assert cnt > 0 and info[4] == 1.0 and info[12] in (1.0, 2.0)
        e = max(abs(info[2] - synth.SOL_R0), abs(info[3]), abs(info[6] - rx), abs(info[7] + zx),
                abs(info[9] - rx), abs(info[10] - zx))
        ev = max(abs(pa), abs(info[8] - psix), abs(info[11] - psix)) / abs(psix)
        errs.append((e, ev))
        assert pb == (info[8] if info[12] == 1.0 else info[11])
    for (e1, v1), (e2, v2) in zip(errs, errs[1:]):
        assert e2 < e1 / 2.0 and v2 < v1 / 3.0, errs
    # 33^2 is pre-asymptotic; over the 8x refinement second order gives 64x
    assert errs[-1][0] < errs[0][0] / 40 and errs[-1][1] < errs[0][1] / 64, errs
    assert errs[-1][0] < 2e-5 and errs[-1][1] < 1e-5


def test_limited_plasma_reduces_to_o8(oracle_mod):
    """No X-point inside the limiter (the default limited Solov'ev): the boundary is O8's limiter
    value and the mask O8's mask (the plasma region is connected); only the axis value is refined,
    towards the analytic psi_S(R0, 0) = 0."""
    for n in (33, 65):
        cfg = synth.small_config(n)
        o8 = oracle_mod.Oracle.from_config(cfg)
        f3 = oracle_mod.Oracle.from_config(cfg)
        f3.set_steps_mode(1)
        psi = synth.solovev_psi(cfg.grid)
        c8, pa8, pb8, m8, _ = o8.normalize(psi)
        c3, pa3, pb3, m3, _ = f3.normalize(psi)
        info = f3.steps_info()
        assert info[12] == 0.0 and np.isnan(info[6]) and np.isnan(info[9])
        assert pb3 == pb8 and c3 == c8 and np.array_equal(m3, m8)
        assert abs(pa3) <= abs(pa8) and abs(pa3) < 1e-5


@pytest.mark.parametrize("n", [65, 129])
def test_diverted_boundary_and_connected_mask(oracle_mod, n):
    """Lower-single-null Solov'ev: the boundary is the lower X-point (above the O8 limiter value,
    which sits in the private flux under the X-point), and the mask is the component of the axis
    node in {inlim, 0 <= psihat < 1}, computed independently by scipy.ndimage.label (4-connected);
    the private-flux regions (psihat < 1 below / above the X-points) are other components."""
    import scipy.ndimage as ndi
    cfg, orc = _oracle(oracle_mod, n)
    psi = synth.solovev_diverted_psi(cfg.grid)
    cnt, pa, pb, mask, ph = orc.normalize(psi)
    info = orc.steps_info()
    assert info[12] == 1.0 and pb == info[8] and info[7] < info[3] < info[10]
    assert info[8] > info[11]  # the lower X-point is the primary one (d > 0)
    assert info[5] < pb  # the wall between the X-point heights is further out than the separatrix
    inl = orc.inlim().astype(bool)
    cand = (inl & (ph >= 0) & (ph < 1)).reshape(n, n)
    lab, nlab = ndi.label(cand)  # default structure: 4-connectivity
    g0 = int(info[15])
    comp = lab.reshape(-1) == lab.reshape(-1)[g0]
    assert np.array_equal(comp, mask.astype(bool)) and cnt == comp.sum()
    assert nlab >= 3
    # private flux below the lower X-point: candidate nodes left out of the mask
    Z = np.broadcast_to(cfg.grid.z()[None, :], (n, n)).reshape(-1)
    priv = cand.reshape(-1) & ~mask.astype(bool) & (Z < info[7])
    assert priv.sum() > 0
    # O8's rule on the same psi takes the private-flux wall as the boundary: a smaller plasma
    o8 = oracle_mod.Oracle.from_config(cfg)
    c8, _, pb8, _, _ = o8.normalize(psi)
    assert pb8 > pb and c8 < cnt


def test_xpoint_is_a_stationary_saddle_of_the_interpolant(oracle_mod):
    """Newton's result checked through the interpolant's values only: a central-difference gradient
    of p at the X-point vanishes and its second differences are indefinite."""
    cfg, orc = _oracle(oracle_mod, 129)
    psi = synth.solovev_diverted_psi(cfg.grid)
    orc.normalize(psi)
    info = orc.steps_info()
    t = (info[6] - cfg.grid.rmin) / cfg.grid.dr
    u = (info[7] - cfg.grid.zmin) / cfg.grid.dz
    p = lambda a, b: orc.hermite_eval(psi, t + a, u + b)[0]
    h = 1e-3
    gt = (p(h, 0) - p(-h, 0)) / (2 * h)
    gu = (p(0, h) - p(0, -h)) / (2 * h)
    scale = abs(info[8]) + abs(info[0])
    assert abs(gt) < 1e-7 * scale and abs(gu) < 1e-7 * scale
    assert abs(p(0, 0) - info[8]) < 1e-15 * scale
    pt2 = p(h, 0) + p(-h, 0) - 2 * p(0, 0)
    pu2 = p(0, h) + p(0, -h) - 2 * p(0, 0)
    ptu = (p(h, h) - p(h, -h) - p(-h, h) + p(-h, -h)) / 4
    assert pt2 * pu2 - ptu * ptu < 0  # indefinite second difference: a saddle


def test_diverted_twin_is_an_exact_fixed_point(oracle_mod):
    """Twin of the diverted Solov'ev in f3 mode: one fit step from psi_S returns psi_S and c_true
    (the twin construction is exact for any normalisation rule)."""
    cfg, orc = _oracle(oracle_mod, 65)
    psi = synth.solovev_diverted_psi(cfg.grid)
    ct = synth.c_true(cfg.basis, sol_c=synth.DIV_C)
    tw = orc.twin(psi, ct)
    st, p1, c1, chi2, eps = orc.fit_step(psi, tw["psi_ext"], tw["y"], tw["sigma"])
    assert st == 0
    assert np.abs(p1 - psi).max() < 1e-14 * np.abs(psi).max()
    assert np.abs(c1 - ct).max() < 1e-10 * np.abs(ct).max()
    assert chi2 < 1e-18 and eps < 1e-12


def test_no_plasma_and_degenerate_inputs(oracle_mod):
    """Flat psi: no X-point, psi_axis == psi_bdry -> no plasma; non-finite psi -> no plasma."""
    cfg, orc = _oracle(oracle_mod, 17)
    cnt, *_ = orc.normalize(np.zeros(cfg.grid.n))
    assert cnt == -1
    psi = synth.solovev_diverted_psi(cfg.grid)
    psi[100] = np.nan
    cnt, *_ = orc.normalize(psi)
    assert cnt == -1
