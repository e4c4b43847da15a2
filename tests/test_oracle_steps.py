"""Pins for oracle steps O6-O11 (basis, axis/boundary/mask, response, current, LSQ)
against library routines (scipy BSpline, numpy lstsq), closed forms and constructed
cases whose answer is known without the oracle (single active node, linearity)."""
import math

import numpy as np
import pytest

import synth

MU0 = 4e-7 * math.pi


@pytest.fixture(scope="module", params=[(2, 3), (5, 5)], ids=["poly2+3", "poly5+5"])
def small(oracle_mod, request):
    cfg = synth.small_config(33, basis=synth.poly_basis(*request.param))
    return cfg, oracle_mod.Oracle.from_config(cfg)


def test_poly_basis_values(oracle_mod, small):
    cfg, orc = small
    for ph, R in [(0.0, 1.3), (0.37, 2.0), (0.999, 1.05)]:
        f = orc.basis_fn(ph, R)
        exp_pp = [R * ph ** k for k in range(cfg.basis.n_pp)]
        exp_ff = [MU0 / (4 * math.pi ** 2 * R) * ph ** k for k in range(cfg.basis.n_ff)]
        np.testing.assert_allclose(f, exp_pp + exp_ff, rtol=1e-15, atol=0)


def test_spline_basis_vs_scipy(oracle_mod):
    from scipy.interpolate import BSpline
    basis = synth.spline_basis(6)
    cfg = synth.small_config(33, basis=basis)
    orc = oracle_mod.Oracle.from_config(cfg)
    t = np.concatenate([[0, 0, 0, 0], basis.knots, [1, 1, 1, 1]])
    nb = len(t) - 4
    xs = np.concatenate([np.linspace(0, 0.999999, 97), basis.knots, [0.5 / 7]])
    for x in xs:
        f = orc.basis_fn(x, 1.0)[: basis.n_pp]
        ref = np.array([BSpline(t, np.eye(nb)[i], 3, extrapolate=False)(x) for i in range(nb)])
        ref = np.nan_to_num(ref)
        np.testing.assert_allclose(f, ref, rtol=0, atol=2e-15)
        assert abs(f.sum() - 1.0) < 4e-16 * 8  # partition of unity


def test_point_in_polygon_vs_winding(oracle_mod, small):
    """Even-odd rule vs an independent winding-number (angle sum) evaluation."""
    cfg, orc = small
    g = cfg.geometry
    inl = orc.inlim().reshape(cfg.grid.nw, cfg.grid.nh)
    R, Z = cfg.grid.r(), cfg.grid.z()
    for i in range(cfg.grid.nw):
        for j in range(cfg.grid.nh):
            dx = g.lim_r - R[i]; dy = g.lim_z - Z[j]
            ang = np.arctan2(dy, dx)
            d = np.diff(np.concatenate([ang, ang[:1]]))
            d = (d + np.pi) % (2 * np.pi) - np.pi
            wind = round(d.sum() / (2 * np.pi))
            assert inl[i, j] == (wind != 0)


def test_bilinear_exact_on_bilinear_function(oracle_mod, small):
    cfg, orc = small
    R, Z = cfg.grid.r()[:, None], cfg.grid.z()[None, :]
    psi = (1.5 + 0.3 * R - 0.7 * Z + 0.2 * R * Z).reshape(-1)
    for (r, z) in [(1.234, 0.567), (2.0, -1.3), (0.9, 1.5)]:
        assert abs(orc.bilinear(psi, r, z) - (1.5 + 0.3 * r - 0.7 * z + 0.2 * r * z)) < 1e-14


def test_normalize_solovev(oracle_mod, small):
    """Axis = in-limiter argmax of psi_S; boundary = max over limiter vertices; the touch
    vertex is the inboard-midplane one; mask = inlim & 0 <= psihat < 1."""
    cfg, orc = small
    psi = synth.solovev_psi(cfg.grid)
    cnt, pa, pb, mask, ph = orc.normalize(psi)
    inl = orc.inlim().astype(bool)
    assert pa == psi[inl].max()
    assert np.argmax(np.where(inl, psi, -np.inf)) == np.flatnonzero(psi == pa)[0]
    vals = [orc.bilinear(psi, r, z) for r, z in zip(cfg.geometry.lim_r, cfg.geometry.lim_z)]
    assert pb == max(vals) and int(np.argmax(vals)) == len(vals) // 2
    np.testing.assert_array_equal(mask.astype(bool), inl & (ph >= 0) & (ph < 1))
    assert cnt == mask.sum() > 0


def _peak_psi(cfg, nodes_vals):
    psi = np.zeros(cfg.grid.n)
    for (i, j), v in nodes_vals:
        psi[i * cfg.grid.nh + j] = v
    return psi


def test_response_single_active_node(oracle_mod, small):
    """psi = 1 at one in-limiter node, 0 elsewhere => axis there, psi_bdry = 0, only that node
    is masked (psihat 0 there, 1 elsewhere): resp[m][0] = Gd(m,g) dRdZ R_g,
    resp[m][n_pp] = Gd(m,g) dRdZ mu0/(4 pi^2 R_g), all other columns 0."""
    cfg, orc = small
    i, j = 16, 16
    psi = _peak_psi(cfg, [((i, j), 1.0)])
    resp, axbd = orc.response(psi)
    assert axbd[0] == 1.0 and axbd[1] == 0.0
    R = cfg.grid.r()[i]; Zs = cfg.grid.z()[j]
    cell = cfg.grid.dr * cfg.grid.dz
    g = cfg.geometry
    exp = []
    for m in range(orc.ndiag):
        if m < len(g.fl_r):
            exp.append(oracle_mod.green_psi(g.fl_r[m], g.fl_z[m], R, Zs))
        else:
            k = m - len(g.fl_r)
            br, bz = oracle_mod.green_brbz(g.mp_r[k], g.mp_z[k], R, Zs)
            exp.append(br * math.cos(g.mp_ang[k]) + bz * math.sin(g.mp_ang[k]))
    exp = np.array(exp)
    np.testing.assert_allclose(resp[:, 0], exp * cell * R, rtol=1e-15)
    npp = cfg.basis.n_pp
    np.testing.assert_allclose(resp[:, npp], exp * cell * MU0 / (4 * math.pi ** 2 * R), rtol=1e-15)
    others = np.delete(resp, [0, npp], axis=1)
    assert np.all(others == 0.0)


def test_response_two_nodes_powers(oracle_mod, small):
    """Second node at psi = 0.5 => psihat = 0.5 there: column k picks up 0.5^k."""
    cfg, orc = small
    a, b = (16, 16), (18, 15)
    psi = _peak_psi(cfg, [(a, 1.0), (b, 0.5)])
    resp, _ = orc.response(psi)
    Gd = orc.table_Gd()
    cell = cfg.grid.dr * cfg.grid.dz
    ga, gb = a[0] * cfg.grid.nh + a[1], b[0] * cfg.grid.nh + b[1]
    Ra, Rb = cfg.grid.r()[a[0]], cfg.grid.r()[b[0]]
    for k in range(cfg.basis.n_pp):
        exp = Gd[:, ga] * cell * Ra * (1.0 if k == 0 else 0.0) + Gd[:, gb] * cell * Rb * 0.5 ** k
        np.testing.assert_allclose(resp[:, k], exp, rtol=1e-13, atol=1e-30)


def test_probe_rows_are_field_of_flux(oracle_mod, small):
    """A probe row equals the directional derivative of a flux-loop-type row: for a
    diagnostic at x, B.n = (-(1/R) dpsi/dZ, (1/R) dpsi/dR).n, psi = sum_g G(x; g) B_g."""
    cfg, orc = small
    Gd = orc.table_Gd()
    g = cfg.geometry
    nfl = len(g.fl_r)
    R, Z = cfg.grid.r(), cfg.grid.z()
    RR, ZZ = np.meshgrid(R, Z, indexing="ij")
    for k in [0, 17, 40]:
        x, z, a = g.mp_r[k], g.mp_z[k], g.mp_ang[k]
        h = 2e-4
        flux = lambda xr, xz: np.array([oracle_mod.green_psi(xr, xz, r, zz) for r, zz in zip(RR.ravel(), ZZ.ravel())])
        d = lambda f0, f1, hh: (f1 - f0) / (2 * hh)
        dr1, dr2 = d(flux(x - h, z), flux(x + h, z), h), d(flux(x - h / 2, z), flux(x + h / 2, z), h / 2)
        dz1, dz2 = d(flux(x, z - h), flux(x, z + h), h), d(flux(x, z - h / 2), flux(x, z + h / 2), h / 2)
        dpdr, dpdz = (4 * dr2 - dr1) / 3, (4 * dz2 - dz1) / 3   # Richardson
        row = (-dpdz / x) * math.cos(a) + (dpdr / x) * math.sin(a)
        np.testing.assert_allclose(Gd[nfl + k], row, rtol=0, atol=1e-8 * np.abs(row).max())


def test_current_linearity_and_total(oracle_mod, small):
    cfg, orc = small
    psi = synth.solovev_psi(cfg.grid)
    c1, c2 = synth.random_coef(cfg.basis, 1), synth.random_coef(cfg.basis, 2)
    I1, I2, I12 = orc.current(psi, c1), orc.current(psi, c2), orc.current(psi, 2 * c1 - 3 * c2)
    np.testing.assert_allclose(I12, 2 * I1 - 3 * I2, rtol=0, atol=1e-14 * np.abs(I12).max())
    cnt, pa, pb, mask, ph = orc.normalize(psi)
    e0 = np.zeros(cfg.basis.nbasis); e0[0] = 1.0
    I = orc.current(psi, e0)
    RR = np.repeat(cfg.grid.r(), cfg.grid.nh)
    assert abs(I.sum() - math.fsum(cfg.grid.dr * cfg.grid.dz * RR[mask.astype(bool)])) < 1e-13 * I.sum()


def test_response_current_consistency(oracle_mod, small):
    """sum_k resp[m][k] c_k = sum_g Gd[m][g] I_g(c) (Eq. (2) is linear in the coefficients)."""
    cfg, orc = small
    psi = synth.perturbed_psi(cfg.grid, seed=5)
    c = synth.c_true(cfg.basis)
    resp, _ = orc.response(psi)
    I = orc.current(psi, c)
    Gd = orc.table_Gd()
    lhs = resp @ c
    rhs = np.array([math.fsum(Gd[m] * I) for m in range(orc.ndiag)])
    np.testing.assert_allclose(lhs, rhs, rtol=0, atol=1e-12 * np.abs(rhs).max())


def test_response_rows_match_full(oracle_mod, small):
    cfg, orc = small
    psi = synth.perturbed_psi(cfg.grid, seed=5)
    resp, _ = orc.response(psi)
    rows = [0, 3, 50, 119]
    sub = orc.response_rows(psi, rows)
    np.testing.assert_allclose(sub, resp[rows], rtol=0, atol=1e-15 * np.abs(resp).max())


def test_no_plasma(oracle_mod, small):
    cfg, orc = small
    with pytest.raises(RuntimeError):
        orc.response(np.zeros(cfg.grid.n))


# ------------------------------------------------------------------ LSQ (O10)

def test_lsq_vs_numpy(oracle_mod):
    rng = np.random.default_rng(3)
    for nd, nb in [(120, 10), (160, 20), (11, 10), (5, 1)]:
        A = rng.standard_normal((nd, nb)) * np.logspace(0, -6, nb)
        y = rng.standard_normal(nd)
        s = rng.uniform(0.5, 2.0, nd)
        st, c, chi2 = oracle_mod.lsq(A, y, s)
        assert st == 0
        ref, *_ = np.linalg.lstsq(A / s[:, None], y / s, rcond=None)
        np.testing.assert_allclose(c, ref, rtol=1e-9)
        assert abs(chi2 - np.sum(((y - A @ ref) / s) ** 2)) < 1e-10 * max(chi2, 1)


def test_lsq_one_parameter_closed_form(oracle_mod):
    rng = np.random.default_rng(4)
    a = rng.standard_normal(30); y = rng.standard_normal(30); s = rng.uniform(0.5, 2, 30)
    st, c, chi2 = oracle_mod.lsq(a[:, None], y, s)
    cref = math.fsum(a * y / s ** 2) / math.fsum(a * a / s ** 2)
    assert abs(c[0] - cref) < 1e-14 * abs(cref)
    assert abs(chi2 - math.fsum(((y - a * cref) / s) ** 2)) < 1e-13 * chi2


def test_lsq_exact_recovery_and_singular(oracle_mod):
    rng = np.random.default_rng(5)
    A = rng.standard_normal((40, 6)); ct = rng.standard_normal(6)
    st, c, chi2 = oracle_mod.lsq(A, A @ ct, np.ones(40))
    np.testing.assert_allclose(c, ct, rtol=1e-13)
    assert chi2 < 1e-25
    A[:, 3] = 2 * A[:, 1]
    st, _, _ = oracle_mod.lsq(A, A @ ct, np.ones(40))
    assert st == -5


def test_internal_bz_rows_are_field_of_flux(oracle_mod):
    """MSE-like internal rows (O5): row m = B_Z at an internal point x from a
    unit current at every node, B_Z = (1/R) dpsi/dR of the flux Green's function (
    B = grad psi x e_phi / R), by Richardson differences of or_green_psi -- pins the row's
    kind (B_Z, not B_R or psi) and its offset after the flux-loop and probe rows."""
    cfg = synth.small_config(65, n_int=10)
    orc = oracle_mod.Oracle.from_config(cfg)
    g = cfg.geometry
    off = len(g.fl_r) + len(g.mp_r)
    assert orc.ndiag == off + 10
    Gd = orc.table_Gd()
    R, Z = cfg.grid.r(), cfg.grid.z()
    RR, ZZ = np.meshgrid(R, Z, indexing="ij")
    for k in [0, 3, 9]:
        x, z = g.int_r[k], g.int_z[k]
        flux = lambda xr, xz: np.array([oracle_mod.green_psi(xr, xz, r, zz) for r, zz in zip(RR.ravel(), ZZ.ravel())])
        h = 2e-4
        d1 = (flux(x + h, z) - flux(x - h, z)) / (2 * h)
        d2 = (flux(x + h / 2, z) - flux(x - h / 2, z)) / h
        row = ((4 * d2 - d1) / 3) / x
        np.testing.assert_allclose(Gd[off + k], row, rtol=0, atol=1e-8 * np.abs(row).max())
        # and it is not B_R (dpsi/dZ): the two differ at O(1) off the midplane sources
        dz = (flux(x, z + h) - flux(x, z - h)) / (2 * h)
        assert np.max(np.abs(Gd[off + k] - (-dz / x))) > 0.1 * np.abs(row).max()
