"""GPU parity on the benched path and the survey's configs at full size.

* C4 (513^2, the bench workload): the chained efit_fit_steps call bench.py times, in the SYM
  (bench default) and TABLE Green's modes, against consecutive or_fit_step calls of the oracle;
  every one of the 2048 edge targets and all 120 response rows.
* C3 (257^2, 10+10 cubic B-splines, 40 MSE-like B_Z rows): one fit step and the spline current.
* The survey's 5+5 polynomial basis (nbasis = 10: k_response_mma + k_lsq<10>) at C1 and C4.
* C5 (1025^2): 64 edge targets (all corners and side ends) and all 120 response rows.
* The C2/C4 full loops converge to the twin's psi_S and c -> c_true.

Tolerances (north_star): 1e-12 normwise on psi / psi_b / response columns, 1e-10 on the fitted
coefficients and chi2 -- except where the least-squares problem is ill-conditioned: the
coefficient error bound of any backward-stable fp64 solver is ~ cond(A_scaled) * u (Higham,
Accuracy and Stability, Thm 20.1), so the coefficient tolerance is max(1e-10, 50 * cond * u)
with cond measured on the oracle's scaled matrix.  Chained steps:
differences of ~1e-15 in psi enter the next fit through the same conditioning, so step k > 1
of a chained run is compared at the coefficient tolerance (psi stays at 1e-12 once the basis
is well conditioned).
"""
import os

import numpy as np
import pytest

import synth

pytestmark = pytest.mark.gpu

TOL = 1e-12
TOL_C = 1e-10
U = 2.0 ** -53


def rel(a, b):
    a, b = np.asarray(a), np.asarray(b)
    return np.max(np.abs(a - b)) / max(np.max(np.abs(b)), 1e-300)


@pytest.fixture(scope="module")
def torch_mod():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch


@pytest.fixture(scope="module")
def efit(torch_mod):
    import paper_conf_sc_anteparawkbml23_b200 as e
    e.lib()
    return e


@pytest.fixture(scope="module")
def orc_mod():
    import oracle
    oracle.build()
    oracle.set_threads(os.cpu_count() or 1)
    return oracle


def T(torch, a):
    return torch.tensor(np.ascontiguousarray(np.asarray(a, dtype=np.float64)), device="cuda")


def scaled_cond(resp, sigma):
    """2-norm condition number of the row-(1/sigma), column-unit-norm scaled LSQ matrix (O10)."""
    A = resp / sigma[:, None]
    A = A / np.linalg.norm(A, axis=0)
    s = np.linalg.svd(A, compute_uv=False)
    return s[0] / s[-1]


def coef_tol(cond):
    return max(TOL_C, 50.0 * cond * U)


# ------------------------------------------------------------------------ C4 (bench workload)

@pytest.fixture(scope="module")
def c4(efit, orc_mod):
    cfg = synth.config("C4")
    orc = orc_mod.Oracle.from_config(cfg)
    psi_s = synth.solovev_psi(cfg.grid)
    ct = synth.c_true(cfg.basis)
    tw = orc.twin(psi_s, ct, noise_seed=1)   # builds the oracle's T and Gd memo tables
    return cfg, orc, psi_s, ct, tw


@pytest.fixture(scope="module")
def c4_ref3(c4):
    """Three consecutive oracle iterations from the bench's start (psi_S + 0.1% modes, seed 5)."""
    cfg, orc, psi_s, ct, tw = c4
    psi = synth.perturbed_psi(cfg.grid, seed=5, rel=1e-3)
    out = []
    for _ in range(3):
        st, psi, coef, chi2, eps = orc.fit_step(psi, tw["psi_ext"], tw["y"], tw["sigma"])
        assert st == 0
        out.append((psi.copy(), coef.copy(), chi2, eps))
    return out


@pytest.mark.parametrize("mode", [2, 0], ids=["sym", "table"])
def test_c4_fit_steps_chained(torch_mod, efit, c4, c4_ref3, mode):
    """The benched call: efit_fit_steps(n) on the bench's inputs, n = 1 and n = 3 (one graph, the
    axis/boundary of iterations 2-3 from the previous update kernel), against or_fit_step x n."""
    torch = torch_mod
    cfg, orc, psi_s, ct, tw = c4
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=mode)
    ext, y, s = T(torch, tw["psi_ext"]), T(torch, tw["y"]), T(torch, tw["sigma"])
    psi0 = synth.perturbed_psi(cfg.grid, seed=5, rel=1e-3)
    resp_ref, _ = orc.response(psi0)
    tc = coef_tol(scaled_cond(resp_ref, tw["sigma"]))
    for n in (1, 3):
        psi = T(torch, psi0)
        coef, chi2, eps = ctx._t(ctx.nbasis), ctx._t(1), ctx._t(1)
        ctx.fit_steps(n, psi, ext, y, s, coef, chi2, eps)
        torch.cuda.synchronize()
        assert ctx.status() == 0
        pr, cr, chr_, er = c4_ref3[n - 1]
        assert rel(psi.cpu().numpy(), pr) < TOL, (n, rel(psi.cpu().numpy(), pr))
        assert rel(coef.cpu().numpy(), cr) < tc, (n, rel(coef.cpu().numpy(), cr), tc)
        assert abs(chi2.item() - chr_) <= tc * max(chr_, 1.0)
        assert abs(eps.item() - er) <= 1e-9 * er
    ctx.close()


@pytest.mark.parametrize("mode", [2, 0], ids=["sym", "table"])
def test_c4_boundary_all_targets(torch_mod, efit, c4, mode):
    """All 2048 edge targets at 513^2 (corners and both ends of every side included)."""
    torch = torch_mod
    cfg, orc, *_ = c4
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=mode)
    for seed, signed in ((2, False), (3, True)):
        I = synth.random_current(cfg.grid, seed=seed, signed=signed)
        ref = orc.boundary(I)
        out = ctx.boundary_flux(T(torch, I)).cpu().numpy()
        assert out.shape == (2048,)
        assert rel(out, ref) < TOL, (seed, rel(out, ref))
    ctx.close()


def test_c4_response_all_rows(torch_mod, efit, c4):
    """All 120 response rows x 5 columns at 513^2 (the benched k_response configuration)."""
    torch = torch_mod
    cfg, orc, psi_s, ct, tw = c4
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=2)
    psi = synth.perturbed_psi(cfg.grid, seed=5, rel=1e-3)
    ref, axbd_ref = orc.response(psi)
    resp, axbd = ctx.response(T(torch, psi))
    torch.cuda.synchronize()
    assert ctx.status() == 0
    assert np.array_equal(axbd.cpu().numpy(), axbd_ref)
    r = resp.cpu().numpy()
    assert r.shape == (120, ctx.nbasis)
    for k in range(ctx.nbasis):
        assert rel(r[:, k], ref[:, k]) < TOL, (k, rel(r[:, k], ref[:, k]))
    ctx.close()


def test_c4_loop_converges_to_twin(torch_mod, efit, c4):
    """Full loop at C4 on the GPU from a 1% start (noise-free twin): eps < 1e-5, and
    continued to eps < 1e-10 the iterate is the twin's psi_S with c = c_true (properties of the
    twin construction, valid at any size; the per-iteration oracle parity is C2's test)."""
    torch = torch_mod
    cfg, orc, psi_s, ct, _ = c4
    tw = orc.twin(psi_s, ct)   # noise-free
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=2)
    ext, y, s = T(torch, tw["psi_ext"]), T(torch, tw["y"]), T(torch, tw["sigma"])
    psi = T(torch, synth.perturbed_psi(cfg.grid, seed=5, rel=1e-2))
    coef, chi2, eps = ctx._t(ctx.nbasis), ctx._t(1), ctx._t(1)
    first = None
    for it in range(600):
        ctx.fit_step(psi, ext, y, s, coef, chi2, eps)
        e = eps.item()
        if first is None and e < 1e-5:
            first = it
        if e < 1e-10:
            break
    assert ctx.status() == 0
    assert first is not None and first < 200
    assert e < 1e-10
    span = np.max(np.abs(psi_s))
    assert np.max(np.abs(psi.cpu().numpy() - psi_s)) < 1e-8 * span
    assert np.max(np.abs(coef.cpu().numpy() - ct)) < 1e-7 * np.max(np.abs(ct))
    ctx.close()


# ------------------------------------------------------------------------ the 5+5 basis (nb = 10)

@pytest.mark.parametrize("name", ["C1", "C4"])
def test_poly55_fit_step(torch_mod, efit, orc_mod, name):
    """The survey's Q8 reading (5+5 monomials, nbasis = 10): the single-slice DMMA response kernel
    (k_response_mma, nb >= 8) and k_lsq<10>, one fit step against the oracle."""
    torch = torch_mod
    base = synth.config(name)
    cfg = synth.Config(name + "-5+5", base.grid, base.geometry, synth.poly_basis(5, 5), "5+5")
    orc = orc_mod.Oracle.from_config(cfg)
    psi_s = synth.solovev_psi(cfg.grid)
    ct = synth.c_true(cfg.basis)
    tw = orc.twin(psi_s, ct, noise_seed=1)
    psi0 = synth.perturbed_psi(cfg.grid, seed=5, rel=1e-3)
    resp_ref, axbd_ref = orc.response(psi0)
    st, pr, cr, chr_, er = orc.fit_step(psi0, tw["psi_ext"], tw["y"], tw["sigma"])
    assert st == 0
    for mode in (0, 2):
        ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=mode)
        assert ctx.nbasis == 10
        resp, axbd = ctx.response(T(torch, psi0))
        r = resp.cpu().numpy()
        for k in range(10):
            assert rel(r[:, k], resp_ref[:, k]) < TOL, (k, rel(r[:, k], resp_ref[:, k]))
        psi = T(torch, psi0)
        coef, chi2, eps = ctx._t(10), ctx._t(1), ctx._t(1)
        ctx.fit_step(psi, T(torch, tw["psi_ext"]), T(torch, tw["y"]), T(torch, tw["sigma"]), coef, chi2, eps)
        torch.cuda.synchronize()
        assert ctx.status() == 0
        tc = coef_tol(scaled_cond(resp_ref, tw["sigma"]))
        # psi_new depends on c only through the current, whose error is ~ u * |I| even when the
        # individual coefficients of the ill-conditioned basis move by cond * u
        assert rel(psi.cpu().numpy(), pr) < max(TOL, tc * 1e-2), rel(psi.cpu().numpy(), pr)
        assert rel(coef.cpu().numpy(), cr) < tc, (rel(coef.cpu().numpy(), cr), tc)
        assert abs(chi2.item() - chr_) <= tc * max(chr_, 1.0)
        ctx.close()


# ------------------------------------------------------------------------ C3 (spline + MSE)

@pytest.fixture(scope="module")
def c3(efit, orc_mod):
    cfg = synth.config("C3")
    orc = orc_mod.Oracle.from_config(cfg)
    psi_s = synth.solovev_psi(cfg.grid)
    ct = synth.c_true(cfg.basis)
    tw = orc.twin(psi_s, ct, noise_seed=1)
    return cfg, orc, psi_s, ct, tw


def test_c3_fit_step(torch_mod, efit, c3):
    """C3: 257^2, 10+10 cubic B-spline basis, 44 flux loops + 76 probes + 40 internal B_Z rows:
    one fit step (response incl. the MSE rows, k_lsq<20>, spline current, boundary, solve)."""
    torch = torch_mod
    cfg, orc, psi_s, ct, tw = c3
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=2)
    assert ctx.ndiag == 160 and ctx.nbasis == 20
    psi0 = synth.perturbed_psi(cfg.grid, seed=5, rel=1e-3)
    resp_ref, _ = orc.response(psi0)
    st, pr, cr, chr_, er = orc.fit_step(psi0, tw["psi_ext"], tw["y"], tw["sigma"])
    assert st == 0
    tc = coef_tol(scaled_cond(resp_ref, tw["sigma"]))
    for n in (1, 2):
        psi = T(torch, psi0)
        coef, chi2, eps = ctx._t(20), ctx._t(1), ctx._t(1)
        if n == 1:
            ctx.fit_step(psi, T(torch, tw["psi_ext"]), T(torch, tw["y"]), T(torch, tw["sigma"]), coef, chi2, eps)
        else:  # graph replay of the same call
            for _ in range(2):
                psi.copy_(T(torch, psi0))
                ctx.fit_step(psi, T(torch, tw["psi_ext"]), T(torch, tw["y"]), T(torch, tw["sigma"]), coef, chi2, eps)
        torch.cuda.synchronize()
        assert ctx.status() == 0
        assert rel(psi.cpu().numpy(), pr) < TOL, rel(psi.cpu().numpy(), pr)
        assert rel(coef.cpu().numpy(), cr) < tc, (rel(coef.cpu().numpy(), cr), tc)
        assert abs(chi2.item() - chr_) <= tc * max(chr_, 1.0)
        assert abs(eps.item() - er) <= 1e-9 * er
    ctx.close()


def test_c3_spline_current(torch_mod, efit, c3):
    """efit_current with the cubic B-spline basis (O6/O11): identical mask, 1e-12."""
    torch = torch_mod
    cfg, orc, psi_s, ct, tw = c3
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=2)
    for seed, psi in ((5, synth.perturbed_psi(cfg.grid, seed=5, rel=1e-3)), (0, psi_s)):
        coef = synth.c_true(cfg.basis, seed=seed + 1)
        ref = orc.current(psi, coef)
        out = ctx.current(T(torch, psi), T(torch, coef)).cpu().numpy()
        assert np.array_equal(out != 0, ref != 0)
        assert rel(out, ref) < TOL, rel(out, ref)
    ctx.close()


# ------------------------------------------------------------------------ C5 (1025^2)

def test_c5_sampled_64_targets_all_rows(torch_mod, efit, orc_mod):
    """configs[4]: 64 edge targets (the corners, both ends of every side, random others) and all
    120 response rows, in the half-table mode (m-chunked SYM kernel) and the full table."""
    torch = torch_mod
    cfg = synth.config("C5")
    orc = orc_mod.Oracle.from_config(cfg)
    nh, nw = cfg.grid.nh, cfg.grid.nw
    n_edge = 2 * nh + 2 * (nw - 2)
    fixed = [0, 1, nh - 2, nh - 1, nh, nh + 1, 2 * nh - 2, 2 * nh - 1, 2 * nh, 2 * nh + 1,
             2 * nh + nw - 3, 2 * nh + nw - 2, 2 * nh + nw - 1, n_edge - 2, n_edge - 1, nh // 2]
    rng = np.random.default_rng(1)
    extra = rng.choice(np.setdiff1d(np.arange(n_edge), fixed), 64 - len(fixed), replace=False)
    tg = np.sort(np.concatenate([fixed, extra]))
    assert len(np.unique(tg)) == 64
    I = synth.random_current(cfg.grid, seed=3, signed=True)
    ref_b = orc.boundary_targets(I, tg)
    psi = synth.perturbed_psi(cfg.grid, seed=5, rel=1e-3)
    ref_r = orc.response_rows(psi, list(range(cfg.geometry.ndiag)))
    for mode in (2, 0):
        ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=mode)
        out = ctx.boundary_flux(T(torch, I)).cpu().numpy()
        assert rel(out[tg], ref_b) < TOL, (mode, rel(out[tg], ref_b))
        if mode == 2:
            resp, _ = ctx.response(T(torch, psi))
            r = resp.cpu().numpy()
            assert r.shape == (120, ctx.nbasis)
            for k in range(ctx.nbasis):
                assert rel(r[:, k], ref_r[:, k]) < TOL, (k, rel(r[:, k], ref_r[:, k]))
        ctx.close()
        del ctx
        torch.cuda.empty_cache()
