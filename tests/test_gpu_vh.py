"""GPU parity of the von Hagenow boundary mode (include/efit.h EFIT_GREEN_VONHAGENOW; SURVEY 8(f)
f2) against the oracle's or_boundary_vh (the same construction; pinned at second order
against the Green's sum in tests/test_oracle_boundary_solve.py).

Tolerance: psi_b is a boundary integral of the normal derivative of the zero-Dirichlet solve
psi0, (4 psi0_1 - psi0_2)/(2h); psi0 agrees with the oracle's solve to ~1e-13 of max|psi0|
(the interior-solve parity), and the difference quotient divides that absolute error by h, so the
bound is ~1e-13 * (L/h) ~ 1e-13 N: 1e-12 * max(1, N/64)."""
import os

import numpy as np
import pytest

import synth

pytestmark = pytest.mark.gpu
VH = 4


def rel(a, b):
    a, b = np.asarray(a), np.asarray(b)
    return np.max(np.abs(a - b)) / max(np.max(np.abs(b)), 1e-300)


def tol_vh(n):
    return 1e-12 * max(1.0, n / 64.0)


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


@pytest.mark.parametrize("name", ["17x17", "33x33", "65x65", "C2", "C4"])
def test_vh_boundary_flux(torch_mod, efit, orc_mod, name):
    torch = torch_mod
    cfg = synth.config(name) if name.startswith("C") else synth.small_config(int(name.split("x")[0]))
    orc = orc_mod.Oracle.from_config(cfg)
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=VH)
    for seed, signed in ((2, False), (3, True)):
        I = synth.random_current(cfg.grid, seed=seed, signed=signed)
        ref = orc.boundary_vh(I)
        out = ctx.boundary_flux(T(torch, I)).cpu().numpy()
        assert rel(out, ref) < tol_vh(cfg.grid.nw), rel(out, ref)
    ctx.close()


@pytest.mark.parametrize("name", ["C1", "C2", "C4"])
def test_vh_fit_step(torch_mod, efit, orc_mod, name):
    """One fit iteration in VH mode against the oracle's fit step with the VH boundary; and the VH
    iterate is within the boundary approximation (second order) of the Green's-sum iterate."""
    torch = torch_mod
    cfg = synth.config(name)
    orc = orc_mod.Oracle.from_config(cfg)
    psi_s = synth.solovev_psi(cfg.grid)
    tw = orc.twin(psi_s, synth.c_true(cfg.basis), noise_seed=1)
    psi0 = synth.perturbed_psi(cfg.grid, seed=5, rel=1e-3)
    orc.set_boundary_method(1)
    st, pr, cr, chr_, er = orc.fit_step(psi0, tw["psi_ext"], tw["y"], tw["sigma"])
    orc.set_boundary_method(0)
    assert st == 0
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=VH)
    psi = T(torch, psi0)
    coef, chi2, eps = ctx._t(ctx.nbasis), ctx._t(1), ctx._t(1)
    ctx.fit_step(psi, T(torch, tw["psi_ext"]), T(torch, tw["y"]), T(torch, tw["sigma"]), coef, chi2, eps)
    torch.cuda.synchronize()
    assert ctx.status() == 0
    assert rel(psi.cpu().numpy(), pr) < tol_vh(cfg.grid.nw), rel(psi.cpu().numpy(), pr)
    assert rel(coef.cpu().numpy(), cr) < 1e-10
    st, pt, ct, _, _ = orc.fit_step(psi0, tw["psi_ext"], tw["y"], tw["sigma"])
    n = cfg.grid.nw
    assert rel(pr, pt) < 2.0 * (65.0 / n) ** 2 * 1e-3     # second order in h
    ctx.close()


def test_vh_loop_converges(torch_mod, efit, orc_mod):
    """C2 full loop in VH mode: converges (eps < 1e-5) to a fixed point within the
    boundary approximation of the twin's psi_S."""
    torch = torch_mod
    cfg = synth.config("C2")
    orc = orc_mod.Oracle.from_config(cfg)
    psi_s = synth.solovev_psi(cfg.grid)
    tw = orc.twin(psi_s, synth.c_true(cfg.basis))
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=VH)
    psi = T(torch, synth.perturbed_psi(cfg.grid, seed=5, rel=1e-2))
    ext, y, s = T(torch, tw["psi_ext"]), T(torch, tw["y"]), T(torch, tw["sigma"])
    coef, chi2, eps = ctx._t(ctx.nbasis), ctx._t(1), ctx._t(1)
    for it in range(300):
        ctx.fit_step(psi, ext, y, s, coef, chi2, eps)
        if eps.item() < 1e-5:
            break
    assert eps.item() < 1e-5
    assert rel(psi.cpu().numpy(), psi_s) < 1e-3
    ctx.close()
