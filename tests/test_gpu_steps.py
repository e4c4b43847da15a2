"""GPU parity of the full steps_ (reading R4; include/efit.h
EFIT_STEPS_FULL) against the oracle's or_normalize in steps mode 1, on the same seeded inputs.

Every steps_ output is a decision or a value taken in the same fp64 operation order on both sides
(oracle -ffp-contract=off, efit_steps.cu -fmad=false), so axis, X-points, boundary, kind, count and
the mask must agree BIT FOR BIT.  Fit steps in this mode: the north_star tolerances (1e-12 on psi,
1e-10 on coefficients and chi2)."""
import os

import numpy as np
import pytest

import synth

pytestmark = pytest.mark.gpu

TOL = 1e-12
TOL_C = 1e-10


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


def _psi(kind, grid):
    if kind == "diverted":
        return synth.solovev_diverted_psi(grid)
    if kind == "double_null":
        return synth.solovev_diverted_psi(grid, d=0.0)
    if kind == "limited":
        return synth.solovev_psi(grid)
    if kind == "diverted_perturbed":
        p = synth.solovev_diverted_psi(grid)
        return p + 1e-3 * (p.max() - p.min()) * synth.smooth_modes(grid, 5) / 3.0
    if kind == "noisy":  # many X-point candidates (exercises the best-8 selection)
        p = synth.solovev_diverted_psi(grid)
        rng = np.random.default_rng(9)
        return p + 1e-4 * (p.max() - p.min()) * rng.standard_normal(p.shape)
    raise ValueError(kind)


def _same_info(g, o):
    g, o = np.asarray(g), np.asarray(o)
    assert np.array_equal(np.isnan(g), np.isnan(o)), (g, o)
    k = ~np.isnan(o)
    assert np.array_equal(g[k], o[k]), np.stack([g, o])[:, k]


@pytest.mark.parametrize("n", [33, 65, 129, 257])
@pytest.mark.parametrize("kind", ["diverted", "double_null", "limited", "diverted_perturbed", "noisy"])
def test_normalize_bitwise(torch_mod, efit, orc_mod, n, kind):
    torch = torch_mod
    cfg = synth.small_config(n)
    orc = orc_mod.Oracle.from_config(cfg)
    orc.set_steps_mode(1)
    psi = _psi(kind, cfg.grid)
    cnt, pa, pb, mask, _ = orc.normalize(psi)
    oinfo = orc.steps_info()
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=efit.EFIT_GREEN_TABLE_SYM)
    ctx.set_steps(efit.EFIT_STEPS_FULL)
    info, gmask = ctx.normalize(T(torch, psi))
    torch.cuda.synchronize()
    st = ctx.status()
    ginfo = info.cpu().numpy()
    if cnt < 0:
        assert st == efit.EFIT_E_NOPLASMA
    else:
        assert st == 0
        assert np.array_equal(gmask.cpu().numpy(), mask)
    _same_info(ginfo, oinfo)
    if kind in ("diverted", "diverted_perturbed") and n >= 65:
        assert ginfo[12] == 1.0  # lower X-point boundary
    ctx.close()


@pytest.mark.parametrize("shape", [(65, 129), (129, 65), (97, 65)], ids=["65x129", "129x65", "97x65"])
@pytest.mark.parametrize("sign", [1, -1], ids=["ip+", "ip-"])
def test_normalize_bitwise_nonsquare_and_sign(torch_mod, efit, orc_mod, shape, sign):
    """Ragged (non-square) grids and a negative plasma current (ip_sign = -1, psi minimal on the
    axis): the same bit-for-bit agreement (nh - 1 need not be a power of two for steps_ itself, but
    the context requires it, so nh is 65 or 129)."""
    import dataclasses
    torch = torch_mod
    g = synth.Grid(*shape)
    geo = dataclasses.replace(synth.make_geometry(g), ip_sign=sign)
    cfg = synth.Config("ns", g, geo, synth.poly_basis(), "non-square")
    orc = orc_mod.Oracle.from_config(cfg)
    orc.set_steps_mode(1)
    psi = sign * synth.solovev_diverted_psi(g)
    cnt, pa, pb, mask, _ = orc.normalize(psi)
    oinfo = orc.steps_info()
    ctx = efit.EfitContext(g, cfg.basis, geo, mode=efit.EFIT_GREEN_TABLE_SYM)
    ctx.set_steps(efit.EFIT_STEPS_FULL)
    info, gmask = ctx.normalize(T(torch, psi))
    torch.cuda.synchronize()
    assert ctx.status() == 0 and cnt > 0
    assert np.array_equal(gmask.cpu().numpy(), mask)
    _same_info(info.cpu().numpy(), oinfo)
    assert oinfo[12] == 1.0  # the lower X-point bounds the plasma for either sign
    ctx.close()


def test_minimum_grid_and_no_plasma(torch_mod, efit, orc_mod):
    """The smallest grid the full rule accepts (9 x 9, nh - 1 a power of two; rejected below 6) and a
    psi with no plasma (a plane: no interior maximum, no X-point): both sides report no plasma."""
    torch = torch_mod
    cfg = synth.small_config(9)
    orc = orc_mod.Oracle.from_config(cfg)
    orc.set_steps_mode(1)
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=efit.EFIT_GREEN_TABLE_SYM)
    ctx.set_steps(efit.EFIT_STEPS_FULL)
    psi = synth.solovev_diverted_psi(cfg.grid)
    cnt, pa, pb, mask, _ = orc.normalize(psi)
    info, gmask = ctx.normalize(T(torch, psi))
    torch.cuda.synchronize()
    st = ctx.status()
    assert (st == 0) == (cnt > 0)
    _same_info(info.cpu().numpy(), orc.steps_info())
    if cnt > 0:
        assert np.array_equal(gmask.cpu().numpy(), mask)
    R = np.repeat(cfg.grid.r(), cfg.grid.nh)
    plane = 0.01 * (R - R.mean())
    cnt, *_ = orc.normalize(plane)
    info, gmask = ctx.normalize(T(torch, plane))
    torch.cuda.synchronize()
    assert cnt < 0 and ctx.status() == efit.EFIT_E_NOPLASMA and int(gmask.sum().item()) == 0
    _same_info(info.cpu().numpy(), orc.steps_info())
    ctx.close()
    small = synth.small_config(5)
    ctx5 = efit.EfitContext(small.grid, small.basis, small.geometry, mode=efit.EFIT_GREEN_TABLE)
    with pytest.raises(efit.EfitError):
        ctx5.set_steps(efit.EFIT_STEPS_FULL)
    ctx5.close()


@pytest.mark.parametrize("kind", ["diverted", "diverted_perturbed"])
def test_c5_normalize_bitwise_global_bitmap(torch_mod, efit, orc_mod, kind):
    """1025^2 (C5): the candidate bitmap no longer fits in shared memory next to the component, so the
    flood fill reads it from global memory (k_steps_fill<false>); same bit-for-bit agreement.  An
    on-the-fly Green's context (no table to build): steps_ does not depend on the Green's mode."""
    torch = torch_mod
    cfg = synth.config("C5")
    orc = orc_mod.Oracle.from_config(cfg)
    orc.set_steps_mode(1)
    psi = _psi(kind, cfg.grid)
    cnt, pa, pb, mask, _ = orc.normalize(psi)
    oinfo = orc.steps_info()
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=efit.EFIT_GREEN_ONTHEFLY_SYM)
    ctx.set_steps(efit.EFIT_STEPS_FULL)
    info, gmask = ctx.normalize(T(torch, psi))
    torch.cuda.synchronize()
    assert ctx.status() == 0 and cnt > 0
    assert np.array_equal(gmask.cpu().numpy(), mask)
    _same_info(info.cpu().numpy(), oinfo)
    assert oinfo[12] == 1.0
    ctx.close()


def test_fit_host_full_steps_matches_device(torch_mod, efit, orc_mod):
    """The host-buffer pipeline (efit_fit_host) under the full steps_ rule equals efit_fit_steps on
    device buffers slice by slice, bit for bit (every iteration normalises under the rule)."""
    torch = torch_mod
    cfg = synth.small_config(129)
    orc = orc_mod.Oracle.from_config(cfg)
    orc.set_steps_mode(1)
    psi_s = synth.solovev_diverted_psi(cfg.grid)
    ct = synth.c_true(cfg.basis, sol_c=synth.DIV_C)
    tw = orc.twin(psi_s, ct, noise_seed=1)
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=efit.EFIT_GREEN_TABLE_SYM)
    ctx.set_steps(efit.EFIT_STEPS_FULL)
    S, iters, n, nb = 3, 2, cfg.grid.n, ctx.nbasis
    starts = [psi_s + 1e-4 * (k + 1) * (psi_s.max() - psi_s.min()) * synth.smooth_modes(cfg.grid, 5 + k) / 3.0
              for k in range(S)]
    ext = T(torch, tw["psi_ext"])
    h_psi0 = torch.tensor(np.concatenate(starts)).pin_memory()
    h_meas = torch.tensor(np.tile(tw["y"], S)).pin_memory()
    h_sig = torch.tensor(np.tile(tw["sigma"], S)).pin_memory()
    outs = [torch.empty(S * n, dtype=torch.float64).pin_memory(), torch.empty(S * nb, dtype=torch.float64).pin_memory(),
            torch.empty(S, dtype=torch.float64).pin_memory(), torch.empty(S, dtype=torch.float64).pin_memory()]
    st = torch.cuda.Stream()
    for _ in range(2):
        ctx.fit_host(S, iters, h_psi0, h_meas, h_sig, ext, *outs, stream=st)
        st.synchronize()
    assert ctx.status() == 0
    for k in range(S):
        psi = T(torch, starts[k])
        coef, chi2, eps = ctx._t(nb), ctx._t(1), ctx._t(1)
        ctx.fit_steps(iters, psi, ext, T(torch, tw["y"]), T(torch, tw["sigma"]), coef, chi2, eps)
        torch.cuda.synchronize()
        assert torch.equal(outs[0][k * n:(k + 1) * n], psi.cpu()), k
        assert torch.equal(outs[1][k * nb:(k + 1) * nb], coef.cpu()), k
    ctx.close()


def test_limiter_mode_normalize_matches_o8(torch_mod, efit, orc_mod):
    torch = torch_mod
    cfg = synth.small_config(65)
    orc = orc_mod.Oracle.from_config(cfg)
    for psi in (synth.solovev_psi(cfg.grid), synth.solovev_diverted_psi(cfg.grid)):
        cnt, pa, pb, mask, _ = orc.normalize(psi)
        ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=efit.EFIT_GREEN_TABLE_SYM)
        info, gmask = ctx.normalize(T(torch, psi))
        torch.cuda.synchronize()
        assert ctx.status() == 0
        ginfo = info.cpu().numpy()
        assert ginfo[0] == pa and ginfo[1] == pb and ginfo[12] == 0.0
        assert np.array_equal(gmask.cpu().numpy(), mask)
        ctx.close()


@pytest.mark.parametrize("n", [65, 129])
@pytest.mark.parametrize("mode", [2, 0], ids=["sym", "table"])
def test_fit_steps_full_steps(torch_mod, efit, orc_mod, n, mode):
    """Diverted twin, 1 and 3 chained iterations from a 1e-4 start (the diverted Picard loop is
    vertically unstable, DESIGN R4, so only a few iterations), vs or_fit_step in steps mode 1."""
    torch = torch_mod
    cfg = synth.small_config(n)
    orc = orc_mod.Oracle.from_config(cfg)
    orc.set_steps_mode(1)
    psi_s = synth.solovev_diverted_psi(cfg.grid)
    ct = synth.c_true(cfg.basis, sol_c=synth.DIV_C)
    tw = orc.twin(psi_s, ct, noise_seed=1)
    psi0 = psi_s + 1e-4 * (psi_s.max() - psi_s.min()) * synth.smooth_modes(cfg.grid, 5) / 3.0
    ref, p = [], psi0.copy()
    for _ in range(3):
        st, p, c, chi2, eps = orc.fit_step(p, tw["psi_ext"], tw["y"], tw["sigma"])
        assert st == 0
        ref.append((p.copy(), c.copy(), chi2, eps, orc.steps_info()))
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=mode)
    ctx.set_steps(efit.EFIT_STEPS_FULL)
    ext, y, s = T(torch, tw["psi_ext"]), T(torch, tw["y"]), T(torch, tw["sigma"])
    for k in (1, 3):
        psi = T(torch, psi0)
        coef, chi2, eps = ctx._t(ctx.nbasis), ctx._t(1), ctx._t(1)
        ctx.fit_steps(k, psi, ext, y, s, coef, chi2, eps)
        torch.cuda.synchronize()
        assert ctx.status() == 0
        pr, cr, chr_, er, _ = ref[k - 1]
        assert rel(psi.cpu().numpy(), pr) < TOL, (k, rel(psi.cpu().numpy(), pr))
        assert rel(coef.cpu().numpy(), cr) < TOL_C, (k, rel(coef.cpu().numpy(), cr))
        assert abs(chi2.item() - chr_) <= TOL_C * max(chr_, 1.0)
        assert abs(eps.item() - er) <= 1e-9 * er
    ctx.close()


def test_fit_step_twin_fixed_point(torch_mod, efit, orc_mod):
    """One full-steps_ iteration from the diverted psi_S returns psi_S and c_true."""
    torch = torch_mod
    cfg = synth.small_config(129)
    orc = orc_mod.Oracle.from_config(cfg)
    orc.set_steps_mode(1)
    psi_s = synth.solovev_diverted_psi(cfg.grid)
    ct = synth.c_true(cfg.basis, sol_c=synth.DIV_C)
    tw = orc.twin(psi_s, ct)
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=efit.EFIT_GREEN_TABLE_SYM)
    ctx.set_steps(efit.EFIT_STEPS_FULL)
    psi = T(torch, psi_s)
    coef, chi2, eps = ctx._t(ctx.nbasis), ctx._t(1), ctx._t(1)
    ctx.fit_step(psi, T(torch, tw["psi_ext"]), T(torch, tw["y"]), T(torch, tw["sigma"]), coef, chi2, eps)
    torch.cuda.synchronize()
    assert ctx.status() == 0
    assert rel(psi.cpu().numpy(), psi_s) < 1e-13
    assert rel(coef.cpu().numpy(), ct) < TOL_C
    assert eps.item() < 1e-12
    ctx.close()


def test_c4_full_steps_fit_step(torch_mod, efit, orc_mod):
    """The benched size (513^2, SYM mode): normalisation bit for bit and one fit step vs the oracle."""
    torch = torch_mod
    cfg = synth.config("C4")
    orc = orc_mod.Oracle.from_config(cfg)
    orc.set_steps_mode(1)
    psi_s = synth.solovev_diverted_psi(cfg.grid)
    ct = synth.c_true(cfg.basis, sol_c=synth.DIV_C)
    tw = orc.twin(psi_s, ct, noise_seed=1)
    psi0 = psi_s + 1e-4 * (psi_s.max() - psi_s.min()) * synth.smooth_modes(cfg.grid, 5) / 3.0
    cnt, pa, pb, mask, _ = orc.normalize(psi0)
    oinfo = orc.steps_info()
    st, pr, cr, chr_, er = orc.fit_step(psi0, tw["psi_ext"], tw["y"], tw["sigma"])
    assert st == 0
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=efit.EFIT_GREEN_TABLE_SYM)
    ctx.set_steps(efit.EFIT_STEPS_FULL)
    info, gmask = ctx.normalize(T(torch, psi0))
    torch.cuda.synchronize()
    assert ctx.status() == 0
    _same_info(info.cpu().numpy(), oinfo)
    assert np.array_equal(gmask.cpu().numpy(), mask)
    psi = T(torch, psi0)
    coef, chi2, eps = ctx._t(ctx.nbasis), ctx._t(1), ctx._t(1)
    ctx.fit_steps(1, psi, T(torch, tw["psi_ext"]), T(torch, tw["y"]), T(torch, tw["sigma"]), coef, chi2, eps)
    torch.cuda.synchronize()
    assert ctx.status() == 0
    assert rel(psi.cpu().numpy(), pr) < TOL
    assert rel(coef.cpu().numpy(), cr) < TOL_C
    assert abs(eps.item() - er) <= 1e-9 * er
    ctx.close()


def test_steps_mode_switch_and_errors(torch_mod, efit, orc_mod):
    """Switching the rule drops the cached graphs (the same pointers give the other rule's result);
    bad modes are rejected on the host."""
    torch = torch_mod
    cfg = synth.small_config(65)
    orc = orc_mod.Oracle.from_config(cfg)
    psi_s = synth.solovev_diverted_psi(cfg.grid)
    ct = synth.c_true(cfg.basis, sol_c=synth.DIV_C)
    orc.set_steps_mode(1)
    tw = orc.twin(psi_s, ct)
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=efit.EFIT_GREEN_TABLE)
    ext, y, s = T(torch, tw["psi_ext"]), T(torch, tw["y"]), T(torch, tw["sigma"])
    coef, chi2, eps = ctx._t(ctx.nbasis), ctx._t(1), ctx._t(1)
    psi = T(torch, psi_s)
    results = []
    for m in (efit.EFIT_STEPS_FULL, efit.EFIT_STEPS_LIMITER, efit.EFIT_STEPS_FULL):
        ctx.set_steps(m)
        psi.copy_(T(torch, psi_s))
        ctx.fit_step(psi, ext, y, s, coef, chi2, eps)
        torch.cuda.synchronize()
        ctx.status()
        results.append(psi.cpu().numpy().copy())
    for m, r in zip((1, 0, 1), results):
        orc.set_steps_mode(m)
        st, pr, *_ = orc.fit_step(psi_s, tw["psi_ext"], tw["y"], tw["sigma"])
        assert rel(r, pr) < TOL
    assert rel(results[0], results[1]) > 1e-6  # the two rules differ on a diverted psi
    with pytest.raises(efit.EfitError):
        ctx.set_steps(7)
    ctx.close()


def test_batch_full_steps_per_slice(torch_mod, efit, orc_mod):
    """A batch of 3 time slices (shared table pass on the tensor cores) under the full steps_ rule:
    every slice normalises its own psi (axis, X-point, connected mask) and equals the oracle's f3
    fit step on that slice (the table pass sums in another order: rounding-level agreement)."""
    torch = torch_mod
    cfg = synth.small_config(65)
    orc = orc_mod.Oracle.from_config(cfg)
    orc.set_steps_mode(1)
    psi_s = synth.solovev_diverted_psi(cfg.grid)
    ct = synth.c_true(cfg.basis, sol_c=synth.DIV_C)
    tw = orc.twin(psi_s, ct, noise_seed=1)
    S, n = 3, cfg.grid.n
    starts = [psi_s + 1e-4 * (k + 1) * (psi_s.max() - psi_s.min()) * synth.smooth_modes(cfg.grid, 5 + k) / 3.0
              for k in range(S)]
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=efit.EFIT_GREEN_TABLE)
    ctx.batch_attach(S)
    ctx.set_steps(efit.EFIT_STEPS_FULL)  # after attaching: propagated to the slices
    P = T(torch, np.concatenate(starts))
    E = T(torch, np.tile(tw["psi_ext"], S))
    Y = T(torch, np.tile(tw["y"], S))
    G = T(torch, np.tile(tw["sigma"], S))
    coef, chi2, eps = ctx._t(S * ctx.nbasis), ctx._t(S), ctx._t(S)
    st = torch.cuda.Stream()
    ctx.fit_step_batch(P, E, Y, G, coef, chi2, eps, stream=st)
    st.synchronize()
    assert ctx.status() == 0
    Pg, Cg = P.cpu().numpy(), coef.cpu().numpy()
    for k in range(S):
        s0, pr, cr, chr_, er = orc.fit_step(starts[k], tw["psi_ext"], tw["y"], tw["sigma"])
        assert s0 == 0
        assert rel(Pg[k * n:(k + 1) * n], pr) < TOL, k
        assert rel(Cg[k * ctx.nbasis:(k + 1) * ctx.nbasis], cr) < TOL_C, k
    ctx.close()


def test_nonfinite_psi_reports_status(torch_mod, efit):
    torch = torch_mod
    cfg = synth.small_config(33)
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=efit.EFIT_GREEN_TABLE_SYM)
    ctx.set_steps(efit.EFIT_STEPS_FULL)
    psi = synth.solovev_diverted_psi(cfg.grid)
    psi[200] = np.nan
    ctx.normalize(T(torch, psi))
    torch.cuda.synchronize()
    assert ctx.status() == efit.EFIT_E_NONFINITE
    # the flag does not stick: a finite psi afterwards normalises cleanly
    info, _ = ctx.normalize(T(torch, synth.solovev_diverted_psi(cfg.grid)))
    torch.cuda.synchronize()
    assert ctx.status() == 0 and info.cpu().numpy()[12] == 1.0
    ctx.close()
