"""GPU parity of the multi-time-slice batch (include/efit.h efit_batch_*):
S slices share one pass over the top/bottom Green's table (k_bnd_tb_mma, FP64 tensor cores).
Every slice is compared with the CPU oracle on that slice's own seeded inputs (1e-12 relative;
1e-10 on coefficients and chi2), at sizes that span several chunks and a ragged tail, plus
sampled targets at the full C4 size."""
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


def cfg_of(name):
    if name.startswith("C"):
        return synth.config(name)
    nw, nh = (int(x) for x in name.split("x"))
    g = synth.Grid(nw, nh)
    return synth.Config(name, g, synth.make_geometry(g, 0), synth.poly_basis(), name)


_ctx = {}


def setup(name, efit, oracle, mode=0):
    if (name, mode) not in _ctx:
        cfg = cfg_of(name)
        _ctx[(name, mode)] = (cfg, oracle.Oracle.from_config(cfg),
                              efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=mode))
    return _ctx[(name, mode)]


def slice_currents(grid, S):
    # alternate positive / signed currents so cancellation is exercised in some columns
    return [synth.random_current(grid, seed=20 + k, signed=bool(k % 2)) for k in range(S)]


@pytest.mark.parametrize("name", ["9x9", "33x33", "40x33", "65x65", "C2"])
@pytest.mark.parametrize("S", [1, 2, 3, 4, 5, 8])
def test_batch_boundary_flux(torch_mod, efit, orc_mod, name, S):
    torch = torch_mod
    cfg, orc, ctx = setup(name, efit, orc_mod)
    ctx.batch_attach(S)
    Is = slice_currents(cfg.grid, S)
    st = torch.cuda.Stream()
    with torch.cuda.stream(st):
        out = ctx.boundary_flux_batch(T(torch, np.stack(Is)), stream=st)
    st.synchronize()
    out = out.cpu().numpy()
    for k in range(S):
        ref = orc.boundary(Is[k])
        assert rel(out[k], ref) < TOL, (k, rel(out[k], ref))


def _twin(orc, cfg, noise_seed):
    psi_s = synth.solovev_psi(cfg.grid)
    ct = synth.c_true(cfg.basis)
    return orc.twin(psi_s, ct, noise_seed=noise_seed)


def _slices(orc, cfg, S):
    """Slice k: same machine and external flux, its own noise draw (seed 1+k) and its own start
    perturbation (seed 5+k): independent fits as EFIT's time slices are."""
    tws = [_twin(orc, cfg, 1 + k) for k in range(S)]
    psi0 = [synth.perturbed_psi(cfg.grid, seed=5 + k, rel=1e-3) for k in range(S)]
    return tws, psi0


@pytest.mark.parametrize("name", ["33x33", "C1", "C2"])
@pytest.mark.parametrize("S", [1, 3, 4, 8])
def test_batch_fit_step(torch_mod, efit, orc_mod, name, S):
    torch = torch_mod
    cfg, orc, ctx = setup(name, efit, orc_mod)
    ctx.batch_attach(S)
    tws, psi0 = _slices(orc, cfg, S)
    psi = T(torch, np.stack(psi0))
    ext = T(torch, np.stack([tw["psi_ext"] for tw in tws]))
    y = T(torch, np.stack([tw["y"] for tw in tws]))
    sg = T(torch, np.stack([tw["sigma"] for tw in tws]))
    coef, chi2, eps = ctx._t(S * ctx.nbasis), ctx._t(S), ctx._t(S)
    st = torch.cuda.Stream()
    with torch.cuda.stream(st):
        ctx.fit_step_batch(psi, ext, y, sg, coef, chi2, eps, stream=st)
    st.synchronize()
    assert ctx.status() == 0
    psi_g, coef_g = psi.cpu().numpy(), coef.cpu().numpy().reshape(S, -1)
    for k in range(S):
        ok, psi_r, c_r, chi2_r, eps_r = orc.fit_step(psi0[k], tws[k]["psi_ext"], tws[k]["y"], tws[k]["sigma"])
        assert ok == 0
        assert rel(psi_g[k], psi_r) < TOL, (k, rel(psi_g[k], psi_r))
        assert rel(coef_g[k], c_r) < TOL_C
        assert abs(chi2[k].item() - chi2_r) <= TOL_C * max(chi2_r, 1.0)
        assert abs(eps[k].item() - eps_r) <= 1e-9 * eps_r


def test_batch_chained_equals_repeated(torch_mod, efit, orc_mod):
    """efit_fit_steps_batch(n) is bitwise n efit_fit_step_batch calls (as for one slice)."""
    torch = torch_mod
    cfg, orc, ctx = setup("C2", efit, orc_mod)
    S = 3
    ctx.batch_attach(S)
    tws, psi0 = _slices(orc, cfg, S)
    ext = T(torch, np.stack([tw["psi_ext"] for tw in tws]))
    y = T(torch, np.stack([tw["y"] for tw in tws]))
    sg = T(torch, np.stack([tw["sigma"] for tw in tws]))
    outs = []
    st = torch.cuda.Stream()
    for chained in (False, True):
        psi = T(torch, np.stack(psi0))
        coef, chi2, eps = ctx._t(S * ctx.nbasis), ctx._t(S), ctx._t(S)
        with torch.cuda.stream(st):
            if chained:
                ctx.fit_steps_batch(4, psi, ext, y, sg, coef, chi2, eps, stream=st)
            else:
                for _ in range(4):
                    ctx.fit_step_batch(psi, ext, y, sg, coef, chi2, eps, stream=st)
        st.synchronize()
        assert ctx.status() == 0
        outs.append((psi.clone(), coef.clone(), eps.clone()))
    for a, b in zip(*outs):
        assert torch.equal(a, b)


def test_batch_matches_single_slice_calls(torch_mod, efit, orc_mod):
    """Each batched slice equals efit_fit_step on that slice alone to rounding (the shared table
    pass sums in another order), and replaying the batch is deterministic."""
    torch = torch_mod
    cfg, orc, ctx = setup("C2", efit, orc_mod)
    S = 4
    ctx.batch_attach(S)
    tws, psi0 = _slices(orc, cfg, S)
    ext = T(torch, np.stack([tw["psi_ext"] for tw in tws]))
    y = T(torch, np.stack([tw["y"] for tw in tws]))
    sg = T(torch, np.stack([tw["sigma"] for tw in tws]))
    st = torch.cuda.Stream()
    res = []
    for _ in range(2):
        psi = T(torch, np.stack(psi0))
        coef, chi2, eps = ctx._t(S * ctx.nbasis), ctx._t(S), ctx._t(S)
        with torch.cuda.stream(st):
            ctx.fit_steps_batch(3, psi, ext, y, sg, coef, chi2, eps, stream=st)
        st.synchronize()
        res.append(psi.clone())
    assert torch.equal(res[0], res[1])
    for k in range(S):
        p1 = T(torch, psi0[k])
        c1, x1, e1 = ctx._t(ctx.nbasis), ctx._t(1), ctx._t(1)
        ctx.fit_steps(3, p1, ext[k].clone(), y[k].clone(), sg[k].clone(), c1, x1, e1)  # 16-B aligned copies
        torch.cuda.synchronize()
        assert rel(res[0][k].cpu().numpy(), p1.cpu().numpy()) < 1e-13


def test_batch_errors(torch_mod, efit, orc_mod):
    torch = torch_mod
    cfg, orc, ctx = setup("33x33", efit, orc_mod)
    for bad in (0, 9):
        with pytest.raises(efit.EfitError) as ei:
            efit.efit_batch_workspace_bytes(ctx.handle, bad)
        assert ei.value.code == efit.EFIT_E_INVAL
    cfg2, orc2, ctx2 = setup("33x33", efit, orc_mod, mode=efit.EFIT_GREEN_TABLE_SYM)
    with pytest.raises(efit.EfitError) as ei:
        ctx2.batch_attach(2)
    assert ei.value.code == efit.EFIT_E_STATE
    x = ctx2._t(ctx2.nw * ctx2.nh * 2)
    with pytest.raises(efit.EfitError) as ei:  # no batch attached
        efit.efit_fit_step_batch(ctx2.handle, x, x, x, x, x, x, x, stream=torch.cuda.Stream())
    assert ei.value.code == efit.EFIT_E_STATE
    small = torch.empty(256, dtype=torch.uint8, device="cuda")
    with pytest.raises(efit.EfitError) as ei:
        efit.efit_batch_attach(ctx.handle, 2, small)
    assert ei.value.code == efit.EFIT_E_NOMEM


def test_c4_batch_boundary_sampled(torch_mod, efit, orc_mod):
    """Full size (513^2), 4 slices through the launch configuration bench.py --slices 4 times."""
    torch = torch_mod
    cfg, orc, ctx = setup("C4", efit, orc_mod)
    S = 4
    ctx.batch_attach(S)
    Is = slice_currents(cfg.grid, S)
    st = torch.cuda.Stream()
    with torch.cuda.stream(st):
        out = ctx.boundary_flux_batch(T(torch, np.stack(Is)), stream=st)
    st.synchronize()
    out = out.cpu().numpy()
    rng = np.random.default_rng(0)
    tg = np.unique(np.concatenate([[0, 512, 513, 1025, 1026, 1536, 2043], rng.integers(0, ctx.n_edge, 24)]))
    for k in range(S):
        ref = orc.boundary_targets(Is[k], tg)
        assert rel(out[k][tg], ref) < TOL, (k, rel(out[k][tg], ref))


@pytest.mark.parametrize("name", ["33x33", "40x33", "C1", "C2"])
def test_boundary_basis(torch_mod, efit, orc_mod, name):
    """the boundary flux of every basis current (efit_boundary_basis) equals the
    oracle's boundary flux of the current with c = e_k, and sum_k c_k R_b[k] equals the paper-order
    path boundary_flux(current(psi, c)) (linearity)."""
    torch = torch_mod
    cfg, orc, ctx = setup(name, efit, orc_mod)
    nb = ctx.nbasis
    ctx.batch_attach(nb)
    psi0 = synth.perturbed_psi(cfg.grid, seed=5, rel=1e-3)
    st = torch.cuda.Stream()
    with torch.cuda.stream(st):
        rb = ctx.boundary_basis(T(torch, psi0), stream=st)
    st.synchronize()
    assert ctx.status() == 0
    rb = rb.cpu().numpy()
    for k in range(nb):
        e = np.zeros(nb)
        e[k] = 1.0
        ref = orc.boundary(orc.current(psi0, e))
        assert rel(rb[k], ref) < TOL, (k, rel(rb[k], ref))
    c = synth.c_true(cfg.basis)
    direct = ctx.boundary_flux(ctx.current(T(torch, psi0), T(torch, c))).cpu().numpy()
    assert rel(c @ rb, direct) < TOL


def test_boundary_basis_needs_batch(torch_mod, efit, orc_mod):
    torch = torch_mod
    cfg, orc, ctx = setup("9x9", efit, orc_mod)
    ctx.batch_attach(1)
    with pytest.raises(efit.EfitError) as ei:
        ctx.boundary_basis(T(torch, synth.perturbed_psi(cfg.grid, seed=5, rel=1e-3)), stream=torch.cuda.Stream())
    assert ei.value.code == efit.EFIT_E_STATE


def test_batch_slice_status_isolated(torch_mod, efit, orc_mod):
    """Every slice has its own status word: a slice without plasma (psi = 0: empty mask, e.g. a
    pre-plasma time slice) gets NaN results and makes efit_status report EFIT_E_NOPLASMA naming
    it, while the healthy slices' results are unaffected (equal the oracle's fit step)."""
    torch = torch_mod
    cfg, orc, ctx = setup("33x33", efit, orc_mod)
    S = 3
    ctx.batch_attach(S)
    tws, psi0 = _slices(orc, cfg, S)
    psi0 = [p.copy() for p in psi0]
    psi0[1][:] = 0.0
    psi = T(torch, np.stack(psi0))
    ext = T(torch, np.stack([tw["psi_ext"] for tw in tws]))
    y = T(torch, np.stack([tw["y"] for tw in tws]))
    sg = T(torch, np.stack([tw["sigma"] for tw in tws]))
    coef, chi2, eps = ctx._t(S * ctx.nbasis), ctx._t(S), ctx._t(S)
    st = torch.cuda.Stream()
    for _ in range(2):   # twice: the failing slice's sticky bit must not leak into the next call
        p = psi.clone()
        with torch.cuda.stream(st):
            ctx.fit_step_batch(p, ext, y, sg, coef, chi2, eps, stream=st)
        st.synchronize()
        cg = coef.cpu().numpy().reshape(S, -1)
        assert np.all(np.isnan(cg[1]))
        for k in (0, 2):
            ok, psi_r, c_r, chi2_r, eps_r = orc.fit_step(psi0[k], tws[k]["psi_ext"], tws[k]["y"], tws[k]["sigma"])
            assert rel(p.cpu().numpy()[k], psi_r) < TOL
            assert rel(cg[k], c_r) < TOL_C
    # the failing slice's own word: empty mask (and the NaN psi it then produces)
    assert ctx.status() in (efit.EFIT_E_NOPLASMA, efit.EFIT_E_NONFINITE)
    assert "slice 1" in efit.efit_last_error(ctx.handle)
    assert ctx.status() == 0


@pytest.mark.parametrize("nb", [5, 10])
@pytest.mark.parametrize("cond", [1e6, 1e10, 1e12])
def test_lsq_ill_conditioned_fallback(torch_mod, efit, orc_mod, nb, cond):
    """Beyond cond ~ 1e8 CholeskyQR2 breaks down; the kernels fall back to shifted CholeskyQR3
    (k_lsq_warp for nb <= 6, k_lsq<NB> above).  Against the oracle's Householder QR on a matrix
    with prescribed singular values: coefficients and chi2 to max(1e-10, 50 cond u), the
    backward-stable bound."""
    torch = torch_mod
    basis = synth.poly_basis(2, 3) if nb == 5 else synth.poly_basis(5, 5)
    g = synth.Grid(33, 33)
    cfg = synth.Config("lsq", g, synth.make_geometry(g, 0), basis, "lsq")
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=0)
    nd = ctx.ndiag
    rng = np.random.default_rng(int(np.log10(cond)) + nb)
    U, _ = np.linalg.qr(rng.standard_normal((nd, nb)))
    V, _ = np.linalg.qr(rng.standard_normal((nb, nb)))
    A = U @ np.diag(np.logspace(0, -np.log10(cond), nb)) @ V.T
    A = A * rng.uniform(0.5, 2.0, nb)[None, :]   # unequal column scales
    x = rng.standard_normal(nb)
    sigma = rng.uniform(0.5, 1.5, nd)
    y = A @ x + 1e-3 * sigma * rng.standard_normal(nd)
    st, cref, chi2ref = orc_mod.lsq(A, y, sigma)
    assert st == 0
    coef, chi2 = ctx.lsq(T(torch, A), T(torch, y), T(torch, sigma))
    assert ctx.status() == 0
    tol = max(1e-10, 50 * cond * 2.0 ** -53)
    assert rel(coef.cpu().numpy(), cref) < tol, rel(coef.cpu().numpy(), cref)
    # the residual's sensitivity to a backward error u|A| is ~ cond * |r| (Higham Thm 20.1)
    assert abs(chi2.item() - chi2ref) <= tol * chi2ref
    ctx.close()
