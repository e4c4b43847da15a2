"""GPU parity: every ABI call of libefit_b200.so against the CPU oracle on the same seeded
synthetic inputs (BASELINE.json north_star: 1e-12 relative, 1e-10 on coefficients and chi2).

Metric: normwise  max|gpu - oracle| / max|oracle|  over the compared array (per column for
the response, whose P' and FF' columns differ by ~1e-8 in scale).  Integer/bit decisions
(in-limiter flags, plasma mask, axis value) must match exactly."""
import math
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


class Case:
    def __init__(self, cfg, efit, oracle, mode=0):
        self.cfg = cfg
        self.orc = oracle.Oracle.from_config(cfg)
        self.ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=mode)


_cases = {}


def case(name, efit, oracle, mode=0, basis=None, n_int=0):
    key = (name, mode, None if basis is None else (basis.kind, basis.n_pp, basis.n_ff), n_int)
    if key not in _cases:
        if name.startswith("C"):
            cfg = synth.config(name)
        else:
            nw, nh = (int(x) for x in name.split("x"))
            g = synth.Grid(nw, nh)
            cfg = synth.Config(name, g, synth.make_geometry(g, n_int), basis or synth.poly_basis(), name)
        _cases[key] = Case(cfg, efit, oracle, mode)
    return _cases[key]


SMALL = ["33x33", "40x33", "65x65", "C1"]


# ------------------------------------------------------------------ a0: tables

@pytest.mark.parametrize("name", ["9x9", "33x33", "40x33", "65x65"])
def test_green_tables(torch_mod, efit, orc_mod, name):
    torch = torch_mod
    c = case(name, efit, orc_mod)
    nw, nh = c.cfg.grid.nw, c.cfg.grid.nh
    S = c.ctx.info.slab_stride
    Tref = c.orc.table_T()  # [i][ii][m]
    nslab = c.ctx.info.bnd_row_hi - c.ctx.info.bnd_row_lo
    # top/bottom slabs i = 1..nw-2 and the edge slabs i = 0, nw-1
    tb = _device_view(torch, c.ctx.table_ptr(0), nslab * S).view(nslab, S)[:, : nw * nh].cpu().numpy()
    edge = _device_view(torch, c.ctx.table_ptr(3), 2 * S).view(2, S)[:, : nw * nh].cpu().numpy()
    ref_tb = Tref[1:nw - 1].reshape(nw - 2, nw * nh)
    assert rel(tb, ref_tb) < 1e-13
    assert rel(edge[0], Tref[0].reshape(-1)) < 1e-13 and rel(edge[1], Tref[nw - 1].reshape(-1)) < 1e-13
    # per-entry relative error (far-field entries are small): < 1e-13 of each entry
    assert np.max(np.abs(tb - ref_tb) / np.abs(ref_tb)) < 1e-12
    Gd = _device_view(torch, c.ctx.table_ptr(1), c.ctx.ndiag * S).view(c.ctx.ndiag, S)[:, : nw * nh].cpu().numpy()
    Gref = c.orc.table_Gd()
    for m in range(c.ctx.ndiag):
        assert rel(Gd[m], Gref[m]) < 1e-12, m
    inl = _device_view(torch, c.ctx.table_ptr(2), nw * nh, dtype=torch.uint8).cpu().numpy()
    assert np.array_equal(inl, c.orc.inlim())


def _device_view(torch, ptr, count, dtype=None):
    """Copy `count` elements from a raw device pointer into a new tensor (test helper)."""
    import ctypes
    dtype = dtype or torch.float64
    out = torch.empty(count, dtype=dtype, device="cuda")
    cudart = ctypes.CDLL("libcudart.so.12") if _CUDART[0] is None else _CUDART[0]
    _CUDART[0] = cudart
    nbytes = count * out.element_size()
    torch.cuda.synchronize()
    err = cudart.cudaMemcpy(ctypes.c_void_p(out.data_ptr()), ctypes.c_void_p(ptr), ctypes.c_size_t(nbytes), 3)
    assert err == 0, f"cudaMemcpy failed {err}"
    return out


_CUDART = [None]


# ------------------------------------------------------------------ a1-a3: response

@pytest.mark.parametrize("name", SMALL + ["C2"])
def test_response(torch_mod, efit, orc_mod, name):
    torch = torch_mod
    c = case(name, efit, orc_mod)
    psi = synth.perturbed_psi(c.cfg.grid, seed=5, rel=1e-3)
    ref, axbd_ref = c.orc.response(psi)
    resp, axbd = c.ctx.response(T(torch, psi))
    torch.cuda.synchronize()
    assert c.ctx.status() == 0
    assert np.array_equal(axbd.cpu().numpy(), axbd_ref)  # same decisions, same formula
    r = resp.cpu().numpy()
    for k in range(c.ctx.nbasis):
        assert rel(r[:, k], ref[:, k]) < TOL, (k, rel(r[:, k], ref[:, k]))


def test_response_spline_mse(torch_mod, efit, orc_mod):
    """C3 ingredients on a smaller grid: 10+10 cubic B-spline basis + 40 MSE-like B_Z rows."""
    torch = torch_mod
    c = case("129x129", efit, orc_mod, basis=synth.spline_basis(6), n_int=40)
    assert c.ctx.ndiag == 160 and c.ctx.nbasis == 20
    psi = synth.perturbed_psi(c.cfg.grid, seed=5, rel=1e-3)
    ref, axbd_ref = c.orc.response(psi)
    resp, axbd = c.ctx.response(T(torch, psi))
    r = resp.cpu().numpy()
    for k in range(20):
        assert rel(r[:, k], ref[:, k]) < TOL, k


@pytest.mark.parametrize("force", ["0", "1"])
@pytest.mark.parametrize("name,spline", [("65x65", False), ("129x129", True), ("129x129", False)])
def test_response_kernel_choice(torch_mod, efit, orc_mod, monkeypatch, name, spline, force):
    """Both single-slice response kernels (scalar stream k_response, EFIT_RESP_MMA=0; DMMA
    k_response_mma, =1) against the oracle, whatever the automatic choice for the grid/basis."""
    torch = torch_mod
    monkeypatch.setenv("EFIT_RESP_MMA", force)
    nw = int(name.split("x")[0])
    g = synth.Grid(nw, nw)
    basis = synth.spline_basis(6) if spline else synth.poly_basis()
    n_int = 40 if spline else 0
    cfg = synth.Config(name, g, synth.make_geometry(g, n_int), basis, name)
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=0)
    orc = orc_mod.Oracle.from_config(cfg)
    psi = synth.perturbed_psi(g, seed=7, rel=1e-3)
    ref, axbd_ref = orc.response(psi)
    resp, axbd = ctx.response(T(torch, psi))
    torch.cuda.synchronize()
    assert ctx.status() == 0
    assert np.array_equal(axbd.cpu().numpy(), axbd_ref)
    r = resp.cpu().numpy()
    for k in range(ctx.nbasis):
        assert rel(r[:, k], ref[:, k]) < TOL, (k, rel(r[:, k], ref[:, k]))


# ------------------------------------------------------------------ a5: current

@pytest.mark.parametrize("name", SMALL)
def test_current(torch_mod, efit, orc_mod, name):
    torch = torch_mod
    c = case(name, efit, orc_mod)
    psi = synth.perturbed_psi(c.cfg.grid, seed=5, rel=1e-3)
    coef = synth.c_true(c.cfg.basis)
    ref = c.orc.current(psi, coef)
    out = c.ctx.current(T(torch, psi), T(torch, coef)).cpu().numpy()
    assert np.array_equal(out != 0, ref != 0)   # identical plasma mask
    assert rel(out, ref) < TOL


# ------------------------------------------------------------------ a6: boundary flux

@pytest.mark.parametrize("name", ["9x9", "33x33", "40x33", "65x65", "C2", "21x1025"])
@pytest.mark.parametrize("signed", [False, True])
@pytest.mark.parametrize("mode", [0, 2])  # EFIT_GREEN_TABLE, EFIT_GREEN_TABLE_SYM (21x1025: m-chunked path)
def test_boundary_flux(torch_mod, efit, orc_mod, name, signed, mode):
    torch = torch_mod
    c = case(name, efit, orc_mod, mode=mode)
    I = synth.random_current(c.cfg.grid, seed=3 if signed else 2, signed=signed)
    ref = c.orc.boundary(I)
    out = c.ctx.boundary_flux(T(torch, I)).cpu().numpy()
    assert rel(out, ref) < TOL, rel(out, ref)


@pytest.mark.parametrize("name", ["9x9", "33x33", "40x33", "21x1025"])
@pytest.mark.parametrize("mode", [0, 2, 3])
def test_boundary_flux_edge_sources(torch_mod, efit, orc_mod, name, mode):
    """Current on every node, the edge ring included: the edge-row sources (ii = 0, nw-1; in SYM
    mode taken from the edge slabs by reciprocity) and the self terms of edge targets."""
    torch = torch_mod
    c = case(name, efit, orc_mod, mode=mode)
    I = synth.random_current(c.cfg.grid, seed=6, signed=True, edge=True)
    ref = c.orc.boundary(I)
    out = c.ctx.boundary_flux(T(torch, I)).cpu().numpy()
    assert rel(out, ref) < TOL, rel(out, ref)


@pytest.mark.parametrize("name", ["9x9", "33x33", "40x33", "65x65"])
def test_green_sym_table(torch_mod, efit, orc_mod, name):
    """SYM half table (include/efit.h, efit_table which = 4): tile t = Q(Q+1)/2 + P, entry
    [p][m][q] = T[1+8P+p][1+8Q+q][m] of the oracle's table, 0 outside the interior rows."""
    torch = torch_mod
    c = case(name, efit, orc_mod, mode=efit.EFIT_GREEN_TABLE_SYM)
    nw, nh = c.cfg.grid.nw, c.cfg.grid.nh
    ni = nw - 2
    nblk = c.ctx.info.sym_nblk
    assert nblk == (ni + 7) // 8
    ntile = nblk * (nblk + 1) // 2
    assert (c.ctx.info.sym_tile_lo, c.ctx.info.sym_tile_hi) == (0, ntile)
    U = _device_view(torch, c.ctx.table_ptr(4), ntile * 64 * nh).view(ntile, 8, nh, 8).cpu().numpy()
    Tref = c.orc.table_T()
    ref = np.zeros_like(U)
    t = 0
    for Q in range(nblk):
        for P in range(Q + 1):
            for p in range(8):
                for q in range(8):
                    rp, rq = 8 * P + p, 8 * Q + q
                    if rp < ni and rq < ni:
                        ref[t, p, :, q] = Tref[1 + rp, 1 + rq, :]
            t += 1
    nz = ref != 0
    assert np.array_equal(U != 0, nz)
    assert np.max(np.abs(U[nz] - ref[nz]) / np.abs(ref[nz])) < 1e-12


def test_boundary_sym_onthefly_bitwise(torch_mod, efit, orc_mod):
    torch = torch_mod
    a = case("65x65", efit, orc_mod, mode=efit.EFIT_GREEN_TABLE_SYM)
    b = case("65x65", efit, orc_mod, mode=efit.EFIT_GREEN_ONTHEFLY_SYM)
    I = T(torch, synth.random_current(a.cfg.grid, seed=3, signed=True, edge=True))
    assert torch.equal(a.ctx.boundary_flux(I), b.ctx.boundary_flux(I))


def test_boundary_sym_matches_full_table(torch_mod, efit, orc_mod):
    """Reciprocity: the half-table nest equals the full-table nest to rounding."""
    torch = torch_mod
    a = case("C2", efit, orc_mod)
    b = case("C2", efit, orc_mod, mode=efit.EFIT_GREEN_TABLE_SYM)
    I = T(torch, synth.random_current(a.cfg.grid, seed=2))
    x, y = a.ctx.boundary_flux(I).cpu().numpy(), b.ctx.boundary_flux(I).cpu().numpy()
    assert rel(y, x) < 1e-14


def test_boundary_literal_fig2(torch_mod, efit, orc_mod):
    """The GPU boundary equals minus the paper's Fig. 2/3 loops transcribed literally."""
    torch = torch_mod
    c = case("33x33", efit, orc_mod)
    I = synth.random_current(c.cfg.grid, seed=4)
    lit = c.orc.pflux_literal(I)
    out = c.ctx.boundary_flux(T(torch, I)).cpu().numpy()
    nh = c.cfg.grid.nh
    ref = np.array([-lit[i * nh + j] for i, j in c.orc.edge_nodes()])
    assert rel(out, ref) < TOL


def test_boundary_onthefly_bitwise(torch_mod, efit, orc_mod):
    torch = torch_mod
    a = case("65x65", efit, orc_mod)
    b = case("65x65", efit, orc_mod, mode=efit.EFIT_GREEN_ONTHEFLY)
    I = T(torch, synth.random_current(a.cfg.grid, seed=2))
    assert torch.equal(a.ctx.boundary_flux(I), b.ctx.boundary_flux(I))


def test_boundary_deterministic(torch_mod, efit, orc_mod):
    torch = torch_mod
    c = case("65x65", efit, orc_mod)
    I = T(torch, synth.random_current(c.cfg.grid, seed=3, signed=True))
    x = [c.ctx.boundary_flux(I) for _ in range(3)]
    assert torch.equal(x[0], x[1]) and torch.equal(x[1], x[2])


# ------------------------------------------------------------------ a7: interior solve

@pytest.mark.parametrize("name", ["9x9", "33x33", "40x33", "65x65", "C2"])
def test_interior_solve(torch_mod, efit, orc_mod, name):
    torch = torch_mod
    c = case(name, efit, orc_mod)
    I = synth.random_current(c.cfg.grid, seed=2)
    psib = c.orc.boundary(I)
    ref = c.orc.interior_solve(I, psib)
    out = c.ctx.interior_solve(T(torch, I), T(torch, psib)).cpu().numpy()
    assert rel(out, ref) < TOL, rel(out, ref)


def test_interior_solve_solovev_exact(torch_mod, efit, orc_mod):
    """Exact discrete Solov'ev identity: the GPU solve reproduces psi_S (independent of the oracle)."""
    torch = torch_mod
    c = case("65x65", efit, orc_mod)
    g = c.cfg.grid
    A, B, C, R0 = 1.2346, 1.0, 0.05, 1.67
    psi = synth.solovev_poly(g, A, B, C, R0)
    R = np.repeat(g.r(), g.nh)
    rhs = (2 * A + 8 * B) * R ** 2 + 2 * C - 2 * B * g.dr ** 2
    I = -rhs * g.dr * g.dz / (4e-7 * math.pi * R)
    psib = np.array([psi[i * g.nh + j] for i, j in c.orc.edge_nodes()])
    out = c.ctx.interior_solve(T(torch, I), T(torch, psib)).cpu().numpy()
    assert rel(out, psi) < TOL


# ------------------------------------------------------------------ a4: LSQ

@pytest.mark.parametrize("name", ["33x33", "C1"])
def test_lsq(torch_mod, efit, orc_mod, name):
    torch = torch_mod
    c = case(name, efit, orc_mod)
    psi = synth.solovev_psi(c.cfg.grid)
    resp, _ = c.orc.response(psi)
    y = resp @ synth.c_true(c.cfg.basis)
    sigma = 1e-3 * np.max(np.abs(y)) * np.ones_like(y)
    y = y + sigma * synth.noise(len(y), seed=1)
    st, cref, chi2ref = orc_mod.lsq(resp, y, sigma)
    coef, chi2 = c.ctx.lsq(T(torch, resp), T(torch, y), T(torch, sigma))
    assert rel(coef.cpu().numpy(), cref) < TOL_C
    assert abs(chi2.item() - chi2ref) <= TOL_C * chi2ref


@pytest.mark.parametrize("n_int", [1, 6])
def test_lsq_spline(torch_mod, efit, orc_mod, n_int):
    """Wide bases (5+5 and 10+10 cubic B-splines, 40 MSE-like rows): the 256-thread CholeskyQR2
    kernel k_lsq<NB> (nb > 6), C3's solve."""
    torch = torch_mod
    c = case("129x129", efit, orc_mod, basis=synth.spline_basis(n_int), n_int=40)
    assert c.ctx.nbasis == 2 * (n_int + 4)
    psi = synth.solovev_psi(c.cfg.grid)
    resp, _ = c.orc.response(psi)
    y = resp @ synth.c_true(c.cfg.basis)
    sigma = 1e-3 * np.max(np.abs(y)) * np.ones_like(y)
    y = y + sigma * synth.noise(len(y), seed=1)
    st, cref, chi2ref = orc_mod.lsq(resp, y, sigma)
    assert st == 0
    coef, chi2 = c.ctx.lsq(T(torch, resp), T(torch, y), T(torch, sigma))
    assert rel(coef.cpu().numpy(), cref) < TOL_C
    assert abs(chi2.item() - chi2ref) <= TOL_C * chi2ref


def test_lsq_singular_flag(torch_mod, efit, orc_mod):
    torch = torch_mod
    c = case("33x33", efit, orc_mod)
    resp = np.random.default_rng(0).standard_normal((c.ctx.ndiag, c.ctx.nbasis))
    resp[:, 2] = 3 * resp[:, 1]
    coef, chi2 = c.ctx.lsq(T(torch, resp), T(torch, np.ones(c.ctx.ndiag)), T(torch, np.ones(c.ctx.ndiag)))
    assert c.ctx.status() == efit.EFIT_E_SINGULAR
    assert np.all(np.isnan(coef.cpu().numpy()))


def test_no_plasma_flag(torch_mod, efit, orc_mod):
    torch = torch_mod
    c = case("33x33", efit, orc_mod)
    resp, axbd = c.ctx.response(T(torch, np.zeros(c.cfg.grid.n)))
    assert c.ctx.status() == efit.EFIT_E_NOPLASMA
    assert c.ctx.status() == 0  # cleared


def test_invalid_pointer_rejected(torch_mod, efit, orc_mod):
    torch = torch_mod
    c = case("33x33", efit, orc_mod)
    psi = torch.zeros(c.cfg.grid.n + 1, dtype=torch.float64, device="cuda")[1:]  # 8-byte offset
    with pytest.raises(efit.EfitError) as ei:
        c.ctx.response(psi)
    assert ei.value.code == efit.EFIT_E_INVAL


# ------------------------------------------------------------------ a1-a9: fit step and loop

def _twin(c, noise_seed=1):
    psi_s = synth.solovev_psi(c.cfg.grid)
    ct = synth.c_true(c.cfg.basis)
    return psi_s, ct, c.orc.twin(psi_s, ct, noise_seed=noise_seed)


@pytest.mark.parametrize("name", ["33x33", "C1", "C2"])
@pytest.mark.parametrize("mode", [0, 2])
def test_fit_step(torch_mod, efit, orc_mod, name, mode):
    torch = torch_mod
    c = case(name, efit, orc_mod, mode=mode)
    psi_s, ct, tw = _twin(c)
    psi0 = synth.perturbed_psi(c.cfg.grid, seed=5, rel=1e-3)
    st, psi_ref, cref, chi2ref, epsref = c.orc.fit_step(psi0, tw["psi_ext"], tw["y"], tw["sigma"])
    assert st == 0
    psi = T(torch, psi0)
    coef, chi2, eps = c.ctx._t(c.ctx.nbasis), c.ctx._t(1), c.ctx._t(1)
    c.ctx.fit_step(psi, T(torch, tw["psi_ext"]), T(torch, tw["y"]), T(torch, tw["sigma"]), coef, chi2, eps)
    assert c.ctx.status() == 0
    assert rel(psi.cpu().numpy(), psi_ref) < TOL
    assert rel(coef.cpu().numpy(), cref) < TOL_C
    assert abs(chi2.item() - chi2ref) <= TOL_C * max(chi2ref, 1.0)
    assert abs(eps.item() - epsref) <= 1e-9 * epsref


def test_fit_step_graph_replay_matches_eager(torch_mod, efit, orc_mod):
    torch = torch_mod
    c = case("C1", efit, orc_mod)
    psi_s, ct, tw = _twin(c)
    ext, y, s = T(torch, tw["psi_ext"]), T(torch, tw["y"]), T(torch, tw["sigma"])
    outs = []
    for _ in range(2):
        psi = T(torch, synth.perturbed_psi(c.cfg.grid, seed=5, rel=1e-3))
        coef, chi2, eps = c.ctx._t(c.ctx.nbasis), c.ctx._t(1), c.ctx._t(1)
        for it in range(3):
            c.ctx.fit_step(psi, ext, y, s, coef, chi2, eps)
        outs.append(psi.clone())
    assert torch.equal(outs[0], outs[1])


def test_fit_loop_c2(torch_mod, efit, orc_mod):
    """C2: full loop to eps < 1e-5 from a 1%-perturbed Solov'ev twin (SURVEY 8(d),
    edge-vanishing profile, reading R2); the GPU loop follows the oracle loop iteration by
    iteration and stops at the same iteration.  Continued to eps < 1e-10 the GPU iterate is the
    twin's psi_S with c = c_true (property of the twin construction)."""
    torch = torch_mod
    c = case("C2", efit, orc_mod)
    psi_s, ct, tw = _twin(c, noise_seed=None)
    psi0 = synth.perturbed_psi(c.cfg.grid, seed=5, rel=1e-2)
    ext, y, s = T(torch, tw["psi_ext"]), T(torch, tw["y"]), T(torch, tw["sigma"])
    psi = T(torch, psi0)
    coef, chi2, eps = c.ctx._t(c.ctx.nbasis), c.ctx._t(1), c.ctx._t(1)
    pr = psi0.copy()
    for it in range(200):
        st, pr, cr, chr_, er = c.orc.fit_step(pr, tw["psi_ext"], tw["y"], tw["sigma"])
        c.ctx.fit_step(psi, ext, y, s, coef, chi2, eps)
        assert rel(psi.cpu().numpy(), pr) < 1e-10, it
        assert (eps.item() < 1e-5) == (er < 1e-5), it
        if er < 1e-5:
            break
    assert er < 1e-5
    for it in range(600):
        c.ctx.fit_step(psi, ext, y, s, coef, chi2, eps)
        if eps.item() < 1e-10:
            break
    assert eps.item() < 1e-10
    assert np.max(np.abs(psi.cpu().numpy() - psi_s)) < 1e-8 * np.max(np.abs(psi_s))
    assert np.max(np.abs(coef.cpu().numpy() - ct)) < 1e-7 * np.max(np.abs(ct))


def test_fit_steps_chained_equals_repeated(torch_mod, efit, orc_mod):
    """efit_fit_steps(n) (axis/boundary of iterations 2..n taken from the previous update kernel)
    is bitwise identical to n separate efit_fit_step calls (each normalising from scratch)."""
    torch = torch_mod
    c = case("C2", efit, orc_mod)
    psi_s, ct, tw = _twin(c, noise_seed=1)
    ext, y, s = T(torch, tw["psi_ext"]), T(torch, tw["y"]), T(torch, tw["sigma"])
    psi0 = synth.perturbed_psi(c.cfg.grid, seed=5, rel=1e-3)
    outs = []
    for chained in (False, True):
        psi = T(torch, psi0)
        coef, chi2, eps = c.ctx._t(c.ctx.nbasis), c.ctx._t(1), c.ctx._t(1)
        if chained:
            c.ctx.fit_steps(5, psi, ext, y, s, coef, chi2, eps)
        else:
            for _ in range(5):
                c.ctx.fit_step(psi, ext, y, s, coef, chi2, eps)
        assert c.ctx.status() == 0
        outs.append((psi.clone(), coef.clone(), eps.clone()))
    for a, b in zip(*outs):
        assert torch.equal(a, b)
