"""Multi-GPU path of the library on one B200 (include/efit.h "Multi-GPU").

* world = 3 emulated serially on one GPU in the caller-exchange mode (efit_dist.nccl_id = NULL):
  every rank's zero-padded slices (response rows; boundary exchange slice from
  efit_boundary_partials: SYM per-tile partials or full-table top/bottom rows) summed on the device
  and finished (efit_boundary_finish) equal the world-1 results BIT FOR BIT -- also for a whole
  fit iteration composed of the step calls.
* The in-library NCCL exchange (efit_dist.nccl_id from efit_nccl_unique_id) with a world-1
  communicator: the exchange nodes are inside the captured fit-step graph, and the results equal
  the plain world-1 path bit for bit (the all-reduce over one rank is the identity).
The world-2 host logic over gloo is tests/test_dist_gloo.py."""
import os

import numpy as np
import pytest

import synth

pytestmark = pytest.mark.gpu


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


def T(torch, a):
    return torch.tensor(np.ascontiguousarray(np.asarray(a, dtype=np.float64)), device="cuda")


def _world(efit, cfg, mode, world):
    return [efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=mode, rank=r, world=world)
            for r in range(world)]


@pytest.mark.parametrize("n", [65, 129, 513])
@pytest.mark.parametrize("mode", [0, 2, 3], ids=["table", "sym", "otf-sym"])
def test_emulated_world3_boundary_bitwise(torch_mod, efit, n, mode):
    torch = torch_mod
    cfg = synth.small_config(n)
    ref = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=mode)
    for seed, signed, edge in ((2, False, False), (3, True, True)):
        I = T(torch, synth.random_current(cfg.grid, seed=seed, signed=signed, edge=edge))
        psib1 = ref.boundary_flux(I)
        ctxs = _world(efit, cfg, mode, 3)
        x = sum(c.boundary_partials(I) for c in ctxs)      # the sum all-reduce (exact: one writer)
        assert x.numel() == ref.info.xbuf_len
        for c in ctxs:                                      # every rank finishes the same psi_b
            assert torch.equal(c.boundary_finish(I, x), psib1)
        for c in ctxs:
            c.close()
        # world 1 through the caller-exchange calls is the same too
        assert torch.equal(ref.boundary_finish(I, ref.boundary_partials(I)), psib1)
    ref.close()


def test_emulated_world3_response_bitwise(torch_mod, efit):
    torch = torch_mod
    cfg = synth.small_config(129)
    psi = T(torch, synth.perturbed_psi(cfg.grid, seed=5, rel=1e-3))
    ref = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=2)
    resp1, _ = ref.response(psi)
    acc = torch.zeros_like(resp1)
    for c in _world(efit, cfg, 2, 3):
        part = torch.zeros_like(resp1)
        efit.efit_response(c.handle, psi, part)
        lo, hi = c.info.resp_row_lo, c.info.resp_row_hi
        assert torch.count_nonzero(part[:lo]) == 0 and torch.count_nonzero(part[hi:]) == 0
        acc += part
        c.close()
    assert torch.equal(acc, resp1)
    ref.close()


def test_boundary_flux_needs_exchange(torch_mod, efit):
    cfg = synth.small_config(33)
    c = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=2, rank=0, world=2)
    I = T(torch_mod, synth.random_current(cfg.grid, seed=2))
    with pytest.raises(efit.EfitError) as ei:
        c.boundary_flux(I)
    assert ei.value.code == efit.EFIT_E_STATE
    coef, chi2, eps = c._t(c.nbasis), c._t(1), c._t(1)
    with pytest.raises(efit.EfitError) as ei:
        c.fit_step(I, I, c._t(c.ndiag), c._t(c.ndiag), coef, chi2, eps)
    assert ei.value.code == efit.EFIT_E_STATE
    c.close()


def _twin_inputs(torch, cfg, ctx):
    """Twin on the GPU via the product API (as bench.py), noise seed 1, 0.1% start."""
    psi_s = T(torch, synth.solovev_psi(cfg.grid))
    ct = T(torch, synth.c_true(cfg.basis))
    I_s = ctx.current(psi_s, ct)
    psib = ctx.boundary_flux(I_s)
    resp, _ = ctx.response(psi_s)
    psi_ext = psi_s - ctx.interior_solve(I_s, psib)
    y = resp @ ct
    sigma = torch.full_like(y, 1e-3) * y.abs().max()
    y = y + sigma * T(torch, synth.noise(ctx.ndiag, seed=1))
    return T(torch, synth.perturbed_psi(cfg.grid, seed=5, rel=1e-3)), psi_ext.contiguous(), y.contiguous(), sigma


@pytest.mark.parametrize("mode", [0, 2])
def test_emulated_world3_fit_iteration_bitwise(torch_mod, efit, mode):
    """A whole fit iteration from the step calls (response -> exchange -> lsq -> current ->
    partials -> exchange -> finish -> solve+update), 3 ranks emulated, 3 iterations: bitwise the
    same step calls at world 1."""
    torch = torch_mod
    cfg = synth.config("C2")
    ref = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=mode)
    psi0, ext, y, s = _twin_inputs(torch, cfg, ref)
    ctxs = _world(efit, cfg, mode, 3)

    def iterate(ranks, psi):
        nd, nb = ref.ndiag, ref.nbasis
        resp = torch.zeros(nd * nb, dtype=torch.float64, device="cuda")
        for c in ranks:
            part = torch.zeros_like(resp)
            efit.efit_response(c.handle, psi, part)
            resp += part
        c0 = ranks[0]
        coef, chi2 = c0.lsq(resp, y, s)
        pcurr = c0.current(psi, coef)
        x = sum(c.boundary_partials(pcurr) for c in ranks)
        psib = c0.boundary_finish(pcurr, x)
        eps = c0._t(1)   # axis/boundary of psi: from the current call above
        efit.efit_solve_update(c0.handle, pcurr, psib, ext, psi, eps)
        return coef, eps

    pa, pb = psi0.clone(), psi0.clone()
    for it in range(3):
        ca, ea = iterate([ref], pa)
        cb, eb = iterate(ctxs, pb)
        assert torch.equal(pa, pb), it
        assert torch.equal(ca, cb) and torch.equal(ea, eb), it
    for c in ctxs:
        c.close()
    ref.close()


@pytest.mark.parametrize("mode", [0, 2])
@pytest.mark.parametrize("name", ["C1", "C4"])
def test_nccl_world1_exchange_bitwise(torch_mod, efit, mode, name):
    """The in-library exchange: a context with an NCCL communicator (world 1) enqueues the response
    and boundary all-reduces inside efit_response / efit_boundary_flux / the captured fit-step
    graph; every output equals the plain path bit for bit."""
    torch = torch_mod
    cfg = synth.config(name)
    plain = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=mode)
    nid = efit.efit_nccl_unique_id()
    xch = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=mode, rank=0, world=1, nccl_id=nid)
    assert xch.info.exchange == 1 and plain.info.exchange == 0
    psi0, ext, y, s = _twin_inputs(torch, cfg, plain)
    ra, _ = plain.response(psi0)
    rb, _ = xch.response(psi0)
    assert torch.equal(ra, rb)
    I = T(torch, synth.random_current(cfg.grid, seed=3, signed=True))
    assert torch.equal(plain.boundary_flux(I), xch.boundary_flux(I))
    outs = []
    for ctx in (plain, xch):
        psi = psi0.clone()
        coef, chi2, eps = ctx._t(ctx.nbasis), ctx._t(1), ctx._t(1)
        for _ in range(2):
            ctx.fit_steps(4, psi, ext, y, s, coef, chi2, eps)   # graph with the exchange nodes
        torch.cuda.synchronize()
        assert ctx.status() == 0
        outs.append((psi, coef, chi2, eps))
    for a, b in zip(*outs):
        assert torch.equal(a, b)
    xch.close()
    plain.close()


@pytest.mark.parametrize("path", ["graphs", "streams"])
@pytest.mark.parametrize("pinned", [True, False])
def test_fit_host_matches_device_steps(torch_mod, efit, monkeypatch, path, pinned):
    """efit_fit_host (the e2e path: host buffers in and out, copies overlapped with the fits of the
    neighbouring slices) equals efit_fit_steps on device buffers slice by slice, bit for bit, in both
    pipelines (per-slice graphs with re-pointed copy nodes, then the whole-call graph of a repeated
    call; the stream fallback) and for pinned and pageable host memory."""
    torch = torch_mod
    if path == "streams":
        monkeypatch.setenv("EFIT_HOST_STREAMS", "1")
    cfg = synth.config("C2")
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=2)
    psi0, ext, y, s = _twin_inputs(torch, cfg, ctx)
    S, iters = 5, 2
    n, nd, nb = psi0.numel(), ctx.ndiag, ctx.nbasis
    P = torch.stack([psi0 * (1.0 + 1e-4 * k) for k in range(S)]).cpu()
    Y = torch.stack([y * (1.0 + 1e-3 * k) for k in range(S)]).cpu()
    G = torch.stack([s for _ in range(S)]).cpu()
    outs = [torch.empty(S * n, dtype=torch.float64), torch.empty(S * nb, dtype=torch.float64),
            torch.empty(S, dtype=torch.float64), torch.empty(S, dtype=torch.float64)]
    ins = [P.reshape(-1).contiguous(), Y.reshape(-1).contiguous(), G.reshape(-1).contiguous()]
    if pinned:
        ins = [t.pin_memory() for t in ins]
        outs = [t.pin_memory() for t in outs]
    st = torch.cuda.Stream()
    for call in range(3):  # 1: per-slice graphs; 2: captured as one whole-call graph; 3: its replay
        for t in outs:
            t.fill_(float("nan"))
        ctx.fit_host(S, iters, *ins, ext, *outs, stream=st)
        st.synchronize()
    assert ctx.status() == 0
    for k in range(S):
        psi = P[k].cuda().contiguous()
        coef, chi2, eps = ctx._t(nb), ctx._t(1), ctx._t(1)
        ctx.fit_steps(iters, psi, ext, Y[k].cuda().contiguous(), G[k].cuda().contiguous(), coef, chi2, eps)
        torch.cuda.synchronize()
        assert torch.equal(outs[0][k * n:(k + 1) * n], psi.cpu()), k
        assert torch.equal(outs[1][k * nb:(k + 1) * nb], coef.cpu()), k
        assert outs[2][k].item() == chi2.item() and outs[3][k].item() == eps.item(), k
    ctx.close()
