"""Small end-to-end run for compute-sanitizer: every per-iteration kernel of the
default SYM and TABLE fit steps, the batch (mbarrier/bulk-copy DMMA kernels), the caller-exchange
boundary partials/finish, the von Hagenow mode and the full steps_ (f3) kernels, on 33x33 (tiny grids keep the tools fast)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("EFIT_NO_GRAPH", "1")   # eager launches: the tools see every kernel

import numpy as np
import torch

import synth
import paper_conf_sc_anteparawkbml23_b200 as efit

dev = torch.device("cuda:0")
T = lambda a: torch.tensor(np.asarray(a, dtype=np.float64), device=dev)
n = int(sys.argv[1]) if len(sys.argv) > 1 else 33
for mode in (2, 0, 4):
    cfg = synth.small_config(n)
    ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=mode, device=dev)
    psi_s = T(synth.solovev_psi(cfg.grid))
    ct = T(synth.c_true(cfg.basis))
    I = ctx.current(psi_s, ct)
    psib = ctx.boundary_flux(I)
    ext = psi_s - ctx.interior_solve(I, psib)
    resp, _ = ctx.response(psi_s)
    y = resp @ ct
    s = torch.full_like(y, 1e-3) * y.abs().max()
    psi = T(synth.perturbed_psi(cfg.grid, seed=5, rel=1e-3))
    coef, chi2, eps = ctx._t(ctx.nbasis), ctx._t(1), ctx._t(1)
    ctx.fit_steps(3, psi, ext.contiguous(), y.contiguous(), s.contiguous(), coef, chi2, eps)
    if mode != 4:
        x = ctx.boundary_partials(I)
        ctx.boundary_finish(I, x)
    if mode == 0:
        ctx.batch_attach(3)
        st = torch.cuda.Stream()
        P = psi.repeat(3).contiguous()
        ctx.fit_step_batch(P, ext.repeat(3).contiguous(), y.repeat(3).contiguous(), s.repeat(3).contiguous(),
                           ctx._t(3 * ctx.nbasis), ctx._t(3), ctx._t(3), stream=st)
        st.synchronize()
    torch.cuda.synchronize()
    assert ctx.status() == 0, efit.efit_last_error(ctx.handle)
    ctx.close()
# full steps_ (f3): scan / final / bits / one-CTA fill (shared-memory bitmaps, atomics) / mask
cfg = synth.small_config(n)
ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=2, device=dev)
ctx.set_steps(efit.EFIT_STEPS_FULL)
psi_s = T(synth.solovev_diverted_psi(cfg.grid))
ct = T(synth.c_true(cfg.basis, sol_c=synth.DIV_C))
I = ctx.current(psi_s, ct)
ext = psi_s - ctx.interior_solve(I, ctx.boundary_flux(I))
resp, _ = ctx.response(psi_s)
y = resp @ ct
s = torch.full_like(y, 1e-3) * y.abs().max()
info, mask = ctx.normalize(psi_s)
coef, chi2, eps = ctx._t(ctx.nbasis), ctx._t(1), ctx._t(1)
psi = psi_s.clone()
ctx.fit_steps(2, psi, ext.contiguous(), y.contiguous(), s.contiguous(), coef, chi2, eps)
torch.cuda.synchronize()
assert ctx.status() == 0, efit.efit_last_error(ctx.handle)
assert info.cpu().numpy()[12] == 1.0
ctx.close()
print("sanitize run ok")
