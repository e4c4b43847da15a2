"""k_lsq<NB> phase clocks inside the fit pipeline (debug build): chained fit steps at C3."""
import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np, torch, synth, bench
import paper_conf_sc_anteparawkbml23_b200 as efit
cfg = synth.config("C3")
ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=2)
psi0, ext, y, s = bench.twin_inputs(ctx, cfg, torch, torch.device("cuda"))
psi = psi0.clone(); coef, chi2, eps = ctx._t(ctx.nbasis), ctx._t(1), ctx._t(1)
for _ in range(4):
    ctx.fit_step(psi, ext, y, s, coef, chi2, eps)
torch.cuda.synchronize()
