import os, sys, json
sys.path.insert(0, os.getcwd())
import numpy as np, torch, synth
import paper_conf_sc_anteparawkbml23_b200 as efit
cfg = synth.config("C4")
ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=2)
I = torch.tensor(synth.random_current(cfg.grid, seed=2), device="cuda")
out = ctx._t(ctx.n_edge)
for _ in range(5): efit.efit_boundary_flux(ctx.handle, I, out)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(200): efit.efit_boundary_flux(ctx.handle, I, out)
e1.record(); torch.cuda.synchronize()
print(os.environ.get("EFIT_B200_LIB", "default").split("/")[-1], round(e0.elapsed_time(e1) / 200 * 1000, 2), "us per efit_boundary_flux")
