"""Round count and clock profile of k_steps_fill (debug build, EFIT_STEPS_DEBUG printf)."""
import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np, torch, synth
import paper_conf_sc_anteparawkbml23_b200 as efit
cfg = synth.config(sys.argv[1] if len(sys.argv) > 1 else "C4")
ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=2)
ctx.set_steps(efit.EFIT_STEPS_FULL)
p = synth.solovev_diverted_psi(cfg.grid)
p = p + 1e-4 * (p.max() - p.min()) * synth.smooth_modes(cfg.grid, 5) / 3.0
psi = torch.tensor(p, device="cuda")
for _ in range(3):
    ctx.normalize(psi)
torch.cuda.synchronize()
