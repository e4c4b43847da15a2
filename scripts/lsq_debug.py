"""Phase clocks of k_lsq<NB> (debug build with EFIT_LSQ_DEBUG) at C3 (nb = 20, 160 rows)."""
import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np, torch, synth, bench
import paper_conf_sc_anteparawkbml23_b200 as efit
cfg = synth.config(sys.argv[1] if len(sys.argv) > 1 else "C3")
ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=2)
psi0, ext, y, s = bench.twin_inputs(ctx, cfg, torch, torch.device("cuda"))
resp, _ = ctx.response(psi0)
for _ in range(3):
    ctx.lsq(resp.reshape(-1).contiguous(), y, s)
torch.cuda.synchronize()
