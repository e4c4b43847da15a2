"""SURVEY 8(f) f4 trade-off on one B200 (C4 513^2, full table): time of the paper-order boundary
pass (current of the fitted coefficients -> efit_boundary_flux, 2 RHS) against the fused variant
(efit_boundary_basis: every basis current, 2 nbasis RHS on the tensor cores, no dependency on the
least squares).  CUDA events around 200 calls each after warm-up; prints one JSON line."""
import json, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np
import torch
import synth
import paper_conf_sc_anteparawkbml23_b200 as efit

cfg = synth.config(os.environ.get("CFG", "C4"))
dev = torch.device("cuda")
ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=efit.EFIT_GREEN_TABLE, device=dev)
ctx.batch_attach(ctx.nbasis)
st = torch.cuda.Stream()
torch.cuda.set_stream(st)
psi = torch.tensor(synth.perturbed_psi(cfg.grid, seed=5, rel=1e-3), device=dev)
coef = torch.tensor(synth.c_true(cfg.basis), device=dev)
pc = torch.zeros(ctx.nw * ctx.nh, dtype=torch.float64, device=dev)
pb = torch.zeros(ctx.n_edge, dtype=torch.float64, device=dev)
rb = torch.zeros(ctx.nbasis * ctx.n_edge, dtype=torch.float64, device=dev)


def paper_order():
    efit.efit_current(ctx.handle, psi, coef, pc, st)
    efit.efit_boundary_flux(ctx.handle, pc, pb, st)


def fused():
    efit.efit_boundary_basis(ctx.handle, psi, rb, None, st)


def timeit(f, n=200):
    for _ in range(10):
        f()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(st)
    for _ in range(n):
        f()
    b.record(st)
    torch.cuda.synchronize()
    return a.elapsed_time(b) / n * 1e3


t0, t1 = timeit(paper_order), timeit(fused)
psib_fused = (coef @ rb.view(ctx.nbasis, ctx.n_edge)).cpu().numpy()
err = float(np.max(np.abs(psib_fused - pb.cpu().numpy())) / np.max(np.abs(pb.cpu().numpy())))
print(json.dumps({"config": cfg.name, "nbasis": ctx.nbasis, "paper_order_us": round(t0, 2),
                  "boundary_basis_us": round(t1, 2), "ratio": round(t1 / t0, 3),
                  "linearity_rel_err": err}))
