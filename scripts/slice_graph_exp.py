"""Per-slice device time of independent one-iteration fits (each from its own psi, so each normalises)
captured 1, 2 or 4 per CUDA graph: the cost of a graph boundary per slice (no copies)."""
import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np, torch, synth, bench
import paper_conf_sc_anteparawkbml23_b200 as efit
cfg = synth.config("C4")
dev = torch.device("cuda:0")
ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=2, device=dev)
psi0, ext, y, s = bench.twin_inputs(ctx, cfg, torch, dev)
slots = [psi0.clone() for _ in range(4)]
coef, chi2, eps = ctx._t(ctx.nbasis), ctx._t(1), ctx._t(1)
st = torch.cuda.Stream()
for per in (1, 2, 4):
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=st, capture_error_mode="thread_local"):
        for k in range(per):
            ctx.fit_steps(1, slots[k], ext, y, s, coef, chi2, eps)
    torch.cuda.synchronize()
    n = 400 // per
    for _ in range(3): g.replay()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(n): g.replay()
    b.record(); torch.cuda.synchronize()
    print(f"{per} slice(s) per graph: {a.elapsed_time(b) / (n * per) * 1000:.1f} us per slice", flush=True)
g = torch.cuda.CUDAGraph()
with torch.cuda.graph(g, stream=st, capture_error_mode="thread_local"):
    ctx.fit_steps(100, slots[0], ext, y, s, coef, chi2, eps)
torch.cuda.synchronize()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record()
for _ in range(4): g.replay()
b.record(); torch.cuda.synchronize()
print(f"chained: {a.elapsed_time(b) / 400 * 1000:.1f} us per iteration")
