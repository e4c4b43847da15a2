"""Host-side cost of efit_fit_host per slice (enqueue wall time) vs its device time, for the per-slice
graph pipeline and the stream pipeline (EFIT_HOST_STREAMS=1): is the e2e path host-bound?"""
import os, sys, time
sys.path.insert(0, os.getcwd())
import numpy as np, torch, synth, bench
import paper_conf_sc_anteparawkbml23_b200 as efit
cfg = synth.config("C4")
dev = torch.device("cuda:0")
ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=2, device=dev)
psi0, ext, y, s = bench.twin_inputs(ctx, cfg, torch, dev)
n, nb, c = psi0.numel(), ctx.nbasis, 50
ins = [psi0.cpu().repeat(c).pin_memory(), y.cpu().repeat(c).pin_memory(), s.cpu().repeat(c).pin_memory()]
outs = [torch.empty(c * n, dtype=torch.float64).pin_memory(), torch.empty(c * nb, dtype=torch.float64).pin_memory(),
        torch.empty(c, dtype=torch.float64).pin_memory(), torch.empty(c, dtype=torch.float64).pin_memory()]
st = torch.cuda.Stream()
for _ in range(2):
    ctx.fit_host(c, 1, *ins, ext, *outs, stream=st)
torch.cuda.synchronize()
a, z = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record(st)
t0 = time.perf_counter()
for _ in range(8):
    ctx.fit_host(c, 1, *ins, ext, *outs, stream=st)
t1 = time.perf_counter()
z.record(st)
torch.cuda.synchronize()
t2 = time.perf_counter()
print(f"{os.environ.get('EFIT_HOST_STREAMS', 'graphs')}: host enqueue {(t1 - t0) / (8 * c) * 1e6:.1f} us/slice, "
      f"device {a.elapsed_time(z) / (8 * c) * 1e3:.1f} us/slice, wall {(t2 - t0) / (8 * c) * 1e6:.1f} us/slice")
