"""the full fitting loop on the 129^2 twin from a 0.1 %-perturbed
Solov'ev start to eps < 1e-5 on one B200: iterations, device time to solution (CUDA events; one
eps read-back per iteration, as a user polling convergence would do), it/s, and |c - c_true| of
the noise-free twin.  Also the same loop with chained iterations checked every 4 (efit_fit_steps).
Prints one JSON line."""
import json, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np
import torch
import oracle
import synth
import paper_conf_sc_anteparawkbml23_b200 as efit

name = os.environ.get("CFG", "C2")
mode = {"table": 0, "sym": 2}[os.environ.get("MODE", "sym")]
cfg = synth.config(name)
orc = oracle.Oracle.from_config(cfg)  # twin construction (test infrastructure: inputs only)
psi_s = synth.solovev_psi(cfg.grid)
ct = synth.c_true(cfg.basis)
tw = orc.twin(psi_s, ct, noise_seed=None)
dev = torch.device("cuda")
ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=mode, device=dev)
T = lambda a: torch.tensor(np.asarray(a, dtype=np.float64), device=dev)
ext, y, s = T(tw["psi_ext"]), T(tw["y"]), T(tw["sigma"])
psi0 = T(synth.perturbed_psi(cfg.grid, seed=5, rel=1e-3))
coef, chi2, eps = ctx._t(ctx.nbasis), ctx._t(1), ctx._t(1)
st = torch.cuda.Stream()
torch.cuda.set_stream(st)


def loop(chunk):
    psi = psi0.clone()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(st)
    it = 0
    while it < 200:
        if chunk == 1:
            ctx.fit_step(psi, ext, y, s, coef, chi2, eps, stream=st)
        else:
            ctx.fit_steps(chunk, psi, ext, y, s, coef, chi2, eps, stream=st)
        it += chunk
        if eps.item() < 1e-5:  # device -> host read of eps (synchronises the stream)
            break
    b.record(st)
    torch.cuda.synchronize()
    return it, a.elapsed_time(b), eps.item(), coef.cpu().numpy()


for _ in range(2):
    loop(1)  # warm-up (graph capture)
it1, ms1, e1, c1 = loop(1)
it4, ms4, e4, c4 = loop(4)
cerr = float(np.max(np.abs(c1 - ct)) / np.max(np.abs(ct)))
print(json.dumps({"config": name, "mode": os.environ.get("MODE", "sym"), "iterations": it1, "eps": e1,
                  "time_to_solution_ms": round(ms1, 3), "it_per_s": round(1000 * it1 / ms1, 1),
                  "chained4_iterations": it4, "chained4_time_ms": round(ms4, 3),
                  "coef_rel_err_vs_c_true": cerr}))
