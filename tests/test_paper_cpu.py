"""The paper-literal CPU comparator (baseline/paper_cpu.c, timed by bench.py's cpu_baseline)
computes the same fit iteration as the oracle: psi to 1e-11 (plain sums, DST by FFT vs the
oracle's compensated sums and explicit sine matrix), coefficients to the normal equations'
conditioning (cond^2 u), on 1 thread and on several threads."""
import numpy as np
import pytest

import synth


@pytest.mark.parametrize("name,basis", [("33", "poly"), ("65", "poly"), ("65", "spline")])
def test_paper_cpu_matches_oracle(oracle_mod, name, basis):
    from baseline import paper_cpu
    n = int(name)
    b = synth.poly_basis() if basis == "poly" else synth.spline_basis(2)
    cfg = synth.small_config(n, basis=b)
    orc = oracle_mod.Oracle.from_config(cfg)
    tw = orc.twin(synth.solovev_psi(cfg.grid), synth.c_true(cfg.basis), noise_seed=1)
    psi0 = synth.perturbed_psi(cfg.grid, seed=5, rel=1e-3)
    st, pr, cr, chr_, er = orc.fit_step(psi0, tw["psi_ext"], tw["y"], tw["sigma"])
    pc = paper_cpu.PaperCPU(cfg, orc)
    for threads in (1, 4):
        paper_cpu.set_threads(threads)
        s2, p2, c2, x2, e2 = pc.fit_step(psi0, tw["psi_ext"], tw["y"], tw["sigma"])
        assert s2 == 0
        # the normal equations square cond(A): the 12-term spline fit moves c (and through the
        # current, psi) by ~cond^2 u ~ 1e-7; the well-conditioned 2+3 basis agrees to 1e-11
        tol = 1e-11 if basis == "poly" else 1e-6
        assert np.max(np.abs(p2 - pr)) <= tol * np.max(np.abs(pr))
        assert np.max(np.abs(c2 - cr)) <= 1e-4 * np.max(np.abs(cr))
        assert abs(x2 - chr_) <= 1e-6 * chr_
        assert abs(e2 - er) <= 1e-5 * er
