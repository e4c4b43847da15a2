"""Experiment: throughput of S independent C4 reconstructions run concurrently (one context and one
stream each; graph-replayed chained fit steps) vs one.  Decides whether a concurrent-slice host
pipeline is worth building."""
import os, sys, json
sys.path.insert(0, os.getcwd())
import numpy as np, torch, synth
import bench
import paper_conf_sc_anteparawkbml23_b200 as efit

cfg = synth.config("C4")
dev = torch.device("cuda:0")
K = 200
res = {}
for S in (1, 2, 3):
    ctxs, graphs, streams = [], [], []
    for k in range(S):
        ctx = efit.EfitContext(cfg.grid, cfg.basis, cfg.geometry, mode=2, device=dev)
        psi0, ext, y, s = bench.twin_inputs(ctx, cfg, torch, dev)
        psi = psi0.clone(); coef, chi2, eps = ctx._t(ctx.nbasis), ctx._t(1), ctx._t(1)
        for _ in range(5):
            ctx.fit_step(psi, ext, y, s, coef, chi2, eps)
        st = torch.cuda.Stream()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=st, capture_error_mode="thread_local"):
            ctx.fit_steps(K, psi, ext, y, s, coef, chi2, eps)
        ctxs.append((ctx, psi0, ext, y, s, psi)); graphs.append(g); streams.append(st)
    torch.cuda.synchronize()
    best = 1e9
    for rep in range(3):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        main = torch.cuda.current_stream()
        a.record(main)
        for st, g in zip(streams, graphs):
            st.wait_stream(main)
            with torch.cuda.stream(st):
                g.replay()
        for st in streams:
            main.wait_stream(st)
        b.record(main)
        torch.cuda.synchronize()
        best = min(best, a.elapsed_time(b))
    res[S] = S * K / (best / 1000.0)
    print(f"S={S}: {res[S]:.1f} fit iterations/s total ({best / K * 1000:.1f} us per round of S)", flush=True)
    for c in ctxs:
        c[0].close()
    del ctxs, graphs
    torch.cuda.empty_cache()
