"""world_size-2 CPU test (gloo) of the multi-GPU host logic: the shard plan of the C ABI
(efit_plan_info, host-only) covers every response row and boundary target exactly once, and the
zero-padded sum all-reduce used by the sharded fit step reproduces the single-rank arrays bit for
bit.  The per-rank slices are computed by the CPU oracle standing in for the GPU kernels (this
container has no GPU); the GPU-side equivalence is tests/test_gpu_parity.py::
test_sharded_matches_single_bitwise."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import synth


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, out_dir, n):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    import paper_conf_sc_anteparawkbml23_b200 as efit
    cfg = synth.small_config(n)
    c = efit._Config(cfg.grid, cfg.basis, cfg.geometry, rank, world)
    info = efit.efit_plan_info(c.grid, c.basis, c.geom, c.dist)
    rows, edge = efit.owned_targets(info)
    orc = oracle.Oracle.from_config(cfg)
    psi = synth.perturbed_psi(cfg.grid, seed=5)
    I = synth.random_current(cfg.grid, seed=2)
    resp = torch.zeros(orc.ndiag, orc.nbasis, dtype=torch.float64)
    if rows:
        resp[rows] = torch.from_numpy(orc.response_rows(psi, rows))
    psib = torch.zeros(orc.n_edge, dtype=torch.float64)
    if edge:
        psib[edge] = torch.from_numpy(orc.boundary_targets(I, edge))
    efit.exchange(resp)
    efit.exchange(psib)
    if rank == 0:
        np.save(os.path.join(out_dir, "resp.npy"), resp.numpy())
        np.save(os.path.join(out_dir, "psib.npy"), psib.numpy())
        np.save(os.path.join(out_dir, "owned.npy"), np.array([len(rows), len(edge)]))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("n,world", [(33, 2), (65, 2)])
def test_sharded_exchange_matches_single(tmp_path, n, world):
    from paper_conf_sc_anteparawkbml23_b200 import build
    build.build()
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path), n), nprocs=world, join=True)
    import oracle
    cfg = synth.small_config(n)
    orc = oracle.Oracle.from_config(cfg)
    psi = synth.perturbed_psi(cfg.grid, seed=5)
    I = synth.random_current(cfg.grid, seed=2)
    ref_resp = orc.response_rows(psi, list(range(orc.ndiag)))
    ref_psib = orc.boundary_targets(I, list(range(orc.n_edge)))
    assert np.array_equal(np.load(tmp_path / "resp.npy"), ref_resp)
    assert np.array_equal(np.load(tmp_path / "psib.npy"), ref_psib)


@pytest.mark.parametrize("n,world", [(65, 2), (129, 3), (513, 8), (1025, 8)])
def test_shard_plan_partitions_targets(n, world):
    import paper_conf_sc_anteparawkbml23_b200 as efit
    from paper_conf_sc_anteparawkbml23_b200 import build
    build.build()
    cfg = synth.small_config(n)
    seen_rows, seen_edge = [], []
    for r in range(world):
        c = efit._Config(cfg.grid, cfg.basis, cfg.geometry, r, world)
        info = efit.efit_plan_info(c.grid, c.basis, c.geom, c.dist)
        rows, edge = efit.owned_targets(info)
        seen_rows += rows
        seen_edge += edge
    assert sorted(seen_rows) == list(range(cfg.geometry.ndiag))
    assert sorted(seen_edge) == list(range(2 * n + 2 * (n - 2)))
