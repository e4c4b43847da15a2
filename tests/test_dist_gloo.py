"""world_size-2/3 CPU tests (gloo) of the multi-GPU host logic (include/efit.h "Multi-GPU").

The shard plan comes from the C ABI itself (efit_plan_info, host-only: response rows, full-table
target rows, SYM row-pair tiles, exchange-slice length); each rank fills its zero-padded exchange
slices exactly as the kernels do -- the per-entry values computed by the CPU oracle standing in for
the GPU kernels (this container has no GPU) -- one gloo sum all-reduce per slice makes them
replicated, and the fixed-order finish must reproduce the single-rank arrays BIT FOR BIT:
  * response rows (zero-padded d_resp, summed),
  * full table: the rank's top/bottom entries of psi_b,
  * SYM half table: the per-tile partial sums [i-1][side][slot] (slot = the tile's other 8-row
    block, k_bnd_sym), summed, then reduced in slot order plus the edge-row sources.
The GPU side of the same equivalence (the library's own kernels, world 3 emulated on one GPU
through efit_boundary_partials / efit_boundary_finish, and the in-library NCCL exchange at world 1)
is tests/test_gpu_multi.py."""
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


def _plan(cfg, rank, world, mode):
    import paper_conf_sc_anteparawkbml23_b200 as efit
    c = efit._Config(cfg.grid, cfg.basis, cfg.geometry, rank, world)
    return efit.efit_plan_info(c.grid, c.basis, c.geom, c.dist, mode)


def _tile_pq(t):
    """Row-pair tile index t = Q(Q+1)/2 + P, P <= Q (include/efit.h, efit_table which = 4)."""
    Q = 0
    while (Q + 1) * (Q + 2) // 2 <= t:
        Q += 1
    return t - Q * (Q + 1) // 2, Q


def _sym_slices(T, I, nw, nh, tiles):
    """Per-tile partial sums of the top/bottom nest for the given tiles, in the exchange layout
    part[(i-1)*2 + side][slot]: row direction targets of block P take slot Q, col direction
    targets of block Q take slot P (diagonal tiles: row direction only)."""
    ni = nw - 2
    nblk = (ni + 7) // 8
    I2 = I.reshape(nw, nh)
    F2 = I2[:, ::-1]
    part = np.zeros((ni, 2, nblk))
    for t in tiles:
        P, Q = _tile_pq(t)
        for side, X in ((0, I2), (1, F2)):
            for p in range(8):
                r = 8 * P + p
                if r >= ni:
                    continue
                # sum over sources ii of block Q, all m: T[i][ii][m] * X[ii][m]
                acc = 0.0
                for q in range(8):
                    rq = 8 * Q + q
                    if rq < ni:
                        acc += float(np.dot(T[1 + r, 1 + rq, :], X[1 + rq, :]))
                part[r, side, Q] = acc
            if P != Q:
                for q in range(8):
                    rq = 8 * Q + q
                    if rq >= ni:
                        continue
                    acc = 0.0
                    for p in range(8):
                        r = 8 * P + p
                        if r < ni:
                            acc += float(np.dot(T[1 + rq, 1 + r, :], X[1 + r, :]))
                    part[rq, side, P] = acc
    return part.reshape(-1)


def _sym_finish(part, T, I, nw, nh):
    """Fixed slot order + edge-row sources (ii = 0, nw-1) -> top/bottom entries."""
    ni = nw - 2
    nblk = (ni + 7) // 8
    part = part.reshape(ni, 2, nblk)
    I2 = I.reshape(nw, nh)
    F2 = I2[:, ::-1]
    out = np.zeros(2 * ni)
    for side, X in ((0, I2), (1, F2)):
        for r in range(ni):
            s = float(np.dot(T[1 + r, 0, :], X[0, :]) + np.dot(T[1 + r, nw - 1, :], X[nw - 1, :]))
            for slot in range(nblk):
                s += part[r, side, slot]
            out[side * ni + r] = s
    return out


def _worker(rank, world, port, out_dir, n, mode):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    cfg = synth.small_config(n)
    info = _plan(cfg, rank, world, mode)
    orc = oracle.Oracle.from_config(cfg)
    psi = synth.perturbed_psi(cfg.grid, seed=5)
    I = synth.random_current(cfg.grid, seed=2)
    nw = nh = n
    # response: the rank's rows, zero-padded
    rows = list(range(info.resp_row_lo, info.resp_row_hi))
    resp = torch.zeros(orc.ndiag, orc.nbasis, dtype=torch.float64)
    if rows:
        resp[rows] = torch.from_numpy(orc.response_rows(psi, rows))
    dist.all_reduce(resp)
    # boundary exchange slice
    xlen = int(info.xbuf_len)
    if mode == 0:   # full table: the rank's top/bottom rows of psi_b
        assert xlen == 2 * (nw - 2)
        x = torch.zeros(xlen, dtype=torch.float64)
        own = [q for i in range(info.bnd_row_lo, info.bnd_row_hi) for q in (i - 1, (nw - 2) + i - 1)]
        if own:
            x[own] = torch.from_numpy(orc.boundary_targets(I, [2 * nh + q for q in own]))
    else:           # SYM: per-tile partials of the rank's tiles
        nblk = (nw - 2 + 7) // 8
        assert xlen == 2 * (nw - 2) * nblk
        T = orc.table_T()
        x = torch.from_numpy(_sym_slices(T, I, nw, nh, range(info.sym_tile_lo, info.sym_tile_hi)))
    dist.all_reduce(x)
    if rank == 0:
        np.save(os.path.join(out_dir, "resp.npy"), resp.numpy())
        np.save(os.path.join(out_dir, "x.npy"), x.numpy())
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("n,world,mode", [(33, 2, 0), (65, 3, 0), (33, 2, 2), (65, 3, 2)])
def test_sharded_exchange_matches_single(tmp_path, n, world, mode):
    """world ranks over gloo vs one rank: the exchanged response and boundary slices are bitwise
    the single-rank ones, and so is the finished psi_b."""
    from paper_conf_sc_anteparawkbml23_b200 import build
    build.build()
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path), n, mode), nprocs=world, join=True)
    import oracle
    cfg = synth.small_config(n)
    orc = oracle.Oracle.from_config(cfg)
    psi = synth.perturbed_psi(cfg.grid, seed=5)
    I = synth.random_current(cfg.grid, seed=2)
    ref_resp = orc.response_rows(psi, list(range(orc.ndiag)))
    assert np.array_equal(np.load(tmp_path / "resp.npy"), ref_resp)
    x = np.load(tmp_path / "x.npy")
    nw = nh = n
    if mode == 0:
        ref = orc.boundary_targets(I, list(range(2 * nh, orc.n_edge)))
        assert np.array_equal(x, ref)
    else:
        T = orc.table_T()
        nblk = (nw - 2 + 7) // 8
        x1 = _sym_slices(T, I, nw, nh, range(nblk * (nblk + 1) // 2))
        assert np.array_equal(x, x1)                       # exchange is exact
        fin = _sym_finish(x, T, I, nw, nh)
        assert np.array_equal(fin, _sym_finish(x1, T, I, nw, nh))
        ref = orc.boundary(I)[2 * nh:]                     # and it is the boundary flux
        assert np.max(np.abs(fin - ref)) <= 1e-13 * np.max(np.abs(ref))


@pytest.mark.parametrize("n,world", [(65, 2), (129, 3), (513, 8), (1025, 8)])
@pytest.mark.parametrize("mode", [0, 2])
def test_shard_plan_partitions_work(n, world, mode):
    """The ABI's plan: response rows and full-table target rows are partitions of [0, ndiag) and
    [1, nw-1); the SYM tiles partition [0, nblk(nblk+1)/2), so every exchanged slot has exactly one
    writer; left/right targets are computed on every rank (replicated)."""
    from paper_conf_sc_anteparawkbml23_b200 import build
    build.build()
    cfg = synth.small_config(n)
    rows, bnd, tiles = [], [], []
    for r in range(world):
        info = _plan(cfg, r, world, mode)
        rows += list(range(info.resp_row_lo, info.resp_row_hi))
        bnd += list(range(info.bnd_row_lo, info.bnd_row_hi))
        tiles += list(range(info.sym_tile_lo, info.sym_tile_hi))
        assert (info.lr_j_lo, info.lr_j_hi) == (0, n)
    assert sorted(rows) == list(range(cfg.geometry.ndiag))
    assert sorted(bnd) == list(range(1, n - 1))
    nblk = (n - 2 + 7) // 8
    assert sorted(tiles) == list(range(nblk * (nblk + 1) // 2))
