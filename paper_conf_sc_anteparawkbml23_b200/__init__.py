"""B200-native EFIT fitting-iteration hot path -- thin Python binding of include/efit.h.

Argument marshalling only: every step runs inside libefit_b200.so (hand-written sm_100a
kernels).  PyTorch provides device memory (tensors), streams and process groups.  There
is no CPU fallback: importing this package without the built library, or calling it
without a CUDA device, raises.

Names follow the C ABI (efit_green_init, efit_response, efit_boundary_flux, efit_fit_step,
...).  `EfitContext` bundles the workspace tensor and the opaque handle.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional

import numpy as np

__all__ = [
    "EfitError", "lib", "lib_path", "efit_workspace_bytes", "efit_green_init", "efit_info", "efit_response",
    "efit_current", "efit_boundary_flux", "efit_interior_solve", "efit_lsq", "efit_fit_step", "efit_status",
    "efit_solve_update", "efit_profile_begin", "efit_profile_end", "efit_fit_steps",
    "efit_table", "efit_shard", "efit_destroy", "efit_strerror", "efit_last_error", "efit_version",
    "EfitContext", "EFIT_GREEN_TABLE", "EFIT_GREEN_ONTHEFLY", "EFIT_GREEN_TABLE_SYM",
    "EFIT_GREEN_ONTHEFLY_SYM", "EFIT_GREEN_VONHAGENOW", "efit_plan_info", "owned_targets", "exchange",
    "efit_batch_workspace_bytes", "efit_batch_attach", "efit_fit_step_batch", "efit_fit_steps_batch",
    "efit_boundary_flux_batch", "efit_boundary_basis", "efit_boundary_partials", "efit_boundary_finish",
    "efit_nccl_unique_id", "efit_fit_host", "efit_set_steps", "efit_normalize", "EFIT_STEPS_LIMITER",
    "EFIT_STEPS_FULL",
]

_HERE = os.path.dirname(os.path.abspath(__file__))
# EFIT_B200_LIB: load an in-tree build variant instead (kernel tuning sweeps, scripts/tune_sym.sh)
lib_path = os.environ.get("EFIT_B200_LIB") or os.path.join(_HERE, "libefit_b200.so")

EFIT_GREEN_TABLE = 0
EFIT_GREEN_ONTHEFLY = 1
EFIT_GREEN_TABLE_SYM = 2       # half table by reciprocity (include/efit.h)
EFIT_GREEN_ONTHEFLY_SYM = 3
EFIT_GREEN_VONHAGENOW = 4      # boundary flux by the von Hagenow construction (no O(N^3) nest)
EFIT_STEPS_LIMITER = 0         # steps_ rule (include/efit.h): limited plasma, O8 / reading Q9
EFIT_STEPS_FULL = 1            # full steps_ (f3): bicubic axis, X-points, connectivity-filtered mask
EFIT_OK, EFIT_E_INVAL, EFIT_E_NOMEM, EFIT_E_CUDA, EFIT_E_NCCL = 0, -1, -2, -3, -4
EFIT_E_SINGULAR, EFIT_E_NOPLASMA, EFIT_E_NONFINITE, EFIT_E_STATE = -5, -6, -7, -8

_dp = ctypes.POINTER(ctypes.c_double)


class efit_grid(ctypes.Structure):
    _fields_ = [("nw", ctypes.c_int32), ("nh", ctypes.c_int32), ("rmin", ctypes.c_double),
                ("rmax", ctypes.c_double), ("zmin", ctypes.c_double), ("zmax", ctypes.c_double)]


class efit_basis(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("n_pp", ctypes.c_int32), ("n_ff", ctypes.c_int32),
                ("n_knots", ctypes.c_int32), ("knots", _dp)]


class efit_geometry(ctypes.Structure):
    _fields_ = [("n_fl", ctypes.c_int32), ("fl_r", _dp), ("fl_z", _dp),
                ("n_mp", ctypes.c_int32), ("mp_r", _dp), ("mp_z", _dp), ("mp_ang", _dp),
                ("n_int", ctypes.c_int32), ("int_r", _dp), ("int_z", _dp),
                ("n_lim", ctypes.c_int32), ("lim_r", _dp), ("lim_z", _dp),
                ("ip_sign", ctypes.c_int32)]


class efit_dist(ctypes.Structure):
    _fields_ = [("rank", ctypes.c_int32), ("world", ctypes.c_int32), ("nccl_id", ctypes.c_void_p)]


class efit_info_t(ctypes.Structure):
    _fields_ = [("nw", ctypes.c_int32), ("nh", ctypes.c_int32), ("ndiag", ctypes.c_int32),
                ("nbasis", ctypes.c_int32), ("n_edge", ctypes.c_int32), ("mode", ctypes.c_int32),
                ("rank", ctypes.c_int32), ("world", ctypes.c_int32),
                ("resp_row_lo", ctypes.c_int32), ("resp_row_hi", ctypes.c_int32),
                ("bnd_row_lo", ctypes.c_int32), ("bnd_row_hi", ctypes.c_int32),
                ("lr_blk_lo", ctypes.c_int32), ("lr_blk_hi", ctypes.c_int32),
                ("lr_j_lo", ctypes.c_int32), ("lr_j_hi", ctypes.c_int32),
                ("slab_stride", ctypes.c_int64), ("sym_nblk", ctypes.c_int32),
                ("sym_tile_lo", ctypes.c_int32), ("sym_tile_hi", ctypes.c_int32),
                ("xbuf_len", ctypes.c_int64), ("exchange", ctypes.c_int32),
                ("workspace_bytes", ctypes.c_size_t)]


class EfitError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"EFIT error {code}: {msg}")
        self.code = code


_lib = None


def lib() -> ctypes.CDLL:
    """Load libefit_b200.so (in-tree).  Fails loudly if it has not been built."""
    global _lib
    if _lib is None:
        if not os.path.exists(lib_path):
            raise ImportError(f"{lib_path} is missing: run `python -c 'import __graft_entry__ as g; g.build()'`")
        L = ctypes.CDLL(lib_path)
        P, I, vp = ctypes.POINTER, ctypes.c_int, ctypes.c_void_p
        sig = {
            "efit_workspace_bytes": (I, [P(efit_grid), P(efit_basis), P(efit_geometry), P(efit_dist), I,
                                         P(ctypes.c_size_t)]),
            "efit_green_init": (I, [P(vp), P(efit_grid), P(efit_basis), P(efit_geometry), P(efit_dist), I, vp,
                                    ctypes.c_size_t, vp]),
            "efit_info": (I, [vp, P(efit_info_t)]),
            "efit_plan_info": (I, [P(efit_grid), P(efit_basis), P(efit_geometry), P(efit_dist), I, P(efit_info_t)]),
            "efit_response": (I, [vp, vp, vp, vp, vp]),
            "efit_current": (I, [vp, vp, vp, vp, vp]),
            "efit_set_steps": (I, [vp, ctypes.c_int32]),
            "efit_normalize": (I, [vp, vp, vp, vp, vp]),
            "efit_boundary_flux": (I, [vp, vp, vp, vp]),
            "efit_boundary_partials": (I, [vp, vp, vp, vp]),
            "efit_boundary_finish": (I, [vp, vp, vp, vp, vp]),
            "efit_nccl_unique_id": (I, [vp]),
            "efit_fit_host": (I, [vp, ctypes.c_int32, ctypes.c_int32, vp, vp, vp, vp, vp, vp, vp, vp, vp]),
            "efit_interior_solve": (I, [vp, vp, vp, vp, vp]),
            "efit_lsq": (I, [vp, vp, vp, vp, vp, vp, vp]),
            "efit_fit_step": (I, [vp, vp, vp, vp, vp, vp, vp, vp, vp]),
            "efit_fit_steps": (I, [vp, ctypes.c_int32, vp, vp, vp, vp, vp, vp, vp, vp]),
            "efit_status": (I, [vp, vp]),
            "efit_solve_update": (I, [vp, vp, vp, vp, vp, vp, vp]),
            "efit_profile_begin": (I, [vp, ctypes.c_int32, ctypes.c_int32]),
            "efit_profile_end": (I, [vp, P(ctypes.c_double), ctypes.c_int32, P(ctypes.c_int32)]),
            "efit_table": (I, [vp, I, P(vp)]),
            "efit_batch_workspace_bytes": (I, [vp, ctypes.c_int32, P(ctypes.c_size_t)]),
            "efit_batch_attach": (I, [vp, ctypes.c_int32, vp, ctypes.c_size_t]),
            "efit_fit_step_batch": (I, [vp, vp, vp, vp, vp, vp, vp, vp, vp]),
            "efit_fit_steps_batch": (I, [vp, ctypes.c_int32, vp, vp, vp, vp, vp, vp, vp, vp]),
            "efit_boundary_flux_batch": (I, [vp, vp, vp, vp]),
            "efit_boundary_basis": (I, [vp, vp, vp, vp, vp]),
            "efit_shard": (None, [ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, P(ctypes.c_int32),
                                  P(ctypes.c_int32)]),
            "efit_destroy": (I, [vp]),
            "efit_strerror": (ctypes.c_char_p, [I]),
            "efit_last_error": (ctypes.c_char_p, [vp]),
            "efit_version": (ctypes.c_char_p, []),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def _check(code: int, ctx=None) -> None:
    if code != EFIT_OK:
        msg = lib().efit_last_error(ctx)
        raise EfitError(code, (msg or b"").decode() or lib().efit_strerror(code).decode())


def _ptr(t) -> Optional[int]:
    """Device pointer of a torch tensor (must be contiguous fp64 on CUDA), or None."""
    if t is None:
        return None
    if not t.is_cuda:
        raise ValueError("expected a CUDA tensor")
    if not t.is_contiguous():
        raise ValueError("expected a contiguous tensor")
    return t.data_ptr()


def _stream(stream) -> Optional[int]:
    import torch
    if stream is None:
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


# ------------------------------------------------------------------------ struct builders

def _arr(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.float64))


class _Config:
    """Holds the ctypes structs + the numpy arrays they point into (kept alive)."""

    def __init__(self, grid, basis, geometry, rank: int = 0, world: int = 1, nccl_id: Optional[bytes] = None):
        self.keep = []

        def P(a):
            a = _arr(a)
            self.keep.append(a)
            return a.ctypes.data_as(_dp)

        self.grid = efit_grid(grid.nw, grid.nh, grid.rmin, grid.rmax, grid.zmin, grid.zmax)
        self.basis = efit_basis(basis.kind, basis.n_pp, basis.n_ff, len(basis.knots), P(basis.knots))
        g = geometry
        self.geom = efit_geometry(len(g.fl_r), P(g.fl_r), P(g.fl_z), len(g.mp_r), P(g.mp_r), P(g.mp_z),
                                  P(g.mp_ang), len(g.int_r), P(g.int_r), P(g.int_z), len(g.lim_r), P(g.lim_r),
                                  P(g.lim_z), int(g.ip_sign))
        if nccl_id is not None:
            if len(nccl_id) != 128:
                raise ValueError("nccl_id must be the 128-byte ncclUniqueId")
            self._nccl_id = ctypes.create_string_buffer(bytes(nccl_id), 128)
            self.dist = efit_dist(rank, world, ctypes.cast(self._nccl_id, ctypes.c_void_p))
        else:
            self.dist = efit_dist(rank, world, None)


# ------------------------------------------------------------------------ ABI functions

def efit_workspace_bytes(grid, basis, geom, dist, mode: int = EFIT_GREEN_TABLE) -> int:
    n = ctypes.c_size_t()
    _check(lib().efit_workspace_bytes(ctypes.byref(grid), ctypes.byref(basis), ctypes.byref(geom),
                                      ctypes.byref(dist), mode, ctypes.byref(n)))
    return n.value


def efit_green_init(grid, basis, geom, dist, mode, workspace, stream=None) -> ctypes.c_void_p:
    h = ctypes.c_void_p()
    _check(lib().efit_green_init(ctypes.byref(h), ctypes.byref(grid), ctypes.byref(basis), ctypes.byref(geom),
                                 ctypes.byref(dist), mode, _ptr(workspace), workspace.numel(), _stream(stream)))
    return h


def efit_info(ctx) -> efit_info_t:
    info = efit_info_t()
    _check(lib().efit_info(ctx, ctypes.byref(info)), ctx)
    return info


def efit_plan_info(grid, basis, geom, dist, mode: int = EFIT_GREEN_TABLE) -> efit_info_t:
    info = efit_info_t()
    _check(lib().efit_plan_info(ctypes.byref(grid), ctypes.byref(basis), ctypes.byref(geom), ctypes.byref(dist),
                                mode, ctypes.byref(info)))
    return info


def owned_targets(info):
    """Host logic of the sharded step: the response rows and the top/bottom edge positions (ABI edge
    order) whose exchange-slice entries this rank writes (full-table mode; SYM modes exchange the
    per-tile partial sums instead, see include/efit.h).  Every other entry of the rank's slice is
    exactly 0, so a sum all-reduce over ranks reproduces the single-GPU arrays bit for bit.  The
    left/right targets are computed on every rank and never exchanged."""
    rows = list(range(info.resp_row_lo, info.resp_row_hi))
    nw, nh = info.nw, info.nh
    edge = []
    for i in range(info.bnd_row_lo, info.bnd_row_hi):
        edge += [2 * nh + (i - 1), 2 * nh + (nw - 2) + (i - 1)]
    return rows, sorted(edge)


def exchange(buf, group=None) -> None:
    """Caller-exchange mode: make a zero-padded rank slice replicated with one sum all-reduce
    (NCCL on GPUs, gloo in tests).  Exact: every entry has one non-zero term."""
    import torch.distributed as dist
    dist.all_reduce(buf, op=dist.ReduceOp.SUM, group=group)


def efit_nccl_unique_id() -> bytes:
    """A fresh 128-byte ncclUniqueId (create on one rank, broadcast to the others)."""
    buf = ctypes.create_string_buffer(128)
    _check(lib().efit_nccl_unique_id(buf))
    return buf.raw


def efit_response(ctx, psi, resp, axbd=None, stream=None) -> None:
    _check(lib().efit_response(ctx, _ptr(psi), _ptr(resp), _ptr(axbd), _stream(stream)), ctx)


def efit_set_steps(ctx, steps_mode: int) -> None:
    _check(lib().efit_set_steps(ctx, int(steps_mode)), ctx)


def efit_normalize(ctx, psi, info, mask=None, stream=None) -> None:
    _check(lib().efit_normalize(ctx, _ptr(psi), _ptr(info), _ptr(mask), _stream(stream)), ctx)


def efit_current(ctx, psi, coef, pcurr, stream=None) -> None:
    _check(lib().efit_current(ctx, _ptr(psi), _ptr(coef), _ptr(pcurr), _stream(stream)), ctx)


def efit_boundary_flux(ctx, pcurr, psib, stream=None) -> None:
    _check(lib().efit_boundary_flux(ctx, _ptr(pcurr), _ptr(psib), _stream(stream)), ctx)


def efit_boundary_partials(ctx, pcurr, xbuf, stream=None) -> None:
    _check(lib().efit_boundary_partials(ctx, _ptr(pcurr), _ptr(xbuf), _stream(stream)), ctx)


def efit_boundary_finish(ctx, pcurr, xbuf, psib, stream=None) -> None:
    _check(lib().efit_boundary_finish(ctx, _ptr(pcurr), _ptr(xbuf), _ptr(psib), _stream(stream)), ctx)


def efit_interior_solve(ctx, pcurr, psib, psi_p, stream=None) -> None:
    _check(lib().efit_interior_solve(ctx, _ptr(pcurr), _ptr(psib), _ptr(psi_p), _stream(stream)), ctx)


def efit_lsq(ctx, resp, meas, sigma, coef, chi2, stream=None) -> None:
    _check(lib().efit_lsq(ctx, _ptr(resp), _ptr(meas), _ptr(sigma), _ptr(coef), _ptr(chi2), _stream(stream)), ctx)


def efit_fit_step(ctx, psi, psi_ext, meas, sigma, coef, chi2, eps, stream=None) -> None:
    _check(lib().efit_fit_step(ctx, _ptr(psi), _ptr(psi_ext), _ptr(meas), _ptr(sigma), _ptr(coef), _ptr(chi2),
                               _ptr(eps), _stream(stream)), ctx)


def efit_solve_update(ctx, pcurr, psib, psi_ext, psi, eps, stream=None) -> None:
    _check(lib().efit_solve_update(ctx, _ptr(pcurr), _ptr(psib), _ptr(psi_ext), _ptr(psi), _ptr(eps),
                                   _stream(stream)), ctx)


PROFILE_FIELDS = ("step", "normalize", "response", "lsq_current", "bnd_tb", "bnd_lr", "tail")


def efit_profile_begin(ctx, nsteps: int, every: int = 1) -> None:
    _check(lib().efit_profile_begin(ctx, nsteps, every), ctx)


def efit_profile_end(ctx):
    """Returns ({field: total ms over the recorded steps}, nsteps)."""
    out = (ctypes.c_double * len(PROFILE_FIELDS))()
    n = ctypes.c_int32()
    _check(lib().efit_profile_end(ctx, out, len(PROFILE_FIELDS), ctypes.byref(n)), ctx)
    return dict(zip(PROFILE_FIELDS, list(out))), n.value


def efit_fit_steps(ctx, nsteps, psi, psi_ext, meas, sigma, coef, chi2, eps, stream=None) -> None:
    _check(lib().efit_fit_steps(ctx, nsteps, _ptr(psi), _ptr(psi_ext), _ptr(meas), _ptr(sigma), _ptr(coef),
                                _ptr(chi2), _ptr(eps), _stream(stream)), ctx)


def _hptr(t) -> int:
    """Host pointer of a contiguous CPU fp64 tensor / numpy array (efit_fit_host)."""
    if isinstance(t, np.ndarray):
        if t.dtype != np.float64 or not t.flags.c_contiguous:
            raise ValueError("expected a C-contiguous float64 array")
        return t.ctypes.data
    if t.is_cuda or not t.is_contiguous():
        raise ValueError("expected a contiguous host tensor")
    return t.data_ptr()


def efit_fit_host(ctx, nslice, iters, h_psi0, h_meas, h_sigma, psi_ext, h_psi, h_coef, h_chi2, h_eps,
                  stream=None) -> None:
    _check(lib().efit_fit_host(ctx, nslice, iters, _hptr(h_psi0), _hptr(h_meas), _hptr(h_sigma), _ptr(psi_ext),
                               _hptr(h_psi), _hptr(h_coef), _hptr(h_chi2), _hptr(h_eps), _stream(stream)), ctx)


def efit_batch_workspace_bytes(ctx, nslice: int) -> int:
    n = ctypes.c_size_t()
    _check(lib().efit_batch_workspace_bytes(ctx, nslice, ctypes.byref(n)), ctx)
    return n.value


def efit_batch_attach(ctx, nslice: int, workspace) -> None:
    _check(lib().efit_batch_attach(ctx, nslice, _ptr(workspace), workspace.numel()), ctx)


def efit_fit_step_batch(ctx, psi, psi_ext, meas, sigma, coef, chi2, eps, stream=None) -> None:
    _check(lib().efit_fit_step_batch(ctx, _ptr(psi), _ptr(psi_ext), _ptr(meas), _ptr(sigma), _ptr(coef),
                                     _ptr(chi2), _ptr(eps), _stream(stream)), ctx)


def efit_fit_steps_batch(ctx, nsteps, psi, psi_ext, meas, sigma, coef, chi2, eps, stream=None) -> None:
    _check(lib().efit_fit_steps_batch(ctx, nsteps, _ptr(psi), _ptr(psi_ext), _ptr(meas), _ptr(sigma),
                                      _ptr(coef), _ptr(chi2), _ptr(eps), _stream(stream)), ctx)


def efit_boundary_flux_batch(ctx, pcurr, psib, stream=None) -> None:
    _check(lib().efit_boundary_flux_batch(ctx, _ptr(pcurr), _ptr(psib), _stream(stream)), ctx)


def efit_boundary_basis(ctx, psi, rb, axbd=None, stream=None) -> None:
    _check(lib().efit_boundary_basis(ctx, _ptr(psi), _ptr(rb), _ptr(axbd), _stream(stream)), ctx)


def efit_status(ctx, stream=None) -> int:
    return lib().efit_status(ctx, _stream(stream))


def efit_table(ctx, which: int) -> int:
    p = ctypes.c_void_p()
    _check(lib().efit_table(ctx, which, ctypes.byref(p)), ctx)
    return p.value


def efit_shard(n: int, rank: int, world: int):
    lo, hi = ctypes.c_int32(), ctypes.c_int32()
    lib().efit_shard(n, rank, world, ctypes.byref(lo), ctypes.byref(hi))
    return lo.value, hi.value


def efit_destroy(ctx) -> None:
    lib().efit_destroy(ctx)


def efit_strerror(code: int) -> str:
    return lib().efit_strerror(code).decode()


def efit_last_error(ctx=None) -> str:
    return (lib().efit_last_error(ctx) or b"").decode()


def efit_version() -> str:
    return lib().efit_version().decode()


# ------------------------------------------------------------------------ convenience context

class EfitContext:
    """Owns the device workspace (a torch uint8 tensor) and the library handle."""

    def __init__(self, grid, basis, geometry, mode: int = EFIT_GREEN_TABLE, rank: int = 0, world: int = 1,
                 device=None, stream=None, nccl_id: Optional[bytes] = None):
        import torch
        self.cfg = _Config(grid, basis, geometry, rank, world, nccl_id)
        self.device = torch.device(device if device is not None else "cuda")
        nbytes = efit_workspace_bytes(self.cfg.grid, self.cfg.basis, self.cfg.geom, self.cfg.dist, mode)
        # 256-byte alignment: allocate a little extra and offset
        raw = torch.empty(nbytes + 256, dtype=torch.uint8, device=self.device)
        off = (-raw.data_ptr()) % 256
        self._raw = raw
        self.workspace = raw[off:off + nbytes]
        self.handle = efit_green_init(self.cfg.grid, self.cfg.basis, self.cfg.geom, self.cfg.dist, mode,
                                      self.workspace, stream)
        self.info = efit_info(self.handle)
        self.nw, self.nh = self.info.nw, self.info.nh
        self.ndiag, self.nbasis, self.n_edge = self.info.ndiag, self.info.nbasis, self.info.n_edge

    def close(self) -> None:
        if getattr(self, "handle", None):
            efit_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def _t(self, n: int):
        import torch
        return torch.zeros(n, dtype=torch.float64, device=self.device)

    # tensor-returning helpers (allocation + one ABI call each)
    def response(self, psi, stream=None):
        resp = self._t(self.ndiag * self.nbasis)
        axbd = self._t(2)
        efit_response(self.handle, psi, resp, axbd, stream)
        return resp.view(self.ndiag, self.nbasis), axbd

    def set_steps(self, steps_mode: int) -> None:
        efit_set_steps(self.handle, steps_mode)

    def normalize(self, psi, stream=None):
        """(info[16], uint8 mask[nw*nh]) of the context's steps_ rule (include/efit.h efit_normalize)."""
        import torch
        info = self._t(16)
        mask = torch.zeros(self.nw * self.nh, dtype=torch.uint8, device=self.device)
        efit_normalize(self.handle, psi, info, mask, stream)
        return info, mask

    def current(self, psi, coef, stream=None):
        out = self._t(self.nw * self.nh)
        efit_current(self.handle, psi, coef, out, stream)
        return out

    def boundary_flux(self, pcurr, stream=None):
        out = self._t(self.n_edge)
        efit_boundary_flux(self.handle, pcurr, out, stream)
        return out

    def boundary_partials(self, pcurr, stream=None):
        """This rank's zero-padded boundary exchange slice (caller-exchange mode)."""
        out = self._t(int(self.info.xbuf_len))
        efit_boundary_partials(self.handle, pcurr, out, stream)
        return out

    def boundary_finish(self, pcurr, xbuf, stream=None):
        out = self._t(self.n_edge)
        efit_boundary_finish(self.handle, pcurr, xbuf, out, stream)
        return out

    def interior_solve(self, pcurr, psib, stream=None):
        out = self._t(self.nw * self.nh)
        efit_interior_solve(self.handle, pcurr, psib, out, stream)
        return out

    def lsq(self, resp, meas, sigma, stream=None):
        coef, chi2 = self._t(self.nbasis), self._t(1)
        efit_lsq(self.handle, resp.reshape(-1).contiguous(), meas, sigma, coef, chi2, stream)
        return coef, chi2

    def fit_step(self, psi, psi_ext, meas, sigma, coef, chi2, eps, stream=None):
        efit_fit_step(self.handle, psi, psi_ext, meas, sigma, coef, chi2, eps, stream)

    def fit_steps(self, nsteps, psi, psi_ext, meas, sigma, coef, chi2, eps, stream=None):
        efit_fit_steps(self.handle, nsteps, psi, psi_ext, meas, sigma, coef, chi2, eps, stream)

    def fit_host(self, nslice, iters, h_psi0, h_meas, h_sigma, psi_ext, h_psi, h_coef, h_chi2, h_eps, stream=None):
        efit_fit_host(self.handle, nslice, iters, h_psi0, h_meas, h_sigma, psi_ext, h_psi, h_coef, h_chi2, h_eps,
                      stream)

    def status(self, stream=None) -> int:
        return efit_status(self.handle, stream)

    # multi-time-slice batch (include/efit.h: efit_batch_attach)
    def batch_attach(self, nslice: int) -> None:
        import torch
        nbytes = efit_batch_workspace_bytes(self.handle, nslice)
        raw = torch.empty(nbytes + 256, dtype=torch.uint8, device=self.device)
        off = (-raw.data_ptr()) % 256
        self._batch_raw = raw
        self.batch_workspace = raw[off:off + nbytes]
        efit_batch_attach(self.handle, nslice, self.batch_workspace)
        self.nslice = nslice

    def fit_step_batch(self, psi, psi_ext, meas, sigma, coef, chi2, eps, stream=None):
        efit_fit_step_batch(self.handle, psi, psi_ext, meas, sigma, coef, chi2, eps, stream)

    def fit_steps_batch(self, nsteps, psi, psi_ext, meas, sigma, coef, chi2, eps, stream=None):
        efit_fit_steps_batch(self.handle, nsteps, psi, psi_ext, meas, sigma, coef, chi2, eps, stream)

    def boundary_basis(self, psi, stream=None):
        """[nbasis, n_edge]: boundary flux of every basis current of psi (efit_boundary_basis)."""
        out = self._t(self.nbasis * self.n_edge)
        efit_boundary_basis(self.handle, psi, out, None, stream)
        return out.view(self.nbasis, self.n_edge)

    def boundary_flux_batch(self, pcurr, stream=None):
        out = self._t(self.nslice * self.n_edge)
        efit_boundary_flux_batch(self.handle, pcurr, out, stream)
        return out.view(self.nslice, self.n_edge)

    def table_ptr(self, which: int) -> int:
        return efit_table(self.handle, which)
