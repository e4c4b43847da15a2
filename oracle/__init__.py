"""CPU fp64 oracle of the EFIT fitting hot path -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
leg may import this package.  The product (paper_conf_sc_anteparawkbml23_b200/) never
does, and this package never imports the product: the two share no code.  Inputs come
from `synth` (geometry + seeded operands, no method arithmetic).

The arithmetic lives in efit_oracle.c (plain C, one function per step O1..O14 of
SURVEY.md §8(c), each citing the PAPER.md passage it follows); this file only builds
it with gcc and marshals numpy arrays through ctypes.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "efit_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

_dp = ctypes.POINTER(ctypes.c_double)
_ip = ctypes.POINTER(ctypes.c_int)
_u8p = ctypes.POINTER(ctypes.c_uint8)


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (fp contraction off so the host rounding is plain IEEE)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp",
                               "-shared", "-fPIC", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        d, i, p = ctypes.c_double, ctypes.c_int, ctypes.c_void_p
        sig = {
            "or_rf": (d, [d, d, d]), "or_rd": (d, [d, d, d]),
            "or_ellip_ke": (None, [d, d, _dp, _dp]),
            "or_green_psi": (d, [d, d, d, d]),
            "or_green_brbz": (None, [d, d, d, d, _dp, _dp]),
            "or_green_self": (d, [d, d, d]),
            "or_in_polygon": (i, [d, d, i, _dp, _dp]),
            "or_create": (p, [i, i, d, d, d, d, i, i, i, i, _dp,
                              i, _dp, _dp, i, _dp, _dp, _dp, i, _dp, _dp, i, _dp, _dp, i]),
            "or_destroy": (None, [p]),
            "or_set_self_scale": (None, [p, d]),
            "or_set_boundary_method": (None, [p, i]),
            "or_set_steps_mode": (None, [p, i]),
            "or_get_steps_info": (None, [p, _dp]),
            "or_hermite_eval": (None, [p, _dp, d, d, _dp]),
            "or_newton_stationary": (i, [p, _dp, d, d, _dp]),
            "or_set_threads": (None, [i]), "or_get_threads": (i, []),
            "or_get_inlim": (None, [p, _u8p]),
            "or_green_node": (d, [p, i, i, i, i]),
            "or_diag_green": (d, [p, i, i, i]),
            "or_get_T": (None, [p, _dp]), "or_get_Gd": (None, [p, _dp]),
            "or_basis_fn": (None, [p, d, d, _dp]),
            "or_bilinear": (d, [p, _dp, d, d]),
            "or_normalize": (i, [p, _dp, _dp, _dp, _u8p, _dp]),
            "or_response": (i, [p, _dp, _dp, _dp]),
            "or_response_rows": (i, [p, _dp, i, _ip, _dp]),
            "or_lsq": (i, [i, i, _dp, _dp, _dp, _dp, _dp]),
            "or_current": (i, [p, _dp, _dp, _dp]),
            "or_edge_node": (None, [p, i, _ip, _ip]),
            "or_n_edge": (i, [p]),
            "or_boundary": (None, [p, _dp, _dp]),
            "or_boundary_targets": (None, [p, _dp, i, _ip, _dp]),
            "or_pflux_literal": (None, [p, _dp, _dp]),
            "or_boundary_vh": (None, [p, _dp, _dp]),
            "or_apply_gs": (None, [p, _dp, _dp]),
            "or_interior_solve": (None, [p, _dp, _dp, _dp]),
            "or_fit_step": (i, [p, _dp, _dp, _dp, _dp, _dp, _dp, _dp]),
            "or_ndiag": (i, [p]), "or_nbasis": (i, [p]),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def _d(a: np.ndarray):
    return a.ctypes.data_as(_dp)


def _f64(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.float64))


# ----------------------------------------------------------------- scalar functions

def ellip_ke(m: float, m1: Optional[float] = None):
    K, E = ctypes.c_double(), ctypes.c_double()
    lib().or_ellip_ke(m, (1.0 - m) if m1 is None else m1, ctypes.byref(K), ctypes.byref(E))
    return K.value, E.value


def green_psi(R, Z, Rs, Zs) -> float:
    return lib().or_green_psi(R, Z, Rs, Zs)


def green_brbz(R, Z, Rs, Zs):
    br, bz = ctypes.c_double(), ctypes.c_double()
    lib().or_green_brbz(R, Z, Rs, Zs, ctypes.byref(br), ctypes.byref(bz))
    return br.value, bz.value


def green_self(R, dR, dZ) -> float:
    return lib().or_green_self(R, dR, dZ)


def set_threads(n: int) -> None:
    lib().or_set_threads(int(n))


def get_threads() -> int:
    return lib().or_get_threads()


def lsq(A, y, sigma):
    A = _f64(A); y = _f64(y); sigma = _f64(sigma)
    nd, nb = A.shape
    c = np.zeros(nb); chi2 = ctypes.c_double()
    st = lib().or_lsq(nd, nb, _d(A), _d(y), _d(sigma), _d(c), ctypes.byref(chi2))
    return st, c, chi2.value


# ----------------------------------------------------------------- context

class Oracle:
    """One grid + basis + machine geometry (mirrors what efit_green_init receives)."""

    def __init__(self, grid, basis, geometry):
        L = lib()
        self.grid, self.basis, self.geometry = grid, basis, geometry
        g = geometry
        self._keep = [_f64(x) for x in (basis.knots, g.fl_r, g.fl_z, g.mp_r, g.mp_z, g.mp_ang,
                                        g.int_r, g.int_z, g.lim_r, g.lim_z)]
        k = self._keep
        self.ptr = L.or_create(grid.nw, grid.nh, grid.rmin, grid.rmax, grid.zmin, grid.zmax,
                               basis.kind, basis.n_pp, basis.n_ff, len(basis.knots), _d(k[0]),
                               len(g.fl_r), _d(k[1]), _d(k[2]),
                               len(g.mp_r), _d(k[3]), _d(k[4]), _d(k[5]),
                               len(g.int_r), _d(k[6]), _d(k[7]),
                               len(g.lim_r), _d(k[8]), _d(k[9]), int(g.ip_sign))
        if not self.ptr:
            raise ValueError("or_create rejected the configuration")
        self.n = grid.nw * grid.nh
        self.ndiag = L.or_ndiag(self.ptr)
        self.nbasis = L.or_nbasis(self.ptr)
        self.n_edge = L.or_n_edge(self.ptr)

    @classmethod
    def from_config(cls, cfg):
        return cls(cfg.grid, cfg.basis, cfg.geometry)

    def __del__(self):
        try:
            if getattr(self, "ptr", None):
                lib().or_destroy(self.ptr)
                self.ptr = None
        except Exception:
            pass

    # -- geometry / tables
    def edge_node(self, p: int):
        i, j = ctypes.c_int(), ctypes.c_int()
        lib().or_edge_node(self.ptr, p, ctypes.byref(i), ctypes.byref(j))
        return i.value, j.value

    def edge_nodes(self) -> np.ndarray:
        return np.array([self.edge_node(p) for p in range(self.n_edge)], dtype=np.int64)

    def inlim(self) -> np.ndarray:
        out = np.zeros(self.n, dtype=np.uint8)
        lib().or_get_inlim(self.ptr, out.ctypes.data_as(_u8p))
        return out

    def green_node(self, i, j, ii, jj) -> float:
        return lib().or_green_node(self.ptr, i, j, ii, jj)

    def diag_green(self, m, ii, jj) -> float:
        return lib().or_diag_green(self.ptr, m, ii, jj)

    def table_T(self) -> np.ndarray:
        nw, nh = self.grid.nw, self.grid.nh
        out = np.zeros((nw, nw, nh))
        lib().or_get_T(self.ptr, _d(out))
        return out

    def table_Gd(self) -> np.ndarray:
        out = np.zeros((self.ndiag, self.n))
        lib().or_get_Gd(self.ptr, _d(out))
        return out

    def set_boundary_method(self, m: int) -> None:
        """fit_step's boundary flux: 0 = the Green's sum (O12), 1 = von Hagenow (f2)."""
        lib().or_set_boundary_method(self.ptr, int(m))

    def set_steps_mode(self, m: int) -> None:
        """Normalisation (steps_): 0 = O8 limited rule (Q9), 1 = full steps_ (f3, reading R4)."""
        lib().or_set_steps_mode(self.ptr, int(m))

    def steps_info(self) -> np.ndarray:
        """f3 record of the last normalisation (layout in efit_oracle.c, f3 section)."""
        out = np.zeros(16)
        lib().or_get_steps_info(self.ptr, _d(out))
        return out

    def hermite_eval(self, psi, xt: float, xu: float) -> np.ndarray:
        """p, pt, pu, ptt, puu, ptu of the f3 bicubic Hermite interpolant (index coordinates)."""
        psi = _f64(psi)
        out = np.zeros(6)
        lib().or_hermite_eval(self.ptr, _d(psi), xt, xu, _d(out))
        return out

    def newton_stationary(self, psi, xt: float, xu: float):
        """f3 Newton search: (converged, [xt, xu, p, det, ptt])."""
        psi = _f64(psi)
        out = np.zeros(5)
        conv = lib().or_newton_stationary(self.ptr, _d(psi), xt, xu, _d(out))
        return bool(conv), out

    def set_self_scale(self, s: float) -> None:
        lib().or_set_self_scale(self.ptr, s)

    # -- steps
    def basis_fn(self, psihat: float, R: float) -> np.ndarray:
        out = np.zeros(self.nbasis)
        lib().or_basis_fn(self.ptr, psihat, R, _d(out))
        return out

    def bilinear(self, psi, R, Z) -> float:
        psi = _f64(psi)
        return lib().or_bilinear(self.ptr, _d(psi), R, Z)

    def normalize(self, psi):
        psi = _f64(psi)
        pa, pb = ctypes.c_double(), ctypes.c_double()
        mask = np.zeros(self.n, dtype=np.uint8)
        ph = np.zeros(self.n)
        cnt = lib().or_normalize(self.ptr, _d(psi), ctypes.byref(pa), ctypes.byref(pb),
                                 mask.ctypes.data_as(_u8p), _d(ph))
        return cnt, pa.value, pb.value, mask, ph

    def response(self, psi):
        psi = _f64(psi)
        out = np.zeros((self.ndiag, self.nbasis)); axbd = np.zeros(2)
        st = lib().or_response(self.ptr, _d(psi), _d(out), _d(axbd))
        if st:
            raise RuntimeError(f"or_response status {st}")
        return out, axbd

    def response_rows(self, psi, rows: Sequence[int]):
        psi = _f64(psi)
        rows = np.ascontiguousarray(np.asarray(rows, dtype=np.int32))
        out = np.zeros((len(rows), self.nbasis))
        st = lib().or_response_rows(self.ptr, _d(psi), len(rows), rows.ctypes.data_as(_ip), _d(out))
        if st:
            raise RuntimeError(f"or_response_rows status {st}")
        return out

    def current(self, psi, coef):
        psi = _f64(psi); coef = _f64(coef)
        out = np.zeros(self.n)
        st = lib().or_current(self.ptr, _d(psi), _d(coef), _d(out))
        if st:
            raise RuntimeError(f"or_current status {st}")
        return out

    def boundary(self, I):
        I = _f64(I)
        out = np.zeros(self.n_edge)
        lib().or_boundary(self.ptr, _d(I), _d(out))
        return out

    def boundary_targets(self, I, targets):
        I = _f64(I)
        t = np.ascontiguousarray(np.asarray(targets, dtype=np.int32))
        out = np.zeros(len(t))
        lib().or_boundary_targets(self.ptr, _d(I), len(t), t.ctypes.data_as(_ip), _d(out))
        return out

    def boundary_vh(self, I):
        """f2: von Hagenow-type boundary flux (zero-Dirichlet solve + boundary Green's operator)."""
        I = _f64(I)
        out = np.zeros(self.n_edge)
        lib().or_boundary_vh(self.ptr, _d(I), _d(out))
        return out

    def pflux_literal(self, pcurr):
        pcurr = _f64(pcurr)
        out = np.zeros(self.n)
        lib().or_pflux_literal(self.ptr, _d(pcurr), _d(out))
        return out

    def apply_gs(self, psi):
        psi = _f64(psi)
        out = np.zeros(self.n)
        lib().or_apply_gs(self.ptr, _d(psi), _d(out))
        return out

    def interior_solve(self, I, psib):
        I = _f64(I); psib = _f64(psib)
        out = np.zeros(self.n)
        lib().or_interior_solve(self.ptr, _d(I), _d(psib), _d(out))
        return out

    def fit_step(self, psi, psi_ext, meas, sigma):
        psi = _f64(psi).copy(); psi_ext = _f64(psi_ext); meas = _f64(meas); sigma = _f64(sigma)
        coef = np.zeros(self.nbasis); chi2 = ctypes.c_double(); eps = ctypes.c_double()
        st = lib().or_fit_step(self.ptr, _d(psi), _d(psi_ext), _d(meas), _d(sigma), _d(coef),
                               ctypes.byref(chi2), ctypes.byref(eps))
        return st, psi, coef, chi2.value, eps.value

    # -- composite helpers (test infrastructure)
    def twin(self, psi_s, coef_true, noise_seed: Optional[int] = None, noise_rel: float = 1e-3):
        """Twin construction: psi_S becomes an exact discrete fixed point.
        I_S = I(psi_S; c_true); psi_p,S = solve(boundary(I_S), I_S); psi_ext = psi_S - psi_p,S;
        y = Gd I_S (+ optional noise, sigma = noise_rel * max|y| per diagnostic class)."""
        I_s = self.current(psi_s, coef_true)
        psib = self.boundary(I_s)
        psi_p = self.interior_solve(I_s, psib)
        psi_ext = _f64(psi_s) - psi_p
        resp, _ = self.response(psi_s)
        y = resp @ _f64(coef_true)
        g = self.geometry
        sigma = np.zeros(self.ndiag)
        bounds = np.cumsum([0, len(g.fl_r), len(g.mp_r), len(g.int_r)])
        for a, b in zip(bounds[:-1], bounds[1:]):
            if b > a:
                sigma[a:b] = noise_rel * np.max(np.abs(y[a:b]))
        if noise_seed is not None:
            y = y + sigma * np.random.default_rng(noise_seed).standard_normal(self.ndiag)
        return dict(I=I_s, psib=psib, psi_p=psi_p, psi_ext=psi_ext, y=y, sigma=sigma)
