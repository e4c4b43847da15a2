"""ctypes wrapper of baseline/paper_cpu.c -- the paper-literal CPU comparator timed by bench.py's
cpu_baseline.  Not test infrastructure, not the product.  Built with
gcc -O3 -march=native -fopenmp on the host that runs it (the file name carries a hash of the CPU
model and flags, so a library built on another machine is never loaded).  Its Green's tables are
the oracle's memo tables (built outside the timed iteration, as EFIT's efund precompute)."""
from __future__ import annotations

import ctypes
import hashlib
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "paper_cpu.c")
_dp = ctypes.POINTER(ctypes.c_double)


def _cpu_tag() -> str:
    try:
        info = open("/proc/cpuinfo").read()
        keys = [ln for ln in info.splitlines() if ln.startswith(("model name", "flags"))][:2]
    except OSError:
        keys = []
    return hashlib.sha1("\n".join(keys).encode()).hexdigest()[:12]


def cpu_model() -> str:
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def build() -> str:
    lib = os.path.join(_HERE, f"libpaper_cpu.{_cpu_tag()}.so")
    if not os.path.exists(lib) or os.path.getmtime(lib) < os.path.getmtime(_SRC):
        tmp = lib + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O3", "-march=native", "-fopenmp", "-shared", "-fPIC", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, lib)
    return lib


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        d, i, p = ctypes.c_double, ctypes.c_int, ctypes.c_void_p
        L.pc_create.restype = p
        L.pc_create.argtypes = [i, i, d, d, d, d, i, i, i, i, _dp, i, _dp, _dp, p, i, _dp, _dp, i]
        L.pc_destroy.argtypes = [p]
        L.pc_set_threads.argtypes = [i]
        L.pc_get_threads.restype = i
        L.pc_fit_step.restype = i
        L.pc_fit_step.argtypes = [p, _dp, _dp, _dp, _dp, _dp, _dp, _dp]
        _lib = L
    return _lib


def set_threads(n: int) -> None:
    lib().pc_set_threads(int(n))


def get_threads() -> int:
    return lib().pc_get_threads()


def _f(a):
    return np.ascontiguousarray(np.asarray(a, dtype=np.float64))


class PaperCPU:
    def __init__(self, cfg, orc):
        g, b, geo = cfg.grid, cfg.basis, cfg.geometry
        self.T = orc.table_T()
        self.Gd = orc.table_Gd()
        self.inlim = np.ascontiguousarray(orc.inlim())
        self.keep = [_f(b.knots), _f(geo.lim_r), _f(geo.lim_z)]
        k = self.keep
        D = lambda a: a.ctypes.data_as(_dp)
        self.ptr = lib().pc_create(g.nw, g.nh, g.rmin, g.rmax, g.zmin, g.zmax, b.kind, b.n_pp, b.n_ff, len(b.knots),
                                   D(k[0]), geo.ndiag, D(self.T), D(self.Gd), self.inlim.ctypes.data, len(geo.lim_r),
                                   D(k[1]), D(k[2]), int(geo.ip_sign))
        self.nbasis = b.nbasis

    def fit_step(self, psi, psi_ext, meas, sigma):
        psi = _f(psi).copy()
        psi_ext, meas, sigma = _f(psi_ext), _f(meas), _f(sigma)
        coef = np.zeros(self.nbasis)
        chi2, eps = ctypes.c_double(), ctypes.c_double()
        D = lambda a: a.ctypes.data_as(_dp)
        st = lib().pc_fit_step(self.ptr, D(psi), D(psi_ext), D(meas), D(sigma), D(coef), ctypes.byref(chi2),
                               ctypes.byref(eps))
        return st, psi, coef, chi2.value, eps.value

    def __del__(self):
        try:
            lib().pc_destroy(self.ptr)
        except Exception:
            pass
