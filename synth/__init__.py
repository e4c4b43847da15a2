"""Seeded synthetic inputs shared by the oracle tests, the GPU tests and bench.py.

This module holds NO arithmetic of the method (no Green's functions, no basis
evaluation, no solve): only the geometry of a DIII-D-shaped machine, an analytic
Solov'ev equilibrium used as the "true" plasma, and seeded random operands.
Everything here is an *input* recipe; DESIGN.md §"Input recipe" restates it.

Why synthetic: the paper's workload is DIII-D shot #186610 at 2.4 s
(PAPER.md L109, L287), which is not available.  The grids are the paper's
(65^2 ... 513^2) plus the 1025^2 stress case of
BASELINE.json configs[4].  The machine box / limiter / diagnostic counts follow
SURVEY.md §8(d) (domain knowledge, not in the paper).
"""
from __future__ import annotations

import dataclasses
import math
from typing import Optional

import numpy as np

# Machine box: R in [0.84, 2.54] m, Z in [-1.6, 1.6] m.
RMIN, RMAX, ZMIN, ZMAX = 0.84, 2.54, -1.6, 1.6

# Polynomial Solov'ev (SURVEY §8(c) pins): psi_S = -scale*(A R^2 Z^2 + B (R^2-R0^2)^2 + C Z^2)
# The overall minus sign makes psi maximal on the axis for a positive toroidal
# current (Eq. 1, with G > 0), i.e. ip_sign = +1.
SOL_R0, SOL_A, SOL_B, SOL_C = 1.67, 1.2346, 1.0, 0.05
SOL_SCALE = 0.05          # Wb/rad per unit polynomial; gives I_p ~ 1 MA at these shapes
SOL_R_OUT = 2.12          # outboard midplane radius of the last closed flux surface


@dataclasses.dataclass(frozen=True)
class Grid:
    nw: int
    nh: int
    rmin: float = RMIN
    rmax: float = RMAX
    zmin: float = ZMIN
    zmax: float = ZMAX

    @property
    def dr(self) -> float:
        return (self.rmax - self.rmin) / (self.nw - 1)

    @property
    def dz(self) -> float:
        return (self.zmax - self.zmin) / (self.nh - 1)

    def r(self) -> np.ndarray:
        return self.rmin + np.arange(self.nw) * self.dr

    def z(self) -> np.ndarray:
        return self.zmin + np.arange(self.nh) * self.dz

    @property
    def n(self) -> int:
        return self.nw * self.nh


@dataclasses.dataclass
class Geometry:
    fl_r: np.ndarray
    fl_z: np.ndarray
    mp_r: np.ndarray
    mp_z: np.ndarray
    mp_ang: np.ndarray
    int_r: np.ndarray
    int_z: np.ndarray
    lim_r: np.ndarray
    lim_z: np.ndarray
    ip_sign: int = 1

    @property
    def ndiag(self) -> int:
        return len(self.fl_r) + len(self.mp_r) + len(self.int_r)


@dataclasses.dataclass
class Basis:
    kind: int          # 0 = polynomial in psi_hat, 1 = clamped cubic B-spline
    n_pp: int
    n_ff: int
    knots: np.ndarray  # interior knots (kind 1); empty for kind 0

    @property
    def nbasis(self) -> int:
        return self.n_pp + self.n_ff


@dataclasses.dataclass
class Config:
    name: str
    grid: Grid
    geometry: Geometry
    basis: Basis
    description: str


def d_shape(r0: float, a: float, kappa: float, delta: float, n: int, phase: float = 0.0):
    """Miller-type D contour R = r0 + a cos(t + delta sin t), Z = kappa a sin t."""
    t = phase + 2.0 * np.pi * np.arange(n) / n
    r = r0 + a * np.cos(t + delta * np.sin(t))
    z = kappa * a * np.sin(t)
    return r, z, t


def solovev_inboard_radius() -> float:
    """Inboard midplane radius of the Solov'ev LCFS (same level as SOL_R_OUT)."""
    level = (SOL_R_OUT ** 2 - SOL_R0 ** 2) ** 2
    return math.sqrt(SOL_R0 ** 2 - math.sqrt(level))


def limiter(n: int = 128):
    """D-shaped limiter (R0=1.67, a=0.70, kappa=1.9, delta=0.35, 128 vertices) with
    one extra vertex at the Solov'ev inboard-midplane LCFS point, so the plasma is
    inner-wall limited.  Counter-clockwise, not closed (last != first)."""
    r, z, t = d_shape(1.67, 0.70, 1.9, 0.35, n)
    # vertex n/2 is t = pi (inboard midplane, Z = 0): replace it by the touch point.
    k = n // 2
    r = r.copy(); z = z.copy()
    r[k] = solovev_inboard_radius()
    z[k] = 0.0
    return r, z


def diagnostics(n_fl: int = 44, n_mp: int = 76, n_int: int = 0, grid: Optional[Grid] = None):
    """Flux loops on a D contour (a=0.78), magnetic probes on a=0.74 oriented along the
    local contour tangent, optional MSE-like internal B_Z points at cell centres along
    Z = dz/2, R in [1.75, 2.25].  Half-step phase offsets keep every
    diagnostic off the grid nodes."""
    fl_r, fl_z, _ = d_shape(1.67, 0.78, 1.9, 0.35, n_fl, phase=np.pi / n_fl)
    mp_r, mp_z, t = d_shape(1.67, 0.74, 1.9, 0.35, n_mp, phase=np.pi / n_mp)
    # tangent of the contour: dR/dt, dZ/dt
    drdt = -0.74 * np.sin(t + 0.35 * np.sin(t)) * (1.0 + 0.35 * np.cos(t))
    dzdt = 1.9 * 0.74 * np.cos(t)
    mp_ang = np.arctan2(dzdt, drdt)
    if n_int > 0:
        assert grid is not None
        dr, dz = grid.dr, grid.dz
        i0 = int(math.ceil((1.75 - grid.rmin) / dr - 0.5))
        i1 = int(math.floor((2.25 - grid.rmin) / dr - 0.5))
        idx = np.round(np.linspace(i0, i1, n_int)).astype(int)
        # alternate the cell row just above / below the midplane so no two points coincide
        # on coarse grids (129^2 has fewer than 40 cells in [1.75, 2.25])
        j0 = (grid.nh - 1) // 2
        rows = np.where(np.arange(n_int) % 2 == 0, j0, j0 - 1)
        int_r = grid.rmin + (idx + 0.5) * dr
        int_z = grid.zmin + (rows + 0.5) * dz
        assert len(set(zip(idx.tolist(), rows.tolist()))) == n_int, "grid too coarse for the MSE-like points"
    else:
        int_r = np.zeros(0)
        int_z = np.zeros(0)
    return fl_r, fl_z, mp_r, mp_z, mp_ang, int_r, int_z


def make_geometry(grid: Grid, n_int: int = 0) -> Geometry:
    fl_r, fl_z, mp_r, mp_z, mp_ang, int_r, int_z = diagnostics(n_int=n_int, grid=grid)
    lim_r, lim_z = limiter()
    return Geometry(fl_r, fl_z, mp_r, mp_z, mp_ang, int_r, int_z, lim_r, lim_z, 1)


def poly_basis(n_pp: int = 2, n_ff: int = 3) -> Basis:
    """Q8 reading: "5-term polynomial p'/FF' basis" = 5 monomial terms in
    total, 2 for P' and 3 for FF'.  The 5+5 reading is supported (poly_basis(5, 5)) but
    makes the magnetics-only fit ill-posed: scaled cond(A) ~ 1.4e7 at 65^2 and the Picard
    fixed point is unstable (measured with the oracle)."""
    return Basis(0, n_pp, n_ff, np.zeros(0))


def spline_basis(n_int: int = 6) -> Basis:
    """Clamped cubic B-spline, uniform interior knots on [0,1]: n_int + 4 functions each."""
    knots = np.arange(1, n_int + 1) / (n_int + 1.0)
    return Basis(1, n_int + 4, n_int + 4, knots)


def config(name: str) -> Config:
    """The five BASELINE.json configs (C1..C5)."""
    name = name.upper()
    table = {
        "C1": (65, 0, poly_basis(), "65x65, flux loops + probes, 2+3 polynomial basis (5 terms, reading Q8), single fit iteration"),
        "C2": (129, 0, poly_basis(), "129x129, full fit loop on a Solov'ev-derived twin"),
        "C3": (257, 40, spline_basis(6), "257x257, 10+10 cubic-spline basis + 40 MSE-like B_Z points"),
        "C4": (513, 0, poly_basis(), "513x513, response + boundary flux (1/2/4/8 GPUs)"),
        "C5": (1025, 0, poly_basis(), "1025x1025 stress case, table vs on-the-fly Green's"),
    }
    n, n_int, basis, desc = table[name]
    g = Grid(n, n)
    return Config(name, g, make_geometry(g, n_int), basis, desc)


def small_config(n: int, n_int: int = 0, basis: Optional[Basis] = None) -> Config:
    g = Grid(n, n)
    return Config(f"N{n}", g, make_geometry(g, n_int), basis or poly_basis(), f"{n}x{n} test grid")


# ----------------------------------------------------------------------------- psi inputs

def solovev_psi(grid: Grid) -> np.ndarray:
    """psi_S(R,Z) = -scale*(A R^2 Z^2 + B (R^2-R0^2)^2 + C Z^2) on the nodes, flattened
    g = i*nh + j (Z fastest, PAPER.md L217 indexing)."""
    R = grid.r()[:, None]
    Z = grid.z()[None, :]
    p = SOL_A * R ** 2 * Z ** 2 + SOL_B * (R ** 2 - SOL_R0 ** 2) ** 2 + SOL_C * Z ** 2
    return (-SOL_SCALE * p).reshape(-1).astype(np.float64)


# Diverted (X-point) Solov'ev for the f3 steps_ row (reading R4): with C < 0 the
# polynomial Solov'ev has saddle points at R_x^2 = -C/A, Z_x^2 = 2B(R0^2 - R_x^2)/A (both inside
# the limiter for R_x = 1.45 m); the homogeneous term D*Z (Delta* Z = 0, same current profile)
# raises the lower one, which becomes the primary X-point (lower single null, DIII-D's usual shape).
DIV_RX = 1.45
DIV_C = -SOL_A * DIV_RX ** 2
DIV_D = 0.045


def solovev_diverted_psi(grid: Grid, d: float = DIV_D) -> np.ndarray:
    """psi = -scale*(A R^2 Z^2 + B (R^2-R0^2)^2 + C_div Z^2 + d Z) on the nodes (g = i*nh + j)."""
    R = grid.r()[:, None]
    Z = grid.z()[None, :]
    p = SOL_A * R ** 2 * Z ** 2 + SOL_B * (R ** 2 - SOL_R0 ** 2) ** 2 + DIV_C * Z ** 2 + d * Z
    return (-SOL_SCALE * p).reshape(-1).astype(np.float64)


def diverted_xpoints(d: float = 0.0):
    """Analytic X-points (R, +-Z, psi) of the d = 0 double null."""
    rx = math.sqrt(-DIV_C / SOL_A)
    zx = math.sqrt(2 * SOL_B * (SOL_R0 ** 2 - rx ** 2) / SOL_A)
    psi_x = -SOL_SCALE * SOL_B * (SOL_R0 ** 2 - rx ** 2) ** 2
    return rx, zx, psi_x


def solovev_poly(grid: Grid, A: float, B: float, C: float, R0: float) -> np.ndarray:
    """Un-negated polynomial Solov'ev A R^2 Z^2 + B (R^2-R0^2)^2 + C Z^2 (interior-solve pin)."""
    R = grid.r()[:, None]
    Z = grid.z()[None, :]
    return (A * R ** 2 * Z ** 2 + B * (R ** 2 - R0 ** 2) ** 2 + C * Z ** 2).reshape(-1)


def smooth_modes(grid: Grid, seed: int, n_modes: int = 6, amp: float = 1.0) -> np.ndarray:
    """Sum of n_modes random smooth Fourier modes over the box (seeded)."""
    rng = np.random.default_rng(seed)
    x = (grid.r() - grid.rmin) / (grid.rmax - grid.rmin)
    y = (grid.z() - grid.zmin) / (grid.zmax - grid.zmin)
    out = np.zeros((grid.nw, grid.nh))
    for _ in range(n_modes):
        kx, ky = rng.integers(1, 4, size=2)
        ph1, ph2 = rng.uniform(0, 2 * np.pi, size=2)
        a = rng.uniform(-1, 1)
        out += a * np.cos(np.pi * kx * x[:, None] + ph1) * np.cos(np.pi * ky * y[None, :] + ph2)
    return (amp * out).reshape(-1)


def perturbed_psi(grid: Grid, seed: int = 5, rel: float = 1e-3) -> np.ndarray:
    """psi_S plus a smooth perturbation of relative size `rel` of (max-min) psi_S."""
    ps = solovev_psi(grid)
    span = ps.max() - ps.min()
    return ps + rel * span * smooth_modes(grid, seed) / 3.0


def random_current(grid: Grid, seed: int = 2, signed: bool = False, edge: bool = False) -> np.ndarray:
    """I ~ U(0,1) (or U(-1,1) if signed) on interior nodes, 0 on the edge ring (edge=True:
    on every node, the edge ring included -- exercises the edge-row sources)."""
    rng = np.random.default_rng(seed)
    lo = -1.0 if signed else 0.0
    I = rng.uniform(lo, 1.0, size=(grid.nw, grid.nh))
    if not edge:
        I[0, :] = 0.0; I[-1, :] = 0.0; I[:, 0] = 0.0; I[:, -1] = 0.0
    return I.reshape(-1)


def c_true(basis: Basis, seed: int = 7, edge_zero: bool = True, sol_c: float = SOL_C) -> np.ndarray:
    """True profile coefficients.  The leading P' and FF' terms are the Solov'ev's
    constant profiles (Delta* psi_S = -scale[(2A+8B)R^2 + 2C] gives
    P'_0 = scale(2A+8B)/mu0 and mu0 FF'_0/(4 pi^2) = 2 C scale/mu0); higher terms are
    seeded at +-10% of the leading one.  For the spline basis every function gets the
    leading value (partition of unity) times (1 +- 10%).

    edge_zero (default; reading R2): the profiles vanish at the plasma boundary,
    P'(1) = FF'(1) = 0 -- the last monomial coefficient is set to minus the sum of the others,
    the last B-spline coefficient (the only function non-zero at psihat = 1) to 0.  With the
    Solov'ev's constant profiles the current jumps at the last closed surface, the discrete
    mask (0 <= psihat < 1) makes the Picard map discontinuous, and a perturbed start converges
    to a spurious nearby fixed point (2-6 mask nodes off, chi2 ~ 245, c far from c_true;
    measured with the oracle at 65^2); with an edge-vanishing profile the loop converges to
    psi_S and c -> c_true (the twin works for any profile: psi_ext absorbs the mismatch)."""
    mu0 = 4e-7 * np.pi
    pp0 = SOL_SCALE * (2 * SOL_A + 8 * SOL_B) / mu0
    ff0 = 2 * sol_c * SOL_SCALE / mu0 * 4 * np.pi ** 2 / mu0
    rng = np.random.default_rng(seed)
    if basis.kind == 0:
        pp = np.concatenate([[pp0], pp0 * 0.1 * rng.uniform(-1, 1, basis.n_pp - 1)])
        ff = np.concatenate([[ff0], ff0 * 0.1 * rng.uniform(-1, 1, basis.n_ff - 1)])
        if edge_zero:
            if basis.n_pp > 1:
                pp[-1] = -np.sum(pp[:-1])
            if basis.n_ff > 1:
                ff[-1] = -np.sum(ff[:-1])
    else:
        pp = pp0 * (1 + 0.1 * rng.uniform(-1, 1, basis.n_pp))
        ff = ff0 * (1 + 0.1 * rng.uniform(-1, 1, basis.n_ff))
        if edge_zero:
            pp[-1] = 0.0
            ff[-1] = 0.0
    return np.concatenate([pp, ff]).astype(np.float64)


def random_coef(basis: Basis, seed: int) -> np.ndarray:
    rng = np.random.default_rng(seed)
    return rng.uniform(-1, 1, basis.nbasis)


def noise(ndiag: int, seed: int = 1) -> np.ndarray:
    return np.random.default_rng(seed).standard_normal(ndiag)
