"""CPU-only checks of the C ABI: the library loads, exports every symbol include/efit.h
declares, validates arguments on the host, and the host-side sharding logic partitions
targets exactly.  No compute calls (no GPU here)."""
import ctypes
import os
import re

import pytest

import synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def efit():
    from paper_conf_sc_anteparawkbml23_b200 import build
    build.build()
    import paper_conf_sc_anteparawkbml23_b200 as e
    e.lib()
    return e


def _declared_functions():
    src = open(os.path.join(ROOT, "include", "efit.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(efit_[a-z_]+)\s*\(", src)))


def test_exports_every_declared_symbol(efit):
    names = _declared_functions()
    assert len(names) >= 15
    L = ctypes.CDLL(efit.lib_path)
    for n in names:
        assert hasattr(L, n), f"missing export {n}"


def test_no_torch_in_abi():
    src = open(os.path.join(ROOT, "include", "efit.h")).read()
    assert "torch" not in src.split("*/", 1)[1].lower()
    assert 'extern "C"' in src


def test_version_and_strerror(efit):
    assert "sm_100a" in efit.efit_version()
    for code in range(0, -9, -1):
        assert efit.efit_strerror(code) != "unknown status"


def _cfg(cfg, rank=0, world=1):
    import paper_conf_sc_anteparawkbml23_b200 as e
    return e._Config(cfg.grid, cfg.basis, cfg.geometry, rank, world)


def test_workspace_bytes_scales(efit):
    sizes = {}
    for name in ["C1", "C4", "C5"]:
        c = _cfg(synth.config(name))
        sizes[name] = efit.efit_workspace_bytes(c.grid, c.basis, c.geom, c.dist)
    # N^3 Green's table dominates: 513^3 * 8 B = 1.08 GB, 1025^3 * 8 B = 8.6 GB
    assert 1.08e9 < sizes["C4"] < 1.5e9
    assert 8.6e9 < sizes["C5"] < 9.9e9
    c = _cfg(synth.config("C4"))
    otf = efit.efit_workspace_bytes(c.grid, c.basis, c.geom, c.dist, efit.EFIT_GREEN_ONTHEFLY)
    assert otf < 0.32e9  # Gd (253 MB) + per-iteration scratch, no boundary table


@pytest.mark.parametrize("mutate,expect", [
    (lambda c: setattr(c.grid, "nw", 2), "grid size"),
    (lambda c: setattr(c.grid, "nh", 100), "power of two"),
    (lambda c: setattr(c.grid, "rmin", 0.0), "rmin"),
    (lambda c: setattr(c.basis, "n_pp", 0) or setattr(c.basis, "n_ff", 0), "n_pp + n_ff"),
    (lambda c: setattr(c.basis, "kind", 7), "kind"),
    (lambda c: setattr(c.geom, "n_lim", 2), "limiter"),
    (lambda c: setattr(c.geom, "ip_sign", 0), "ip_sign"),
    (lambda c: setattr(c.dist, "world", 0), "world"),
])
def test_host_validation(efit, mutate, expect):
    c = _cfg(synth.small_config(33))
    mutate(c)
    with pytest.raises(efit.EfitError) as ei:
        efit.efit_workspace_bytes(c.grid, c.basis, c.geom, c.dist)
    assert ei.value.code == efit.EFIT_E_INVAL
    assert expect in str(ei.value)


def test_spline_validation(efit):
    cfg = synth.small_config(33, basis=synth.spline_basis(6))
    c = _cfg(cfg)
    assert efit.efit_workspace_bytes(c.grid, c.basis, c.geom, c.dist) > 0
    c.basis.n_pp = 9
    with pytest.raises(efit.EfitError):
        efit.efit_workspace_bytes(c.grid, c.basis, c.geom, c.dist)


@pytest.mark.parametrize("n,world", [(120, 1), (120, 2), (120, 7), (511, 8), (3, 8), (1023, 3)])
def test_shard_partition(efit, n, world):
    prev = 0
    sizes = []
    for r in range(world):
        lo, hi = efit.efit_shard(n, r, world)
        assert lo == prev and hi >= lo
        sizes.append(hi - lo)
        prev = hi
    assert prev == n and max(sizes) - min(sizes) <= 1


def test_sharded_workspace_is_smaller(efit):
    cfg = synth.config("C4")
    full = _cfg(cfg)
    half = _cfg(cfg, 0, 2)
    b1 = efit.efit_workspace_bytes(full.grid, full.basis, full.geom, full.dist)
    b2 = efit.efit_workspace_bytes(half.grid, half.basis, half.geom, half.dist)
    assert b2 < 0.6 * b1
