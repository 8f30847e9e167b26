"""ctypes wrapper of the plain-C oracle ``liblfd_ref.so`` (TEST INFRASTRUCTURE ONLY).

Every function takes NumPy arrays (complex128 / float64, C-contiguous, host memory) in the layouts
documented at the top of ``oracle/lfd_ref.c`` and mirrors one ``lfd_ref_*`` entry point. Citations
for the arithmetic are in the C file; this module only marshals arguments.
"""
from __future__ import annotations

import ctypes as C
from dataclasses import dataclass

import numpy as np

from . import build as _build

BC_PERIODIC = 0
BC_ZERO = 1
C_LIGHT = 137.035999084  # R1 (atomic units)


class _Cfg(C.Structure):
    _fields_ = [("ndom", C.c_int32), ("nx", C.c_int32), ("ny", C.c_int32), ("nz", C.c_int32),
                ("hx", C.c_double), ("hy", C.c_double), ("hz", C.c_double), ("bc", C.c_int32),
                ("norb", C.c_int32), ("nproj", C.c_int32), ("dt", C.c_double)]


@dataclass
class RefConfig:
    ndom: int
    nx: int
    ny: int
    nz: int
    hx: float
    hy: float
    hz: float
    bc: int
    norb: int
    nproj: int
    dt: float

    def c(self) -> _Cfg:
        return _Cfg(self.ndom, self.nx, self.ny, self.nz, self.hx, self.hy, self.hz, self.bc,
                    self.norb, self.nproj, self.dt)

    @property
    def ngrid(self) -> int:
        return self.nx * self.ny * self.nz

    @property
    def dV(self) -> float:
        return self.hx * self.hy * self.hz


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(_build.build())
        P = C.c_void_p
        cfgp = C.POINTER(_Cfg)
        _lib.lfd_ref_link_sweep.argtypes = [cfgp, P, C.c_int, C.c_int, C.c_double, C.c_double]
        _lib.lfd_ref_kinetic.argtypes = [cfgp, P, C.c_int, C.c_double, C.c_double]
        _lib.lfd_ref_local.argtypes = [cfgp, P, P, P]
        _lib.lfd_ref_nl_half.argtypes = [cfgp, P, P, P]
        _lib.lfd_ref_step.argtypes = [cfgp, P, P, P, P, P, C.c_int]
        _lib.lfd_ref_nl_half_exact.argtypes = [cfgp, P, P, P]
        _lib.lfd_ref_step_exact.argtypes = [cfgp, P, P, P, P, P, C.c_int]
        _lib.lfd_ref_density_current.argtypes = [cfgp, P, P, P, P, P, P]
        _lib.lfd_ref_kinetic_energy.argtypes = [cfgp, P, P, P]
        _lib.lfd_ref_kinetic_energy.restype = C.c_double
        _lib.lfd_ref_energy.argtypes = [cfgp, P, P, P, P, P, P, P]
        _lib.lfd_ref_energy.restype = C.c_int
        _lib.lfd_ref_remap_occ.argtypes = [cfgp, P, P, P, C.c_int, P]
        _lib.lfd_ref_remap_occ.restype = C.c_int
        _lib.lfd_ref_nl_half_dense.argtypes = [cfgp, P, P, P]
        _lib.lfd_ref_nl_half_exact_dense.argtypes = [cfgp, P, P, P]
        _lib.lfd_ref_step_dense.argtypes = [cfgp, P, P, P, P, P, C.c_int, C.c_int]
        _lib.lfd_ref_energy_nl_dense.argtypes = [cfgp, P, P, P, P, P]
        for f in ("nl_half_dense", "nl_half_exact_dense", "step_dense", "energy_nl_dense"):
            getattr(_lib, "lfd_ref_" + f).restype = C.c_int
        for f in ("link_sweep", "kinetic", "local", "nl_half", "step", "density_current", "nl_half_exact",
                  "step_exact"):
            getattr(_lib, "lfd_ref_" + f).restype = C.c_int
    return _lib


def _ptr(a: np.ndarray | None, dtype) -> C.c_void_p | None:
    if a is None:
        return None
    if a.dtype != dtype or not a.flags.c_contiguous:
        raise TypeError(f"expected C-contiguous {dtype}, got {a.dtype}")
    return C.c_void_p(a.ctypes.data)


def _ok(rc: int, what: str) -> None:
    if rc != 0:
        raise RuntimeError(f"{what} failed with status {rc}")


def link_sweep(cfg: RefConfig, psi: np.ndarray, axis: int, parity: int, tau: float, a: float) -> None:
    """In place: one E (parity 0) / O (parity 1) sweep of one domain ``psi[nx,ny,nz,norb]``."""
    c = cfg.c()
    _ok(lib().lfd_ref_link_sweep(C.byref(c), _ptr(psi, np.complex128), axis, parity, tau, a), "link_sweep")


def kinetic(cfg: RefConfig, psi: np.ndarray, axis: int, tau: float, a: float) -> None:
    c = cfg.c()
    _ok(lib().lfd_ref_kinetic(C.byref(c), _ptr(psi, np.complex128), axis, tau, a), "kinetic")


def local(cfg: RefConfig, psi: np.ndarray, vloc: np.ndarray, A: np.ndarray) -> None:
    c = cfg.c()
    _ok(lib().lfd_ref_local(C.byref(c), _ptr(psi, np.complex128), _ptr(vloc, np.float64),
                            _ptr(np.ascontiguousarray(A, np.float64), np.float64)), "local")


def nl_half(cfg: RefConfig, psi: np.ndarray, proj: np.ndarray | None, dnl: np.ndarray | None) -> None:
    c = cfg.c()
    _ok(lib().lfd_ref_nl_half(C.byref(c), _ptr(psi, np.complex128), _ptr(proj, np.complex128),
                              _ptr(dnl, np.float64)), "nl_half")


def nl_half_exact(cfg: RefConfig, psi: np.ndarray, proj: np.ndarray | None, dnl: np.ndarray | None) -> None:
    """In place: the exactly unitary nonlocal factor (dV-orthonormal projector columns)."""
    c = cfg.c()
    _ok(lib().lfd_ref_nl_half_exact(C.byref(c), _ptr(psi, np.complex128), _ptr(proj, np.complex128),
                                    _ptr(dnl, np.float64)), "nl_half_exact")


def step_exact(cfg: RefConfig, psi: np.ndarray, proj: np.ndarray | None, dnl: np.ndarray | None,
               vloc: np.ndarray, A: np.ndarray, nsteps: int = 1) -> None:
    """In place: ``nsteps`` steps N_exact o Local o N_exact of every domain."""
    c = cfg.c()
    A = np.ascontiguousarray(A, np.float64)
    _ok(lib().lfd_ref_step_exact(C.byref(c), _ptr(psi, np.complex128), _ptr(proj, np.complex128),
                                 _ptr(dnl, np.float64), _ptr(vloc, np.float64), _ptr(A, np.float64), nsteps),
        "step_exact")


def step(cfg: RefConfig, psi: np.ndarray, proj: np.ndarray | None, dnl: np.ndarray | None,
         vloc: np.ndarray, A: np.ndarray, nsteps: int = 1) -> None:
    """In place: ``nsteps`` Eq.-6 steps of every domain with v, A held fixed."""
    c = cfg.c()
    A = np.ascontiguousarray(A, np.float64)
    _ok(lib().lfd_ref_step(C.byref(c), _ptr(psi, np.complex128), _ptr(proj, np.complex128),
                           _ptr(dnl, np.float64), _ptr(vloc, np.float64), _ptr(A, np.float64), nsteps),
        "step")


def density_current(cfg: RefConfig, psi: np.ndarray, occ: np.ndarray, A: np.ndarray,
                    want_j: bool = True):
    """Returns (rho [ndom,ng], j [ndom,3,ng] or None, J [ndom,3])."""
    c = cfg.c()
    ng = cfg.ngrid
    rho = np.zeros((cfg.ndom, ng))
    j = np.zeros((cfg.ndom, 3, ng)) if want_j else None
    J = np.zeros((cfg.ndom, 3))
    A = np.ascontiguousarray(A, np.float64)
    _ok(lib().lfd_ref_density_current(C.byref(c), _ptr(psi, np.complex128),
                                      _ptr(np.ascontiguousarray(occ, np.float64), np.float64),
                                      _ptr(A, np.float64), _ptr(rho, np.float64), _ptr(j, np.float64),
                                      _ptr(J, np.float64)), "density_current")
    return rho, j, J


def kinetic_energy(cfg: RefConfig, psi: np.ndarray, occ: np.ndarray, A: np.ndarray) -> float:
    """E_kin of ONE domain (cfg.ndom is ignored beyond the first domain)."""
    c = cfg.c()
    return float(lib().lfd_ref_kinetic_energy(C.byref(c), _ptr(psi, np.complex128),
                                              _ptr(np.ascontiguousarray(occ, np.float64), np.float64),
                                              _ptr(np.ascontiguousarray(A, np.float64), np.float64)))


def energy(cfg: RefConfig, psi: np.ndarray, occ: np.ndarray, vloc: np.ndarray, A: np.ndarray,
           proj: np.ndarray | None = None, dnl: np.ndarray | None = None) -> np.ndarray:
    """[ndom, 4]: kinetic, local, nonlocal, total (calc_energy)."""
    c = cfg.c()
    E = np.zeros((cfg.ndom, 4))
    _ok(lib().lfd_ref_energy(C.byref(c), _ptr(psi, np.complex128),
                             _ptr(np.ascontiguousarray(occ, np.float64), np.float64), _ptr(vloc, np.float64),
                             _ptr(np.ascontiguousarray(A, np.float64), np.float64), _ptr(proj, np.complex128),
                             _ptr(None if dnl is None else np.ascontiguousarray(dnl, np.float64), np.float64),
                             _ptr(E, np.float64)), "energy")
    return E


def remap_occ(cfg: RefConfig, psi: np.ndarray, occ: np.ndarray, refb: np.ndarray) -> np.ndarray:
    """[ndom, nref]: sum_s f_s |<ref_k|psi_s>|^2 (remap_occ)."""
    c = cfg.c()
    nref = refb.shape[-1]
    out = np.zeros((cfg.ndom, nref))
    _ok(lib().lfd_ref_remap_occ(C.byref(c), _ptr(psi, np.complex128),
                                _ptr(np.ascontiguousarray(occ, np.float64), np.float64),
                                _ptr(refb, np.complex128), nref, _ptr(out, np.float64)), "remap_occ")
    return out


def _dmat(Dm):
    return np.ascontiguousarray(Dm, np.complex128)


def nl_half_dense(cfg: RefConfig, psi: np.ndarray, proj: np.ndarray, Dm: np.ndarray) -> None:
    """In place: the renormalised first-order factor with a dense Hermitian D [nproj, nproj] (one domain)."""
    c = cfg.c()
    _ok(lib().lfd_ref_nl_half_dense(C.byref(c), _ptr(psi, np.complex128), _ptr(proj, np.complex128),
                                    _ptr(_dmat(Dm), np.complex128)), "nl_half_dense")


def nl_half_exact_dense(cfg: RefConfig, psi: np.ndarray, proj: np.ndarray, Dm: np.ndarray) -> None:
    """In place: exp(-i (Delta/2) B D B^H dV) for dV-orthonormal B (one domain)."""
    c = cfg.c()
    _ok(lib().lfd_ref_nl_half_exact_dense(C.byref(c), _ptr(psi, np.complex128), _ptr(proj, np.complex128),
                                          _ptr(_dmat(Dm), np.complex128)), "nl_half_exact_dense")


def step_dense(cfg: RefConfig, psi: np.ndarray, proj: np.ndarray | None, Dm: np.ndarray | None,
               vloc: np.ndarray, A: np.ndarray, nsteps: int = 1, exact: bool = False) -> None:
    """In place: nsteps Eq.-6 steps with a dense D [ndom, nproj, nproj] (exact: the unitary factor)."""
    c = cfg.c()
    A = np.ascontiguousarray(A, np.float64)
    _ok(lib().lfd_ref_step_dense(C.byref(c), _ptr(psi, np.complex128), _ptr(proj, np.complex128),
                                 _ptr(None if Dm is None else _dmat(Dm), np.complex128), _ptr(vloc, np.float64),
                                 _ptr(A, np.float64), nsteps, 1 if exact else 0), "step_dense")


def energy_nl_dense(cfg: RefConfig, psi: np.ndarray, occ: np.ndarray, proj: np.ndarray, Dm: np.ndarray) -> np.ndarray:
    """[ndom]: sum_s f_s C_s^H D C_s, C = dV B^H Psi."""
    c = cfg.c()
    E = np.zeros(cfg.ndom)
    _ok(lib().lfd_ref_energy_nl_dense(C.byref(c), _ptr(psi, np.complex128),
                                      _ptr(np.ascontiguousarray(occ, np.float64), np.float64),
                                      _ptr(proj, np.complex128), _ptr(_dmat(Dm), np.complex128),
                                      _ptr(E, np.float64)), "energy_nl_dense")
    return E
