"""CPU oracle of the self-consistent LFD time step -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline / ``--impl reference`` leg
may import this module; the product path never does. It shares no code with the CUDA library.

What it computes (PAPER.md = /root/reference/PAPER.md, "P:n" = line n; readings R23-R28 are listed in
DESIGN.md §3): the LFD step of Eq. 6 whose Hamiltonian depends on the propagated orbitals ("the
time-propagation operator itself depends on the wave functions being propagated"):

  v_loc = v_ion + v_H[rho] + v_xc[rho]     (Eq. 5: local pseudopotential + Hartree + local xc)
  A     = A_ext(t) + A_ind(t)              (Eq. 2 A_X(alpha); "We solve Maxwell's equation for A")

on the GLOBAL grid that the domain cores tile (Fig. 1; R18). Every step calls the plain-C step of
``oracle/lfd_ref.c`` (``ref.step`` / ``ref.step_exact``) with v_loc and A at the step midpoint (Eq. 4,
P:54); the library primitive used beyond it is numpy's FFT for the Poisson equation (R23).

  R23 Hartree: periodic global cell, nabla^2 v_H = -4 pi (rho - mean rho) in the plane-wave (spectral)
      form v_H = sum_{G != 0} 4 pi / |G|^2 rho_G e^{i G.r}, G_d = 2 pi m_d / (N_d h_d),
      m_d in [-N_d/2, N_d/2) (the uniform background neutralises G = 0).
  R24 xc: spin-unpolarised LDA exchange (Dirac-Slater), v_x = -(3 rho / pi)^{1/3},
      E_x = -(3/4)(3/pi)^{1/3} dV sum rho^{4/3} (rho clamped at 0).
  R25 Maxwell: one macroscopic (long-wavelength) induced field for the whole cell,
      d^2 A_ind / dt^2 = 4 pi c J_e = -4 pi c Jbar, Jbar = the electron-NUMBER current (R13) averaged
      over the global grid (electric current = -Jbar).  Energy E_field = V |dA_ind/dt|^2 / (8 pi c^2).
  R26 Maxwell integrator: velocity Verlet at integer times, the step midpoint takes
      A_mid = A_ext(t_n + Delta/2) + (A_ind(t_n) + A_ind(t_n+1)) / 2.
  R27 self-consistency ("self-consistent, time-reversible"): predictor v_Hxc,mid^(0) =
      (3/2) v_Hxc(t_n) - (1/2) v_Hxc(t_n-1); n_corr corrector sweeps, each re-propagating Psi(t_n)
      with v_Hxc,mid^(k+1) = (v_Hxc(t_n) + v_Hxc[rho(Psi^(k)(t_n+1))]) / 2 (implicit midpoint in v;
      time-reversible at convergence).
  R28 A_ext is given at half steps: Aext[2k] = A_ext(t_n0 + k Delta), Aext[2k+1] = its midpoint value,
      the same vector for every domain (the single-cell Maxwell field is uniform).

Parity status (tests/test_oracle_sc.py): hartree pinned (single Fourier modes of an anisotropic grid
against 4 pi / |G|^2; zero mean; mode superposition), vx/ex pinned (uniform gas closed form; functional
derivative by central differences), maxwell pinned (uniform electron gas: plasma frequency
omega_p^2 = 4 pi rho and the pendulum equation of the k = 0 state against scipy's ODE solver),
sc_step pinned (flags = 0 reduces to ref.step with v_ion and A_ext; O(Delta^2) total-energy drift;
time reversal of the converged step; domain tiling = one big domain's density assembly).
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

from . import ref

C_LIGHT = ref.C_LIGHT
SC_HARTREE = 1
SC_XC = 2
SC_MAXWELL = 4


# ---- global grid assembly (R18: domain cores tile the global grid, buffer b = 0) -----------------
def check_tiling(cfg: ref.RefConfig, offsets: np.ndarray, gdims) -> None:
    cover = np.zeros(tuple(gdims), dtype=np.int64)
    for dm in range(cfg.ndom):
        o = offsets[dm]
        if min(o) < 0 or o[0] + cfg.nx > gdims[0] or o[1] + cfg.ny > gdims[1] or o[2] + cfg.nz > gdims[2]:
            raise ValueError("domain outside the global grid")
        cover[o[0]:o[0] + cfg.nx, o[1]:o[1] + cfg.ny, o[2]:o[2] + cfg.nz] += 1
    if not np.all(cover == 1):
        raise ValueError("domain cores must tile the global grid exactly once")


def assemble(cfg: ref.RefConfig, dom_field: np.ndarray, offsets: np.ndarray, gdims) -> np.ndarray:
    """[ndom, ng] per-domain field -> [GX, GY, GZ] global field (each domain writes its core)."""
    g = np.zeros(tuple(gdims))
    for dm in range(cfg.ndom):
        o = offsets[dm]
        g[o[0]:o[0] + cfg.nx, o[1]:o[1] + cfg.ny, o[2]:o[2] + cfg.nz] = \
            dom_field[dm].reshape(cfg.nx, cfg.ny, cfg.nz)
    return g


def restrict(cfg: ref.RefConfig, g: np.ndarray, offsets: np.ndarray) -> np.ndarray:
    """[GX, GY, GZ] global field -> [ndom, ng] per-domain field."""
    out = np.empty((cfg.ndom, cfg.ngrid))
    for dm in range(cfg.ndom):
        o = offsets[dm]
        out[dm] = g[o[0]:o[0] + cfg.nx, o[1]:o[1] + cfg.ny, o[2]:o[2] + cfg.nz].reshape(-1)
    return out


# ---- R23 Hartree, R24 exchange ---------------------------------------------------------------------
def hartree(rho_g: np.ndarray, h) -> np.ndarray:
    """v_H on the periodic global grid (R23): v_H = sum_{G != 0} (4 pi / |G|^2) rho_G e^{iG.r}."""
    N = rho_g.shape
    rho_G = np.fft.fftn(rho_g) / rho_g.size
    G2 = np.zeros(N)
    for d in range(3):
        G = 2.0 * np.pi * np.fft.fftfreq(N[d], d=h[d])   # 2 pi m / (N h), m in [-N/2, N/2)
        shape = [1, 1, 1]
        shape[d] = N[d]
        G2 = G2 + (G * G).reshape(shape)
    vG = np.zeros_like(rho_G)
    nz = G2 > 0
    vG[nz] = 4.0 * np.pi * rho_G[nz] / G2[nz]
    return np.real(np.fft.ifftn(vG) * rho_g.size)


def vx_lda(rho: np.ndarray) -> np.ndarray:
    """Dirac-Slater exchange potential of the spin-unpolarised density (R24)."""
    return -np.cbrt(3.0 * np.maximum(rho, 0.0) / np.pi)


def ex_lda(rho: np.ndarray, dV: float) -> float:
    return float(-0.75 * np.cbrt(3.0 / np.pi) * dV * np.sum(np.maximum(rho, 0.0) ** (4.0 / 3.0)))


def v_hxc(rho_g: np.ndarray, h, flags: int) -> np.ndarray:
    v = np.zeros_like(rho_g)
    if flags & SC_HARTREE:
        v = v + hartree(rho_g, h)
    if flags & SC_XC:
        v = v + vx_lda(rho_g)
    return v


# ---- the self-consistent step ---------------------------------------------------------------------
@dataclass
class SCState:
    psi: np.ndarray                 # [ndom, nx, ny, nz, norb] complex128 (Psi(t_n))
    vh: np.ndarray                  # [GX, GY, GZ] v_Hxc[rho(t_n)]
    vh_prev: np.ndarray             # [GX, GY, GZ] v_Hxc[rho(t_{n-1})] (= vh at the start)
    A_ind: np.ndarray = field(default_factory=lambda: np.zeros(3))
    Adot: np.ndarray = field(default_factory=lambda: np.zeros(3))
    Jbar: np.ndarray = field(default_factory=lambda: np.zeros(3))   # global mean current at t_n
    rho_g: np.ndarray | None = None   # [GX, GY, GZ] rho(t_n)


@dataclass
class SCProblem:
    cfg: ref.RefConfig
    proj: np.ndarray | None
    dnl: np.ndarray | None
    occ: np.ndarray                 # [ndom, norb]
    vion: np.ndarray                # [ndom, ng] local pseudopotential of each domain
    offsets: np.ndarray             # [ndom, 3] int
    gdims: tuple
    flags: int = SC_HARTREE | SC_XC | SC_MAXWELL
    n_corr: int = 1
    exact_nl: bool = False

    @property
    def h(self):
        return (self.cfg.hx, self.cfg.hy, self.cfg.hz)

    @property
    def volume(self) -> float:
        return float(np.prod(self.gdims)) * self.cfg.dV


def _density(p: SCProblem, psi: np.ndarray, A: np.ndarray):
    """rho_g [GX,GY,GZ] and Jbar [3] of psi with the uniform vector potential A [3]."""
    Ad = np.tile(np.asarray(A, np.float64), (p.cfg.ndom, 1))
    rho, _, J = ref.density_current(p.cfg, psi, p.occ, Ad, want_j=False)
    # the grid mean over the global cell: every domain core has the same number of points
    return assemble(p.cfg, rho, p.offsets, p.gdims), J.mean(axis=0)


def sc_init(p: SCProblem, psi0: np.ndarray, Aext0, A_ind0=None, Adot0=None) -> SCState:
    """State at t_0: rho, Jbar with A(t_0) = A_ext(t_0) + A_ind(t_0); v_Hxc(t_-1) := v_Hxc(t_0)."""
    check_tiling(p.cfg, p.offsets, p.gdims)
    st = SCState(psi=psi0.copy(), vh=np.zeros(p.gdims), vh_prev=np.zeros(p.gdims))
    if A_ind0 is not None:
        st.A_ind = np.array(A_ind0, np.float64)
    if Adot0 is not None:
        st.Adot = np.array(Adot0, np.float64)
    A0 = np.asarray(Aext0, np.float64) + (st.A_ind if p.flags & SC_MAXWELL else 0.0)
    st.rho_g, st.Jbar = _density(p, st.psi, A0)
    st.vh = v_hxc(st.rho_g, p.h, p.flags)
    st.vh_prev = st.vh.copy()
    return st


def _propagate(p: SCProblem, psi: np.ndarray, vmid_g: np.ndarray, A_mid: np.ndarray) -> None:
    v = p.vion + restrict(p.cfg, vmid_g, p.offsets)
    v = np.ascontiguousarray(v.reshape(p.cfg.ndom, p.cfg.nx, p.cfg.ny, p.cfg.nz))
    Ad = np.tile(A_mid, (p.cfg.ndom, 1))
    if p.exact_nl:
        ref.step_exact(p.cfg, psi, p.proj, p.dnl, v, Ad, 1)
    else:
        ref.step(p.cfg, psi, p.proj, p.dnl, v, Ad, 1)


def sc_step(p: SCProblem, st: SCState, Aext: np.ndarray, nsteps: int = 1) -> SCState:
    """In place on st: nsteps self-consistent LFD steps (R23-R28). Aext [2*nsteps+1, 3] (R28)."""
    Aext = np.asarray(Aext, np.float64).reshape(-1, 3)
    if Aext.shape[0] < 2 * nsteps + 1:
        raise ValueError("Aext needs 2*nsteps+1 half-step samples")
    dt = p.cfg.dt
    maxwell = bool(p.flags & SC_MAXWELL)
    for n in range(nsteps):
        # R26: Verlet half kick with J(t_n) and drift of A_ind to t_n+1
        if maxwell:
            Adot_half = st.Adot - 2.0 * np.pi * C_LIGHT * dt * st.Jbar
            A_ind_new = st.A_ind + dt * Adot_half
            A_mid = Aext[2 * n + 1] + 0.5 * (st.A_ind + A_ind_new)
            A_end = Aext[2 * n + 2] + A_ind_new
        else:
            A_mid = Aext[2 * n + 1].copy()
            A_end = Aext[2 * n + 2].copy()
        # R27: predictor, then n_corr corrector sweeps from Psi(t_n)
        vmid = 1.5 * st.vh - 0.5 * st.vh_prev
        for k in range(p.n_corr + 1):
            psi = st.psi.copy()
            _propagate(p, psi, vmid, A_mid)
            rho_g, Jbar = _density(p, psi, A_end)
            vnew = v_hxc(rho_g, p.h, p.flags)
            vmid = 0.5 * (st.vh + vnew)
        st.psi = psi
        st.rho_g = rho_g
        st.vh_prev = st.vh
        st.vh = vnew
        st.Jbar = Jbar
        if maxwell:
            st.A_ind = A_ind_new
            st.Adot = Adot_half - 2.0 * np.pi * C_LIGHT * dt * Jbar
    return st


def total_energy(p: SCProblem, st: SCState, Aext_now) -> dict:
    """E = sum_domains [E_kin(A) + dV sum v_ion rho + E_nl] + E_H + E_x + E_field at the state's time
    (A = A_ext + A_ind). E_H = (1/2) dV sum rho v_H (R23), E_x (R24), E_field = V |Adot|^2/(8 pi c^2) (R25)."""
    A = np.asarray(Aext_now, np.float64) + (st.A_ind if p.flags & SC_MAXWELL else 0.0)
    Ad = np.tile(A, (p.cfg.ndom, 1))
    vi = np.ascontiguousarray(p.vion.reshape(p.cfg.ndom, p.cfg.nx, p.cfg.ny, p.cfg.nz))
    E = ref.energy(p.cfg, st.psi, p.occ, vi, Ad, p.proj, p.dnl)
    out = {"kinetic": float(E[:, 0].sum()), "ion": float(E[:, 1].sum()), "nonlocal": float(E[:, 2].sum())}
    out["hartree"] = 0.5 * p.cfg.dV * float(np.sum(st.rho_g * hartree(st.rho_g, p.h))) \
        if p.flags & SC_HARTREE else 0.0
    out["xc"] = ex_lda(st.rho_g, p.cfg.dV) if p.flags & SC_XC else 0.0
    out["field"] = p.volume * float(st.Adot @ st.Adot) / (8.0 * np.pi * C_LIGHT**2) if p.flags & SC_MAXWELL \
        else 0.0
    out["total"] = sum(out.values())
    return out
