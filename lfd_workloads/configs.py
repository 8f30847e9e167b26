"""Named workloads: BASELINE.json configs C1..C5 and the small parity shapes.

Cell geometry: tetragonal PbTiO3, a = 3.90 A = 7.370 bohr, c = 4.15 A = 7.842 bohr.
C2's 70x70x72 mesh is the paper's per-rank LFD mesh over a 2x2x2 cell
(40 atoms per rank); 64 KS orbitals.
"""
from __future__ import annotations

from dataclasses import dataclass, field, replace

BOHR_A = 7.370   # a axis [bohr]
BOHR_C = 7.842   # c axis [bohr]
DT_QD = 0.0413414  # Delta_QD = 1 as in a.u. (R19)
DELTA_SCI = 0.07   # scissor shift [Ha] (R19, synthetic)
BC_PERIODIC = 0
BC_ZERO = 1


@dataclass(frozen=True)
class Workload:
    name: str
    ndom: int
    nx: int
    ny: int
    nz: int
    cells: tuple = (1, 1, 1)   # unit cells spanned by one domain along x, y, z
    norb: int = 22
    nocc: int = 22             # first nocc orbitals have f = 2 (R14)
    nproj: int = 10
    bc: int = BC_PERIODIC
    dt: float = DT_QD
    laser: bool = False        # A(t) on (C2-C4) or A = 0 (C1)
    basis: str = "gauss"       # "gauss" (MGS-orthonormal) or "planewave" (large shapes)
    steps: int = 10
    pol: tuple = (0.0, 0.0, 1.0)  # laser polarisation (unit vector)
    a_spread: float = 0.0       # per-domain factor (1 + a_spread*dom) on A (parity shapes only)
    vnoise: float = 0.0         # amplitude of seeded white noise added to v_loc (parity shapes only)
    e0: float = 0.005           # laser field amplitude E0 [a.u.]; parity shapes use 10x
    note: str = ""

    @property
    def hx(self) -> float:
        return BOHR_A * self.cells[0] / self.nx

    @property
    def hy(self) -> float:
        return BOHR_A * self.cells[1] / self.ny

    @property
    def hz(self) -> float:
        return BOHR_C * self.cells[2] / self.nz

    @property
    def ngrid(self) -> int:
        return self.nx * self.ny * self.nz

    @property
    def dV(self) -> float:
        return self.hx * self.hy * self.hz

    @property
    def ogp_per_step(self) -> int:
        """orbital-gridpoint updates per LFD step (all domains)."""
        return self.ndom * self.ngrid * self.norb

    def with_(self, **kw) -> "Workload":
        return replace(self, **kw)


WORKLOADS = {
    # C1: 1 domain, 5-atom unit cell, 24^3, 22 occupied orbitals, 10 steps, A = 0.
    "C1": Workload("C1", 1, 24, 24, 24, (1, 1, 1), norb=22, nocc=22, nproj=10, laser=False, steps=10,
                   note="BASELINE.json configs[0]"),
    # C2: paper's single-GPU benchmark size: 70x70x72, 64 orbitals (32 occupied), 64 projectors, laser.
    "C2": Workload("C2", 1, 70, 70, 72, (2, 2, 2), norb=64, nocc=32, nproj=64, laser=True,
                   basis="planewave", steps=100, note="BASELINE.json configs[1]; bench workload"),
    # C2 with the paper-timing-consistent projector count.
    "C2p16": Workload("C2p16", 1, 70, 70, 72, (2, 2, 2), norb=64, nocc=32, nproj=16, laser=True,
                      basis="planewave", steps=100),
    # C3: 40-atom 2x2x2 supercell as 8 domains of C1 shape (cores tile a 48^3 global grid).
    "C3": Workload("C3", 8, 24, 24, 24, (1, 1, 1), norb=22, nocc=22, nproj=10, laser=True, steps=1000,
                   note="BASELINE.json configs[2]"),
    # C4: weak scaling, one C2 domain per GPU (ndom is per rank).
    "C4": Workload("C4", 1, 70, 70, 72, (2, 2, 2), norb=64, nocc=32, nproj=64, laser=True,
                   basis="planewave", steps=100, note="BASELINE.json configs[3]; per-rank load"),
    # Small parity shapes (several tiles + ragged tails; odd norb / nproj).
    "P0": Workload("P0", 1, 6, 8, 10, (1, 1, 1), norb=7, nocc=5, nproj=5, laser=True, steps=100, pol=(0.48, -0.6, 0.64), a_spread=0.1, vnoise=0.05, e0=0.05),
    "P1": Workload("P1", 2, 8, 6, 4, (1, 1, 1), norb=33, nocc=20, nproj=1, laser=True, steps=20, pol=(0.48, -0.6, 0.64), a_spread=0.1, vnoise=0.05, e0=0.05),
    "P2z": Workload("P2z", 1, 7, 5, 9, (1, 1, 1), norb=3, nocc=3, nproj=4, bc=BC_ZERO, laser=True, steps=20, pol=(0.48, -0.6, 0.64), a_spread=0.1, vnoise=0.05, e0=0.05),
    "P3": Workload("P3", 1, 10, 12, 14, (1, 1, 1), norb=40, nocc=40, nproj=65, laser=True, steps=5, pol=(0.48, -0.6, 0.64), a_spread=0.1, vnoise=0.05, e0=0.05),
}


def workload(name: str) -> Workload:
    return WORKLOADS[name]


# C5: nonlocal-projector sweep (GEMM shapes only; Ngrid = 352,800).
C5_NORB = (32, 64, 128, 256, 512)
C5_NPROJ = (64, 128, 256, 512, 1024)


def domain_tiling(ndom: int, dims) -> tuple:
    """Place ndom same-shape domains on a global grid (R18: cores tile it, buffer b = 0).

    Domains are laid out as a (px, py, pz) block grid, px * py * pz == ndom, filled x first
    (ndom = 8 -> 2x2x2 as the 2x2x2 PbTiO3 supercell of C3; 2 -> 2x1x1; 4 -> 2x2x1). Returns
    (offsets [ndom][3] int32, gdims (GX, GY, GZ)). Pure geometry, no arithmetic of the method.
    """
    import numpy as np

    p = [1, 1, 1]
    n, axis = ndom, 0
    while n > 1:
        f = 2 if n % 2 == 0 else n
        p[axis] *= f
        n //= f
        axis = (axis + 1) % 3
    offsets = np.zeros((ndom, 3), dtype=np.int32)
    for dm in range(ndom):
        ix, iy, iz = dm % p[0], (dm // p[0]) % p[1], dm // (p[0] * p[1])
        offsets[dm] = (ix * dims[0], iy * dims[1], iz * dims[2])
    return offsets, (p[0] * dims[0], p[1] * dims[1], p[2] * dims[2])
