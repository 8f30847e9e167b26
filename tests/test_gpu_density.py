"""Density / current kernel against the oracle over the geometries that select its different
decompositions: the y-marching kernel's shape (x planes per CTA, z points per plane, y chunks, ring depths) is
picked at lfd_init from the grid and the active-orbital count, so varying those covers the specialisations
(4 lanes per point with 8 or 16 orbitals each, the runtime-length loop, padded rows for odd and even counts,
warps that straddle two x planes, the periodic halo wrap and the zero-BC edges) and the generic fallback (more
active orbitals than the y-marching kernel takes). Psi is random (no propagation), the occupations are random on
the active prefix, A is generic; complex128 and complex64 (the SP variant accumulates in FP64 from the stored
single-precision values, compared with the oracle on the same values widened)."""
import numpy as np
import pytest

from lfd_workloads import make_inputs, workload

pytestmark = pytest.mark.gpu
TOL = 1e-12
TOL_SP = 1e-5

CASES = [  # (nx, ny, nz, bc, norb, nact)
    (70, 6, 72, 0, 64, 32),    # the bench's shape class (C2 planes, 32 of 64 active)
    (10, 12, 16, 0, 64, 64),   # 16 orbitals per lane
    (10, 8, 24, 0, 40, 31),    # odd active count: two pad values, runtime loop
    (6, 10, 18, 0, 33, 33),    # nz not a multiple of 8
    (7, 5, 9, 1, 5, 5),        # zero BC, odd sizes
    (8, 9, 10, 1, 64, 32),     # zero BC, 32 active
    (24, 24, 24, 0, 22, 22),   # C1
    (12, 8, 40, 0, 128, 126),  # past the y-marching kernel's limit: the generic kernel
    (4, 6, 8, 0, 3, 1),        # one active orbital
]


@pytest.mark.parametrize("sp", [False, True])
@pytest.mark.parametrize("case", CASES)
def test_density_current_shapes(case, sp):
    import torch
    from oracle import ref
    from paper_conf_ipps_razakhllknvn24_b200 import Context
    nx, ny, nz, bc, norb, nact = case
    if sp and norb % 2:
        norb += 1  # complex64 rows of an even length (TMA strides)
    w = workload("P0").with_(nx=nx, ny=ny, nz=nz, bc=bc, norb=norb, nocc=min(nact, norb), nproj=0)
    x = make_inputs(w, seed=91)
    rng = np.random.default_rng(nx * 1000 + nz + norb)
    occ = np.zeros((1, norb))
    occ[0, :nact] = rng.uniform(0.1, 2.0, size=nact)
    occ[0, nact - 1] = 1.5  # the last active orbital is occupied
    psi0 = x.psi0.astype(np.complex64) if sp else x.psi0.copy()
    dev = torch.device("cuda:0")
    psi = torch.from_numpy(psi0).to(dev)
    ctx = Context(psi, None, None, occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc)
    A = np.array([[0.31, -0.17, 0.52]])
    ctx.set_vector_potential(A)
    rho, j, J = ctx.density_current()
    ctx.sync()
    rho, j, J = rho.cpu().numpy().reshape(1, -1), j.cpu().numpy().reshape(1, 3, -1), J.cpu().numpy()
    ctx.close()
    cfg = ref.RefConfig(1, nx, ny, nz, w.hx, w.hy, w.hz, w.bc, norb, 0, w.dt)
    rr, jr, Jr = ref.density_current(cfg, psi0.astype(np.complex128), occ, A)
    e_rho = np.linalg.norm(rho - rr) / np.linalg.norm(rr)
    e_j = np.linalg.norm(j - jr) / max(np.linalg.norm(jr), 1e-3 * np.linalg.norm(rr))
    e_J = np.abs(J - Jr).max() / max(np.abs(jr).mean(), 1e-3 * np.abs(rr).mean())
    tol = TOL_SP if sp else TOL
    assert e_rho < tol and e_j < tol and e_J < tol, (case, sp, e_rho, e_j, e_J)


def test_density_active_count_changes():
    """lfd_set_occupations moves the active-orbital count across the y-marching kernel's limit (32 -> 126 -> 20 of
    128): the shape is re-chosen, then the generic kernel takes over (and stays), with the same results."""
    import torch
    from oracle import ref
    from paper_conf_ipps_razakhllknvn24_b200 import Context
    nx, ny, nz, norb = 8, 6, 24, 128
    w = workload("P0").with_(nx=nx, ny=ny, nz=nz, norb=norb, nocc=32, nproj=0)
    x = make_inputs(w, seed=17)
    dev = torch.device("cuda:0")
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    occ0 = np.zeros((1, norb))
    occ0[0, :32] = 2.0
    ctx = Context(psi, None, None, occ0, (w.hx, w.hy, w.hz), w.dt, bc=w.bc)
    A = np.array([[0.2, 0.1, -0.3]])
    ctx.set_vector_potential(A)
    cfg = ref.RefConfig(1, nx, ny, nz, w.hx, w.hy, w.hz, w.bc, norb, 0, w.dt)
    rng = np.random.default_rng(3)
    for nact in (32, 126, 20):
        occ = np.zeros((1, norb))
        occ[0, :nact] = rng.uniform(0.5, 2.0, size=nact)
        ctx.set_occupations(np.ascontiguousarray(occ))
        rho, j, J = ctx.density_current()
        ctx.sync()
        rr, jr, Jr = ref.density_current(cfg, x.psi0, occ, A)
        rho, j = rho.cpu().numpy().reshape(1, -1), j.cpu().numpy().reshape(1, 3, -1)
        assert np.linalg.norm(rho - rr) / np.linalg.norm(rr) < TOL, nact
        assert np.linalg.norm(j - jr) / max(np.linalg.norm(jr), 1e-3 * np.linalg.norm(rr)) < TOL, nact
        assert np.abs(J.cpu().numpy() - Jr).max() / max(np.abs(jr).mean(), 1e-3 * np.abs(rr).mean()) < TOL, nact
    ctx.close()
