"""GPU-vs-oracle parity (the contract of SURVEY §8(c)): the CUDA path through the C ABI against the
plain-C oracle on identical seeded inputs, element by element.

Criterion (FP64, SURVEY §8(c) "GPU-vs-oracle parity criterion"):
  ||Psi_gpu - Psi_ref||_F / ||Psi_ref||_F <= 1e-10, the same 2-norm ratio for rho and for j (j's
  denominator floored at 1e-3 ||rho||_2 / min(h)), and |J_gpu - J_ref| <= 1e-10 mean|j_ref| (floored
  likewise). Legitimate differences are roundoff only: DMMA / FMA contraction and summation order in the
  K = Ngrid reductions, the Gram-closed-form norm (GPU) vs direct grid sums (oracle), CUDA sincos vs
  libm (reading R22).
"""
from __future__ import annotations

import numpy as np
import pytest

from lfd_workloads import make_inputs, workload
from lfd_workloads.generate import midpoint_A

pytestmark = pytest.mark.gpu

TOL = 1e-10


def _torch():
    import torch
    return torch


def run_gpu(w, x, steps, A_fn, dnl=None, flags=0):
    torch = _torch()
    from paper_conf_ipps_razakhllknvn24_b200 import Context
    dev = torch.device("cuda:0")
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    proj = torch.from_numpy(x.proj).to(dev) if w.nproj > 0 else None
    ctx = Context(psi, proj, x.dnl if dnl is None else dnl, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc,
                  flags=flags)
    ctx.set_potential(torch.from_numpy(x.vloc).to(dev))
    A = np.zeros((w.ndom, 3))
    for n in range(steps):
        A = A_fn(n)
        ctx.set_vector_potential(A)
        ctx.step(1)
    ctx.set_vector_potential(A)
    rho, j, J = ctx.density_current()
    ctx.sync()
    out = (psi.cpu().numpy(), rho.cpu().numpy().reshape(w.ndom, -1), j.cpu().numpy().reshape(w.ndom, 3, -1),
           J.cpu().numpy())
    ctx.close()
    return out


def run_ref(w, x, steps, A_fn, dnl=None):
    from oracle import ref
    cfg = ref.RefConfig(w.ndom, w.nx, w.ny, w.nz, w.hx, w.hy, w.hz, w.bc, w.norb, w.nproj, w.dt)
    p = x.psi0.copy()
    A = np.zeros((w.ndom, 3))
    d = x.dnl if dnl is None else dnl
    for n in range(steps):
        A = A_fn(n)
        ref.step(cfg, p, x.proj if w.nproj else None, d if w.nproj else None, x.vloc, A, 1)
    rho, j, J = ref.density_current(cfg, p, x.occ, A)
    return p, rho, j, J


def rel(a, b):
    return np.linalg.norm(a - b) / np.linalg.norm(b)


def assert_parity(w, got, want, tol=TOL):
    psi, rho, j, J = got
    rpsi, rrho, rj, rJ = want
    e_psi = rel(psi, rpsi)
    e_rho = rel(rho, rrho)
    floor = 1e-3 * np.linalg.norm(rrho) / min(w.hx, w.hy, w.hz)
    e_j = np.linalg.norm(j - rj) / max(np.linalg.norm(rj), floor)
    jscale = max(np.abs(rj).mean(), 1e-3 * np.abs(rrho).mean() / min(w.hx, w.hy, w.hz))
    e_J = np.abs(J - rJ).max() / jscale
    assert e_psi <= tol and e_rho <= tol and e_j <= tol and e_J <= tol, (e_psi, e_rho, e_j, e_J)
    return e_psi, e_rho, e_j, e_J


def laser(w):
    return lambda n: midpoint_A(w, n)


@pytest.mark.parametrize("name,steps", [("P0", 100), ("P1", 20), ("P2z", 20), ("P3", 5)])
def test_step_parity_small_shapes(name, steps):
    w = workload(name)
    x = make_inputs(w, seed=7)
    assert_parity(w, run_gpu(w, x, steps, laser(w)), run_ref(w, x, steps, laser(w)))


def test_c1_as_specified_10_steps_A0():
    """BASELINE configs[0]: 1 domain, 24^3, 22 occupied orbitals, 10 steps, A = 0."""
    w = workload("C1")
    x = make_inputs(w, seed=1)
    A0 = lambda n: np.zeros((1, 3))
    assert_parity(w, run_gpu(w, x, 10, A0), run_ref(w, x, 10, A0))


def test_c1_contract_100_steps_laser_and_scissor():
    """100 steps, A(t) != 0 and D != 0 (C1 shape, laser along a generic direction)."""
    w = workload("C1").with_(laser=True, pol=(0.3, -0.4, 0.87), e0=0.02)
    x = make_inputs(w, seed=2)
    assert_parity(w, run_gpu(w, x, 100, laser(w)), run_ref(w, x, 100, laser(w)))


def test_c3_eight_domain_batch():
    """BASELINE configs[2]: 8 DC domains of the C1 shape batched in one context (20 steps)."""
    w = workload("C3").with_(a_spread=0.1, vnoise=0.02)
    x = make_inputs(w, seed=3)
    assert_parity(w, run_gpu(w, x, 20, laser(w)), run_ref(w, x, 20, laser(w)))


def test_local_only_nproj0():
    w = workload("P0").with_(nproj=0)
    x = make_inputs(w, seed=4)
    assert_parity(w, run_gpu(w, x, 50, laser(w)), run_ref(w, x, 50, laser(w)))


@pytest.mark.parametrize("dims,bc,norb,nproj", [((2, 4, 2), 0, 1, 1), ((3, 2, 5), 1, 1, 0), ((2, 2, 2), 1, 2, 1),
                                                ((4, 6, 130), 0, 2, 3), ((130, 4, 2), 0, 3, 2)])
def test_edge_shapes(dims, bc, norb, nproj):
    w = workload("P0").with_(nx=dims[0], ny=dims[1], nz=dims[2], bc=bc, norb=norb, nocc=norb, nproj=nproj)
    x = make_inputs(w, seed=5)
    assert_parity(w, run_gpu(w, x, 7, laser(w)), run_ref(w, x, 7, laser(w)))


def test_ragged_gemm_tiles():
    """norb and nproj not multiples of the 64-wide tiles / 16-row chunks; several tiles each way."""
    w = workload("P0").with_(nx=8, ny=10, nz=12, norb=70, nocc=35, nproj=67)
    x = make_inputs(w, seed=6)
    assert_parity(w, run_gpu(w, x, 3, laser(w)), run_ref(w, x, 3, laser(w)))


def test_nonorthonormal_projectors_and_mixed_D():
    """B need not be orthonormal (G = dV B^H B is used); D_u of both signs."""
    w = workload("P3")
    x = make_inputs(w, seed=8)
    rng = np.random.default_rng(0)
    x.proj = np.ascontiguousarray(x.proj * (0.5 + rng.random(x.proj.shape[-1])))
    d = np.ascontiguousarray(rng.uniform(-0.3, 0.3, size=x.dnl.shape))
    assert_parity(w, run_gpu(w, x, 5, laser(w), dnl=d), run_ref(w, x, 5, laser(w), dnl=d))


def test_c2_full_size_one_step():
    """BASELINE configs[1] at full size (70x70x72, 64 orbitals, 64 projectors, laser), same launch
    configuration bench.py times: 2 steps compared element by element with the oracle (~20 s CPU)."""
    w = workload("C2")
    x = make_inputs(w, seed=1)
    assert_parity(w, run_gpu(w, x, 2, laser(w)), run_ref(w, x, 2, laser(w)))


def test_deterministic_bitwise():
    w = workload("P3")
    x = make_inputs(w, seed=9)
    a = run_gpu(w, x, 3, laser(w))
    b = run_gpu(w, x, 3, laser(w))
    for u, v in zip(a, b):
        assert np.array_equal(u, v)


def test_norm_conservation_on_gpu():
    w = workload("P0")
    x = make_inputs(w, seed=10)
    psi, *_ = run_gpu(w, x, 100, laser(w))
    P = psi.reshape(-1, w.norb)
    assert np.abs(w.dV * np.einsum("rs,rs->s", P.conj(), P).real - 1).max() < 1e-12


def test_host_buffer_pipeline_double_buffered():
    """the host-buffer calls with their copies on side streams: a caller that double-buffers v_loc and the
    outputs and reads step n's rho / J (lfd_wait_host_outputs(1)) while step n+1 runs gets, step by step,
    exactly the device-path values"""
    torch = _torch()
    from paper_conf_ipps_razakhllknvn24_b200 import Context, lfd
    w = workload("C1")
    x = make_inputs(w, seed=12)
    dev = torch.device("cuda:0")
    nsteps = 6
    vs = [x.vloc * (1.0 + 0.02 * n) for n in range(nsteps)]
    # reference: device buffers, synchronous reads
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    ctx = Context(psi, torch.from_numpy(x.proj).to(dev), x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt)
    want = []
    for n in range(nsteps):
        ctx.set_potential(torch.from_numpy(vs[n]).to(dev))
        ctx.set_vector_potential(midpoint_A(w, n))
        ctx.step(1)
        rho, _, J = ctx.density_current()
        ctx.sync()
        want.append((rho.cpu().clone(), J.cpu().clone()))
    ctx.close()
    # pipelined host-buffer loop
    psi2 = torch.from_numpy(x.psi0.copy()).to(dev)
    ctx2 = Context(psi2, torch.from_numpy(x.proj).to(dev), x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt)
    vh = [torch.empty(vs[0].shape, dtype=torch.float64).pin_memory() for _ in range(2)]
    rh = [torch.empty((w.ndom, w.nx, w.ny, w.nz), dtype=torch.float64).pin_memory() for _ in range(2)]
    Jh = [torch.empty((w.ndom, 3), dtype=torch.float64).pin_memory() for _ in range(2)]
    got = []
    for n in range(nsteps):
        vh[n % 2].copy_(torch.from_numpy(vs[n]))  # its previous H2D (step n-2) has run: see the wait below
        lfd.lfd_set_potential_host(ctx2.ctx, vh[n % 2])
        lfd.lfd_set_vector_potential(ctx2.ctx, midpoint_A(w, n))
        lfd.lfd_step(ctx2.ctx, 1)
        lfd.lfd_density_current_host(ctx2.ctx, rh[n % 2], Jh[n % 2])
        if n >= 1:
            lfd.lfd_wait_host_outputs(ctx2.ctx, 1)
            got.append((rh[(n - 1) % 2].clone(), Jh[(n - 1) % 2].clone()))
    lfd.lfd_wait_host_outputs(ctx2.ctx, 0)
    got.append((rh[(nsteps - 1) % 2].clone(), Jh[(nsteps - 1) % 2].clone()))
    with pytest.raises(lfd.LFDError):
        lfd.lfd_wait_host_outputs(ctx2.ctx, 2)
    ctx2.sync()
    assert torch.equal(psi, psi2)
    for (r1, J1), (r2, J2) in zip(want, got):
        assert torch.equal(r1.reshape(r2.shape), r2) and torch.equal(J1, J2)
    ctx2.close()


def test_global_layout_and_host_variants():
    torch = _torch()
    from paper_conf_ipps_razakhllknvn24_b200 import Context, lfd
    w = workload("P1")
    x = make_inputs(w, seed=11)
    dev = torch.device("cuda:0")
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    ctx = Context(psi, torch.from_numpy(x.proj).to(dev), x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt)
    ctx.set_potential(x.vloc)  # host path
    ctx.set_vector_potential(midpoint_A(w, 0))
    ctx.step(2)
    rho, j, J = ctx.density_current()
    gd = np.array([w.nx * 2, w.ny, w.nz], dtype=np.int32)
    off = np.array([[0, 0, 0], [w.nx, 0, 0]], dtype=np.int32)
    rg = torch.zeros(tuple(gd), dtype=torch.float64, device=dev)
    jg = torch.zeros((3,) + tuple(gd), dtype=torch.float64, device=dev)
    Jg = torch.zeros((2, 3), dtype=torch.float64, device=dev)
    lfd.lfd_density_current_global(ctx.ctx, rg, jg, Jg, off, gd)
    rh = torch.empty((2, w.nx, w.ny, w.nz), dtype=torch.float64).pin_memory()
    Jh = torch.empty((2, 3), dtype=torch.float64).pin_memory()
    lfd.lfd_density_current_host(ctx.ctx, rh, Jh)
    ctx.sync()
    assert torch.equal(rg[: w.nx].cpu(), rho[0].cpu()) and torch.equal(rg[w.nx:].cpu(), rho[1].cpu())
    assert torch.equal(jg[:, : w.nx].cpu(), j[0].cpu()) and torch.equal(jg[:, w.nx:].cpu(), j[1].cpu())
    assert torch.equal(Jg.cpu(), J.cpu()) and torch.equal(Jh, J.cpu()) and torch.equal(rh, rho.cpu())
    # device-path potential gives the same state as the host path
    psi2 = torch.from_numpy(x.psi0.copy()).to(dev)
    ctx2 = Context(psi2, torch.from_numpy(x.proj).to(dev), x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt)
    ctx2.set_potential(torch.from_numpy(x.vloc).to(dev))
    ctx2.set_vector_potential(midpoint_A(w, 0))
    ctx2.step(2)
    ctx2.sync()
    assert torch.equal(psi, psi2)
    ctx.close()
    ctx2.close()


def test_abi_errors_change_no_state():
    torch = _torch()
    from paper_conf_ipps_razakhllknvn24_b200 import Context, lfd
    w = workload("P0")
    x = make_inputs(w, seed=12)
    dev = torch.device("cuda:0")
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    ctx = Context(psi, torch.from_numpy(x.proj).to(dev), x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt)
    before = psi.clone()
    with pytest.raises(lfd.LFDError) as e:
        lfd.lfd_step(ctx.ctx, -1)
    assert e.value.status == -1
    with pytest.raises(lfd.LFDError):
        lfd.lfd_set_vector_potential(ctx.ctx, np.full((1, 3), np.nan))
    with pytest.raises(lfd.LFDError):  # host memory where device memory is required
        lfd._check(lfd.load().lfd_set_potential(ctx.ctx, lfd.C.c_void_p(x.vloc.ctypes.data)), ctx.ctx)
    ctx.sync()
    assert torch.equal(psi, before)
    # workspace too small
    cfg = ctx.cfg
    small = torch.empty(256, dtype=torch.uint8, device=dev)
    with pytest.raises(lfd.LFDError) as e:
        lfd.lfd_init(cfg, psi, torch.from_numpy(x.proj).to(dev), x.dnl, x.occ, small)
    assert e.value.status == -2
    # host psi rejected
    with pytest.raises(lfd.LFDError):
        occ = np.ascontiguousarray(x.occ)
        lfd._check(lfd.load().lfd_init(lfd.C.byref(cfg), lfd.C.c_void_p(x.psi0.ctypes.data),
                                       lfd.C.c_void_p(x.proj.ctypes.data), lfd.C.c_void_p(x.dnl.ctypes.data),
                                       lfd.C.c_void_p(occ.ctypes.data), lfd.C.c_void_p(small.data_ptr()),
                                       1 << 30, None, lfd.C.byref(lfd.C.c_void_p())))
    h = ctx.ctx
    ctx.close()
    with pytest.raises(lfd.LFDError) as e:
        lfd.lfd_step(h, 1)
    assert e.value.status == -4  # LFD_ESTATE after destroy


def test_launch_count_and_profile():
    torch = _torch()
    from paper_conf_ipps_razakhllknvn24_b200 import Context, lfd
    w = workload("P0")
    x = make_inputs(w, seed=13)
    dev = torch.device("cuda:0")
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    ctx = Context(psi, torch.from_numpy(x.proj).to(dev), x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt)
    n0 = lfd.lfd_launch_count(ctx.ctx)
    lfd.lfd_profile_enable(ctx.ctx, True)
    ctx.step(2)
    prof = lfd.lfd_profile_read(ctx.ctx)
    # step 1: N (GEMM-1, reduce, norm, GEMM-2), the stencil passes (Phi.K_x, then Phi.K_y K_z fused), N;
    # step 2's first N takes C and n from the projection carry (one kernel) instead of GEMM-1 + reduce + norm
    assert prof["kin_x"][1] == 2 and prof["kin_yz"][1] == 2 and prof["kin_y"][1] == 0
    assert lfd.lfd_launch_count(ctx.ctx) - n0 == sum(v[1] for v in prof.values()) == 10 + 8
    assert prof["nl_proj"][1] == 3 and prof["nl_back"][1] == 4 and prof["nl_norm"][1] == 3
    assert prof["nl_carry"][1] == 1
    assert all(v[0] >= 0 for v in prof.values())
    ctx.close()


def run_gpu_sequence(w, x, steps, A_fn, chunk=None, flags=0):
    torch = _torch()
    from paper_conf_ipps_razakhllknvn24_b200 import Context
    dev = torch.device("cuda:0")
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    proj = torch.from_numpy(x.proj).to(dev) if w.nproj > 0 else None
    ctx = Context(psi, proj, x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc, flags=flags)
    ctx.set_potential(torch.from_numpy(x.vloc).to(dev))
    A_seq = np.stack([A_fn(n) for n in range(steps)])
    chunk = chunk or steps
    for s0 in range(0, steps, chunk):
        ctx.step_sequence(A_seq[s0:s0 + chunk])
    rho, j, J = ctx.density_current()
    ctx.sync()
    out = (psi.cpu().numpy(), rho.cpu().numpy().reshape(w.ndom, -1), j.cpu().numpy().reshape(w.ndom, 3, -1),
           J.cpu().numpy())
    ctx.close()
    return out


@pytest.mark.parametrize("name,steps,chunk", [("P0", 100, None), ("P1", 20, 7), ("P2z", 20, None), ("P3", 6, None),
                                              ("C1", 30, None)])
def test_step_sequence_parity(name, steps, chunk):
    """lfd_step_sequence (adjacent nonlocal factors merged, N o N = renormalised L^2) equals the oracle
    stepping one Eq.-6 step at a time with the same per-step A."""
    w = workload(name) if name != "C1" else workload("C1").with_(laser=True, e0=0.02, pol=(0.3, -0.4, 0.87))
    x = make_inputs(w, seed=31)
    assert_parity(w, run_gpu_sequence(w, x, steps, laser(w), chunk), run_ref(w, x, steps, laser(w)))


def test_c2_full_size_sequence():
    """The merged-factor sequence at the bench size (C2), 3 steps, vs the oracle."""
    w = workload("C2")
    x = make_inputs(w, seed=2)
    assert_parity(w, run_gpu_sequence(w, x, 3, laser(w)), run_ref(w, x, 3, laser(w)))


@pytest.mark.parametrize("name,steps", [("P0", 60), ("P3", 6), ("C1", 12)])
def test_projection_carry_vs_no_carry(name, steps):
    """The projection carry (C of a factor that directly follows another from C_new = (C + G C') n)
    agrees with recomputing C by GEMM-1 every factor (LFD_FLAG_NO_CARRY) to roundoff, and both meet
    the oracle."""
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    w = workload(name) if name != "C1" else workload("C1").with_(laser=True, e0=0.02, pol=(0.3, -0.4, 0.87))
    x = make_inputs(w, seed=41)
    a = run_gpu(w, x, steps, laser(w))
    b = run_gpu(w, x, steps, laser(w), flags=lfd.LFD_FLAG_NO_CARRY)
    assert rel(a[0], b[0]) < 1e-13
    want = run_ref(w, x, steps, laser(w))
    assert_parity(w, a, want)
    assert_parity(w, b, want)


def test_psi_modified_drops_the_carry():
    """Writing psi between steps and calling lfd_psi_modified gives the oracle's result from the
    written state (the kept projection is not reused)."""
    torch = _torch()
    from oracle import ref
    from paper_conf_ipps_razakhllknvn24_b200 import Context
    w = workload("P0")
    x = make_inputs(w, seed=42)
    dev = torch.device("cuda:0")
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    ctx = Context(psi, torch.from_numpy(x.proj).to(dev), x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc)
    ctx.set_potential(torch.from_numpy(x.vloc).to(dev))
    cfg = ref.RefConfig(w.ndom, w.nx, w.ny, w.nz, w.hx, w.hy, w.hz, w.bc, w.norb, w.nproj, w.dt)
    p = x.psi0.copy()
    phase = np.exp(0.7j * np.arange(w.norb))
    for n in range(6):
        A = midpoint_A(w, n)
        if n == 3:  # the caller rotates every orbital's phase and swaps two orbitals
            ctx.sync()
            q = psi.cpu().numpy() * phase
            q[..., [0, 1]] = q[..., [1, 0]]
            psi.copy_(torch.from_numpy(np.ascontiguousarray(q)))
            ctx.psi_modified()
            p = p * phase
            p[..., [0, 1]] = p[..., [1, 0]]
            p = np.ascontiguousarray(p)
        ctx.set_vector_potential(A)
        ctx.step(1)
        ref.step(cfg, p, x.proj, x.dnl, x.vloc, A, 1)
    ctx.sync()
    assert rel(psi.cpu().numpy(), p) < TOL
    ctx.close()


def test_set_occupations_changes_active_orbitals():
    """The density reads only orbitals up to the last nonzero occupation; lfd_set_occupations moves
    that bound (here from 20 to all 33 orbitals of P1 and back to 5) and the results follow the
    oracle's full sums exactly as before."""
    torch = _torch()
    from oracle import ref
    from paper_conf_ipps_razakhllknvn24_b200 import Context
    w = workload("P1")
    x = make_inputs(w, seed=43)
    dev = torch.device("cuda:0")
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    ctx = Context(psi, torch.from_numpy(x.proj).to(dev), x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc)
    ctx.set_potential(torch.from_numpy(x.vloc).to(dev))
    A = midpoint_A(w, 0)
    ctx.set_vector_potential(A)
    ctx.step(2)
    cfg = ref.RefConfig(w.ndom, w.nx, w.ny, w.nz, w.hx, w.hy, w.hz, w.bc, w.norb, w.nproj, w.dt)
    p = x.psi0.copy()
    ref.step(cfg, p, x.proj, x.dnl, x.vloc, A, 2)
    rng = np.random.default_rng(1)
    for occ in (rng.uniform(0.0, 2.0, size=(w.ndom, w.norb)), np.pad(np.full((w.ndom, 5), 2.0), ((0, 0), (0, w.norb - 5))),
                x.occ):
        occ = np.ascontiguousarray(occ)
        ctx.set_occupations(occ)
        rho, j, J = ctx.density_current()
        ctx.sync()
        rr, jr, Jr = ref.density_current(cfg, p, occ, A)
        assert rel(rho.cpu().numpy().reshape(rr.shape), rr) < TOL
        assert np.linalg.norm(j.cpu().numpy().reshape(jr.shape) - jr) <= TOL * max(np.linalg.norm(jr), 1e-3 * np.linalg.norm(rr))
    ctx.close()


def test_c2_contract_100_steps():
    """The north-star contract at the bench configuration: C2 (70x70x72, 64 orbitals, 64 projectors, laser;
    the default int8-digit GEMMs that bench.py times) for 100 steps. The oracle runs the same 100 steps on 6
    orbital columns spread over both halves of the orbital range (orbitals evolve independently under Eq. 6,
    so these are exactly those columns of a full run; tests/_oracle_par.py), compared at 1e-10 in Psi; rho, j
    and J of those columns (occupations moved onto them with lfd_set_occupations) at 1e-10."""
    torch = _torch()
    from oracle import ref
    from paper_conf_ipps_razakhllknvn24_b200 import Context, lfd
    from tests._oracle_par import oracle_columns
    w = workload("C2")
    x = make_inputs(w, seed=5)
    cols = [0, 1, 17, 31, 32, 63]
    steps = 100
    dev = torch.device("cuda:0")
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    ctx = Context(psi, torch.from_numpy(x.proj).to(dev), x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc)
    assert lfd.lfd_nl_path(ctx.ctx) == 1  # the bench configuration: int8-digit tensor-core GEMMs
    ctx.set_potential(torch.from_numpy(x.vloc).to(dev))
    for n in range(steps):
        ctx.set_vector_potential(midpoint_A(w, n))
        ctx.step(1)
    occ = np.zeros((1, w.norb))
    occ[0, cols] = 2.0
    ctx.set_occupations(occ)
    rho, j, J = ctx.density_current()
    ctx.sync()
    got = psi.cpu().numpy()[..., cols]
    rho, j, J = rho.cpu().numpy().reshape(1, -1), j.cpu().numpy().reshape(1, 3, -1), J.cpu().numpy()
    ctx.close()
    want, A = oracle_columns("C2", 5, cols, steps)
    cfg = ref.RefConfig(1, w.nx, w.ny, w.nz, w.hx, w.hy, w.hz, w.bc, len(cols), w.nproj, w.dt)
    rr, jr, Jr = ref.density_current(cfg, want, np.full((1, len(cols)), 2.0), A)
    ws = w.with_(norb=len(cols))
    errs = assert_parity(ws, (got, rho, j, J), (want, rr, jr, Jr))
    print(f"C2 100 steps (int8 GEMMs) vs oracle: psi {errs[0]:.2e} rho {errs[1]:.2e} j {errs[2]:.2e} J {errs[3]:.2e}")


def test_step_prologue_overlap_schedule_bitwise():
    """The multi-GPU overlap schedule on one process (a dry run of bench.py's N > 1 loop): the first nonlocal
    factor of step n+1 enqueued by lfd_step_prologue right after step n's density (where the density
    all-gather would run on a side stream), then v / A and lfd_step. Bitwise equal to the serial call order
    (same kernels, same data dependencies), and observers of Psi are refused while a prologue is pending."""
    torch = _torch()
    from paper_conf_ipps_razakhllknvn24_b200 import Context, lfd
    w = workload("P0")
    x = make_inputs(w, seed=14)
    dev = torch.device("cuda:0")
    outs = []
    for overlap in (False, True):
        psi = torch.from_numpy(x.psi0.copy()).to(dev)
        ctx = Context(psi, torch.from_numpy(x.proj).to(dev), x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc)
        v = torch.from_numpy(x.vloc).to(dev)
        rhos, Js = [], []
        for n in range(12):
            lfd.lfd_set_vector_potential(ctx.ctx, midpoint_A(w, n))
            lfd.lfd_set_potential(ctx.ctx, v)
            lfd.lfd_step(ctx.ctx, 1)
            rho, _, J = ctx.density_current()
            rhos.append(rho.clone())
            Js.append(J.clone())
            if overlap and n < 11:
                lfd.lfd_step_prologue(ctx.ctx)
                if n == 3:
                    with pytest.raises(lfd.LFDError) as e:
                        ctx.density_current()
                    assert e.value.status == -4
                    with pytest.raises(lfd.LFDError):
                        lfd.lfd_step_prologue(ctx.ctx)
        ctx.sync()
        outs.append((psi.cpu().numpy(), torch.stack(rhos).cpu().numpy(), torch.stack(Js).cpu().numpy()))
        ctx.close()
    for a, b in zip(*outs):
        assert np.array_equal(a, b)


@pytest.mark.parametrize("norb,nproj,dims", [(20, 100, (8, 10, 12)), (32, 65, (10, 12, 14)), (9, 40, (8, 6, 10))])
def test_narrow_orbital_tiles(norb, nproj, dims):
    """norb <= 32 (C5's first row): GEMM-1 with 32-wide orbital tiles and, for nproj > 64, the 128 x 32 GEMM-2
    tile -- ragged in every direction -- against the oracle."""
    w = workload("P0").with_(nx=dims[0], ny=dims[1], nz=dims[2], norb=norb, nocc=min(norb, 12), nproj=nproj)
    x = make_inputs(w, seed=15)
    assert_parity(w, run_gpu(w, x, 4, laser(w)), run_ref(w, x, 4, laser(w)))


@pytest.mark.parametrize("norb,nproj,dims", [(512, 64, (8, 10, 12)), (130, 64, (8, 6, 10)), (200, 30, (10, 8, 6))])
def test_wide_orbital_sets_short_projector_tile(norb, nproj, dims):
    """norb > 64 with nproj <= 64 (C5's nproj = 64 column: the TMA GEMM-2 over several orbital tiles, GEMM-1 with
    one projector tile and several orbital tiles) against the oracle."""
    w = workload("P0").with_(nx=dims[0], ny=dims[1], nz=dims[2], norb=norb, nocc=min(norb, 40), nproj=nproj)
    x = make_inputs(w, seed=16)
    assert_parity(w, run_gpu(w, x, 3, laser(w)), run_ref(w, x, 3, laser(w)))


def test_large_nproj_carry_and_sequence():
    """nproj = 1300 (> 1228: the projection carry's D / x / DC staging needs more than the 48 KB default dynamic
    shared memory, k_nlmerge too): steps with the carry and a merged-factor sequence against the oracle."""
    w = workload("P0").with_(nx=8, ny=8, nz=8, norb=4, nocc=4, nproj=1300)
    x = make_inputs(w, seed=97)
    dnl = np.ascontiguousarray(np.full((1, w.nproj), 0.07))
    A = laser(w)
    assert_parity(w, run_gpu(w, x, 2, A, dnl=dnl), run_ref(w, x, 2, A, dnl=dnl))
    assert_parity(w, run_gpu_sequence(w, x, 2, A), run_ref(w, x, 2, A))
