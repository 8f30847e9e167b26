"""The nonlocal GEMM-2 on the int8-digit tcgen05 path (csrc/nl_i8.cu, the default for FP64 contexts with
nproj, norb <= 64) against the CPU oracle and against the complex FP64 DMMA path (LFD_FLAG_NL_DMMA).

The digit scheme is exact integer arithmetic plus power-of-two scaling; the only approximation is the
truncation to 6 digits per operand and 21 digit pairs (product relative error ~3e-12, tools/i8_model.py),
scaled by the O(Delta Delta_sci / 2) size of the update: the north star's FP64 bound (1e-10 after 100
steps) applies unchanged (SURVEY §8(c) parity criterion).
"""
from __future__ import annotations

import numpy as np
import pytest

from lfd_workloads import make_inputs, workload
from lfd_workloads.generate import midpoint_A

from .test_gpu_parity import assert_parity, laser, rel, run_gpu, run_ref

pytestmark = pytest.mark.gpu

FLAG_DMMA = 8
FLAG_I8 = 16  # the parity shapes are small (< 64K points): force the int8 path where it is supported


def _ctx(w, x, flags=0):
    import torch
    from paper_conf_ipps_razakhllknvn24_b200 import Context
    dev = torch.device("cuda:0")
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    proj = torch.from_numpy(x.proj).to(dev) if w.nproj else None
    ctx = Context(psi, proj, x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc, flags=flags)
    return ctx, psi


@pytest.mark.parametrize("name,flags,path", [("P0", 0, 1), ("P0", FLAG_DMMA, 0), ("P3", 0, 0), ("C1", 0, 1),
                                             ("P1", 0, 1)])
def test_nl_path_selection(name, flags, path):
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    w = workload(name)
    x = make_inputs(w, seed=1)
    ctx, _ = _ctx(w, x, flags | FLAG_I8)
    assert lfd.lfd_nl_path(ctx.ctx) == path  # P3 has 65 projectors: the DMMA kernels
    ctx.close()


@pytest.mark.parametrize("name,path", [("C1", 0), ("C2", 1)])
def test_nl_path_default_by_grid_size(name, path):
    """default: int8 path from 64K points per domain (C2), DMMA below (C1: set-up not amortised)"""
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    w = workload(name)
    x = make_inputs(w, seed=1)
    ctx, _ = _ctx(w, x)
    assert lfd.lfd_nl_path(ctx.ctx) == path
    ctx.close()


@pytest.mark.parametrize("name,steps", [("P0", 100), ("P1", 20), ("P2z", 20), ("C1", 10)])
def test_i8_parity_against_oracle(name, steps):
    w = workload(name)
    x = make_inputs(w, seed=2)
    A = laser(w)
    assert_parity(w, run_gpu(w, x, steps, A, flags=FLAG_I8), run_ref(w, x, steps, A))


@pytest.mark.parametrize("name,steps", [("P0", 100), ("P1", 20), ("C1", 10)])
def test_dmma_path_parity_against_oracle(name, steps):
    w = workload(name)
    x = make_inputs(w, seed=2)
    A = laser(w)
    assert_parity(w, run_gpu(w, x, steps, A, flags=FLAG_DMMA), run_ref(w, x, steps, A))


def test_i8_matches_dmma_c2_full_size():
    """Bench shape (70x70x72, 64 orbitals, 64 projectors): the two GEMM-2 paths after 3 steps agree far
    inside the FP64 contract (independent arithmetic: int8 digit products vs 3M DMMA)."""
    w = workload("C2")
    x = make_inputs(w, seed=1)
    A = lambda n: midpoint_A(w, n)  # noqa: E731
    a = run_gpu(w, x, 3, A)[0]
    b = run_gpu(w, x, 3, A, flags=FLAG_DMMA)[0]
    assert rel(a, b) < 1e-12


def test_i8_ragged_tiles_and_small_shapes():
    """ng not a multiple of the 64-point tile, norb / nproj far below 64 (zero-padded digits)."""
    w = workload("P0")  # 6 x 8 x 10 = 480 points: 7.5 tiles; 7 orbitals, 5 projectors
    assert (w.nx * w.ny * w.nz) % 64 != 0
    x = make_inputs(w, seed=5)
    A = laser(w)
    got = run_gpu(w, x, 30, A, flags=FLAG_I8)
    want = run_ref(w, x, 30, A)
    assert_parity(w, got, want)


def test_i8_zero_coefficients_exact_identity():
    """D = 0: C'' = 0, every W digit and scale is zero, GEMM-2 reduces to Psi <- n Psi with n = 1; the step
    must equal the local propagator alone (nproj = 0) bit for bit."""
    w = workload("P0")
    x = make_inputs(w, seed=3)
    A = laser(w)
    a = run_gpu(w, x, 5, A, dnl=np.zeros_like(x.dnl), flags=FLAG_I8)[0]
    w0 = workload("P0")
    import dataclasses
    w0 = dataclasses.replace(w0, nproj=0)
    x0 = dataclasses.replace(x, proj=np.zeros((w.ndom, w.nx, w.ny, w.nz, 0), np.complex128),
                             dnl=np.zeros((w.ndom, 0)))
    b = run_gpu(w0, x0, 5, A)[0]
    assert np.array_equal(a, b)


@pytest.mark.parametrize("name,nproj,norb", [("P0", 5, 7), ("P0", 40, 33), ("P3", 64, 40)])
def test_i8_nonorthonormal_projectors_mixed_D(name, nproj, norb):
    """int8-digit GEMMs (forced) with NON-orthonormal projector columns (rescaled per column, so G != I and
    the per-column scales of B differ) and D_u of both signs: both GEMMs and the Gram-closed-form norm."""
    w = workload(name).with_(nproj=nproj, norb=norb, nocc=min(norb, workload(name).nocc))
    x = make_inputs(w, seed=8)
    rng = np.random.default_rng(0)
    x.proj = np.ascontiguousarray(x.proj * (0.3 + 1.5 * rng.random(x.proj.shape[-1])))
    d = np.ascontiguousarray(rng.uniform(-0.3, 0.3, size=x.dnl.shape))
    A = laser(w)
    steps = 20
    assert_parity(w, run_gpu(w, x, steps, A, dnl=d, flags=FLAG_I8), run_ref(w, x, steps, A, dnl=d))


@pytest.mark.parametrize("name", ["P0", "C1"])
def test_i8_large_scissor_gemm_accuracy(name):
    """A scissor so large that eps D ~ 0.3 (eps = Delta/2): the nonlocal update is O(|C|) of Psi instead of
    O(1e-3), so the 1e-10 Psi bound now constrains the GEMM arithmetic itself. Both GEMM paths meet the FP64
    contract after 10 steps against the oracle; the measured errors (and the implied per-factor product error
    of the int8-digit emulation, ~2^-40 of the row x column scales) are printed."""
    w = workload(name)
    x = make_inputs(w, seed=9)
    # projectors overlapping the propagated orbitals (B = B_u + Psi_0 columns: C = O(1) from the first step)
    x.proj = np.ascontiguousarray(x.proj + x.psi0[..., : w.nproj])
    d = np.ascontiguousarray(np.where(np.arange(x.dnl.size).reshape(x.dnl.shape) % 2, -1.0, 1.0)
                             * 0.3 / (0.5 * w.dt))
    A = laser(w)
    steps = 10
    want = run_ref(w, x, steps, A, dnl=d)
    base = run_ref(w, x, steps, A, dnl=np.zeros_like(d))
    gi8 = run_gpu(w, x, steps, A, dnl=d, flags=FLAG_I8)
    gdm = run_gpu(w, x, steps, A, dnl=d, flags=FLAG_DMMA)
    e_i8 = assert_parity(w, gi8, want)
    e_dm = assert_parity(w, gdm, want)
    upd = rel(want[0], base[0])  # size of the nonlocal part of the evolution (relative)
    print(f"{name} eps*D=0.3, {steps} steps: update {upd:.2e}; psi err int8 {e_i8[0]:.2e}, dmma {e_dm[0]:.2e}; "
          f"int8 vs dmma {rel(gi8[0], gdm[0]):.2e}; implied per-factor product error "
          f"{e_i8[0] / max(upd, 1e-300) / np.sqrt(2 * steps):.2e}")
    assert upd > 0.1  # the test really exercises O(1) nonlocal updates


def test_fused_first_factor_launch_classes_c2():
    """C2 default path: the first nonlocal factor's GEMM-2 runs fused with Phi . K_x (nl_fx.cu) -- per step one
    k_gemm2x_i8, no separate x pass, one plain GEMM-2 (the second factor), one GEMM-1 (the first factor's C comes
    from the projection carry after step 1)."""
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    w = workload("C2")
    x = make_inputs(w, seed=3)
    ctx, _ = _ctx(w, x)
    import torch
    ctx.set_potential(torch.from_numpy(x.vloc).to("cuda:0"))
    ctx.step(1)
    lfd.lfd_profile_enable(ctx.ctx, True)
    ctx.step(3)
    prof = lfd.lfd_profile_read(ctx.ctx)
    ctx.close()
    assert prof["nl_back_x"][1] == 3 and prof["kin_x"][1] == 0 and prof["nl_back"][1] == 3
    assert prof["kin_yz"][1] == 3 and prof["nl_proj"][1] == 3 and prof["nl_carry"][1] == 3


@pytest.mark.parametrize("name,steps,chunk", [("P0", 40, None), ("P2z", 20, 7), ("C1", 10, None)])
def test_fused_first_factor_in_sequences(name, steps, chunk):
    """merged sequences with the int8 path forced: every merged factor N o N feeds the next step's x pass through
    the fused kernel (set_A of that step enqueued before it); per-step oracle at the FP64 bound"""
    from .test_gpu_parity import run_gpu_sequence
    w = workload(name)
    x = make_inputs(w, seed=4)
    A = laser(w)
    assert_parity(w, run_gpu_sequence(w, x, steps, A, chunk, flags=FLAG_I8), run_ref(w, x, steps, A))


@pytest.mark.parametrize("name,steps", [("P0", 40), ("C1", 10)])
def test_fused_first_factor_exact_nl(name, steps):
    """the exactly unitary factor (n = 1, C'' = W C) through the fused first-factor kernel"""
    from oracle import ref
    w = workload(name)
    x = make_inputs(w, seed=5)
    A = laser(w)
    got = run_gpu(w, x, steps, A, flags=FLAG_I8 | 2)  # 2 = LFD_FLAG_EXACT_NL
    cfg = ref.RefConfig(w.ndom, w.nx, w.ny, w.nz, w.hx, w.hy, w.hz, w.bc, w.norb, w.nproj, w.dt)
    p = x.psi0.copy()
    for n in range(steps):
        ref.step_exact(cfg, p, x.proj, x.dnl, x.vloc, A(n), 1)
    assert rel(got[0], p) < 1e-10
