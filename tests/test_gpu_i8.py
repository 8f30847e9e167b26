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


def _ctx(w, x, flags=0):
    import torch
    from paper_conf_ipps_razakhllknvn24_b200 import Context
    dev = torch.device("cuda:0")
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    proj = torch.from_numpy(x.proj).to(dev) if w.nproj else None
    ctx = Context(psi, proj, x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc, flags=flags)
    return ctx, psi


@pytest.fixture(autouse=True)
def force_i8(monkeypatch):
    """the parity shapes are small (< 64K points): force the int8 path where it is supported"""
    monkeypatch.setenv("LFD_NL_I8", "1")


@pytest.mark.parametrize("name,flags,path", [("P0", 0, 1), ("P0", FLAG_DMMA, 0), ("P3", 0, 0), ("C1", 0, 1),
                                             ("P1", 0, 1)])
def test_nl_path_selection(name, flags, path):
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    w = workload(name)
    x = make_inputs(w, seed=1)
    ctx, _ = _ctx(w, x, flags)
    assert lfd.lfd_nl_path(ctx.ctx) == path  # P3 has 65 projectors: the DMMA kernels
    ctx.close()


@pytest.mark.parametrize("name,path", [("C1", 0), ("C2", 1)])
def test_nl_path_default_by_grid_size(name, path, monkeypatch):
    """default: int8 path from 64K points per domain (C2), DMMA below (C1: set-up not amortised)"""
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    monkeypatch.delenv("LFD_NL_I8")
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
    assert_parity(w, run_gpu(w, x, steps, A), run_ref(w, x, steps, A))


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
    got = run_gpu(w, x, 30, A)
    want = run_ref(w, x, 30, A)
    assert_parity(w, got, want)


def test_i8_zero_coefficients_exact_identity():
    """D = 0: C'' = 0, every W digit and scale is zero, GEMM-2 reduces to Psi <- n Psi with n = 1; the step
    must equal the local propagator alone (nproj = 0) bit for bit."""
    w = workload("P0")
    x = make_inputs(w, seed=3)
    A = laser(w)
    a = run_gpu(w, x, 5, A, dnl=np.zeros_like(x.dnl))[0]
    w0 = workload("P0")
    import dataclasses
    w0 = dataclasses.replace(w0, nproj=0)
    x0 = dataclasses.replace(x, proj=np.zeros((w.ndom, w.nx, w.ny, w.nz, 0), np.complex128),
                             dnl=np.zeros((w.ndom, 0)))
    b = run_gpu(w0, x0, 5, A)[0]
    assert np.array_equal(a, b)
