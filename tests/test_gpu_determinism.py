"""Run-to-run determinism at full size (races show up as rare, nondeterministic differences).

Every kernel of the path has a fixed reduction order, so two runs on the same inputs must agree bit for bit.
The regression these guard: a warp's mbarrier release of a TMA-refilled shared-memory stage that did not wait
for its own shared loads still in flight -- one 8-lane phase of an LDS.128 then returned the next refill's
bytes (two rows of a GEMM-2 DMMA tile wrong in about half the runs at norb = 512, nproj = 64 on the C2 grid;
found by the C5 sweep's accuracy check). Releases now go through mbar_release (lfd_tma.cuh)."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _factor_runs(nx, ny, nz, no, npj, reps, flags=0):
    import torch
    from paper_conf_ipps_razakhllknvn24_b200 import Context, lfd
    from lfd_workloads.configs import workload
    w = workload("C2")
    ng = nx * ny * nz
    g = torch.Generator(device="cuda").manual_seed(no * 7919 + npj)
    shape = (1, nx, ny, nz)
    psi = torch.randn(shape + (no,), dtype=torch.complex128, device="cuda", generator=g) * (1.0 / (w.dV * ng)) ** 0.5
    proj = torch.randn(shape + (npj,), dtype=torch.complex128, device="cuda", generator=g) * (1.0 / (w.dV * ng)) ** 0.5
    before = psi.clone()
    outs = []
    for _ in range(reps):
        psi.copy_(before)
        ctx = Context(psi, proj, np.full((1, npj), 0.07), np.full((1, no), 2.0), (w.hx, w.hy, w.hz), w.dt, flags=flags)
        lfd.lfd_step_prologue(ctx.ctx)  # one nonlocal factor N(Psi), in place
        ctx.sync()
        outs.append(psi.reshape(ng, no).clone())
        ctx.close()
    P = before.reshape(ng, no)
    B = proj.reshape(ng, npj)
    R = P + B @ ((-0.5j * w.dt * 0.07) * (w.dV * (B.mH @ P)))
    R = R * (torch.linalg.vector_norm(P, dim=0) / torch.linalg.vector_norm(R, dim=0))
    acc = [float(torch.linalg.vector_norm(o - R) / torch.linalg.vector_norm(R - P)) for o in outs]
    same = [bool(torch.equal(o, outs[0])) for o in outs[1:]]
    return acc, same


def test_wide_orbital_factor_deterministic_at_c2_grid():
    """(norb, nproj) = (512, 64) on the 352,800-point grid (FP64 DMMA GEMMs, k_gemm2_tma): 4 runs, bitwise equal,
    each within 1e-9 of a cuBLAS ZGEMM evaluation of the factor (relative to the update)"""
    acc, same = _factor_runs(70, 70, 72, 512, 64, 4)
    assert all(same), (acc, same)
    assert max(acc) < 1e-9, acc


@pytest.mark.parametrize("flags", [0, 8])  # default (int8-digit GEMMs + fused x pass), LFD_FLAG_NL_DMMA
def test_c2_steps_bitwise_repeatable(flags):
    """three C2 steps + density from the same inputs, twice: Psi and rho bit for bit"""
    import torch
    from paper_conf_ipps_razakhllknvn24_b200 import Context
    from lfd_workloads import make_inputs, workload
    from lfd_workloads.generate import midpoint_A
    w = workload("C2")
    x = make_inputs(w, seed=5)
    dev = torch.device("cuda:0")
    res = []
    for _ in range(2):
        psi = torch.from_numpy(x.psi0).to(dev)
        ctx = Context(psi, torch.from_numpy(x.proj).to(dev), x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt, flags=flags)
        ctx.set_potential(torch.from_numpy(x.vloc).to(dev))
        ctx.step_sequence(np.stack([midpoint_A(w, n) for n in range(3)]))
        rho, _, J = ctx.density_current()
        ctx.sync()
        res.append((psi.clone(), rho.clone(), J.clone()))
        ctx.close()
    for a, b in zip(res[0], res[1]):
        assert torch.equal(a, b)
