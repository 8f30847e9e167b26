"""GPU parity of the self-consistent LFD step (lfd_sc_*; readings R23-R28) against the
oracle's sc_step (oracle/sc.py), through the C ABI: one and several domains tiling the global grid, the
Hartree / exchange / Maxwell couplings, corrector sweeps with the projection carry, the exactly unitary
nonlocal factor, the 1-rank NCCL all-reduce path, the reduction to the plain step (flags = 0, bitwise),
and the ABI error behaviour. Tolerance: the north star's 1e-10 (FP64)."""
import numpy as np
import pytest

from lfd_workloads import domain_tiling, make_inputs, workload
from lfd_workloads.generate import laser_A

pytestmark = pytest.mark.gpu

ALL = 1 | 2 | 4


def aext_half(w, nsteps, t0=0.0):
    """A_ext at t0 + k dt/2, k = 0..2 nsteps (R28): the workload's laser, domain 0's vector."""
    return np.stack([laser_A(w, t0 + 0.5 * k * w.dt)[0] for k in range(2 * nsteps + 1)])


def _problem(w, x, flags, n_corr, exact):
    from oracle import ref, sc
    cfg = ref.RefConfig(w.ndom, w.nx, w.ny, w.nz, w.hx, w.hy, w.hz, w.bc, w.norb, w.nproj, w.dt)
    offs, gd = domain_tiling(w.ndom, (w.nx, w.ny, w.nz))
    return sc.SCProblem(cfg, x.proj, x.dnl if w.nproj else None, x.occ, x.vloc.reshape(w.ndom, -1), offs, gd,
                        flags=flags, n_corr=n_corr, exact_nl=exact)


def _ref(w, x, steps, flags, n_corr, exact=False, adot0=(3.0, -2.0, 1.0)):
    from oracle import sc
    p = _problem(w, x, flags, n_corr, exact)
    A = aext_half(w, steps)
    st = sc.sc_init(p, x.psi0.copy(), A[0], Adot0=adot0)
    sc.sc_step(p, st, A, steps)
    return st


def _gpu(w, x, steps, flags, n_corr, exact=False, adot0=(3.0, -2.0, 1.0), chunks=(None,), nccl=False, ctx_flags=0):
    import torch
    from paper_conf_ipps_razakhllknvn24_b200 import Context, lfd
    dev = torch.device("cuda:0")
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    proj = torch.from_numpy(x.proj).to(dev) if w.nproj else None
    ctx = Context(psi, proj, x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc,
                  flags=(lfd.LFD_FLAG_EXACT_NL if exact else 0) | ctx_flags)
    offs, gd = domain_tiling(w.ndom, (w.nx, w.ny, w.nz))
    vion = torch.from_numpy(x.vloc.copy()).to(dev)
    A = aext_half(w, steps)
    if nccl:  # a 1-rank communicator: lfd_sc_step then all-reduces [rho_g | Jbar] through NCCL
        lfd.lfd_sc_comm_init(ctx.ctx, 1, 0, lfd.lfd_comm_unique_id())
    ctx.sc_init(gd, offs, vion, flags=flags, n_corr=n_corr, Aext0=A[0], Adot0=adot0)
    done = 0
    for c in chunks:  # several lfd_sc_step calls continue the same trajectory
        n = steps - done if c is None else c
        ctx.sc_step(A[2 * done: 2 * (done + n) + 1])
        done += n
    assert done == steps
    st, rho, v = ctx.sc_read()
    ctx.sync()
    out = psi.cpu().numpy(), st.cpu().numpy(), rho.cpu().numpy(), v.cpu().numpy()
    ctx.close()
    return out


def rel(a, b):
    return np.linalg.norm(a - b) / max(np.linalg.norm(b), 1e-300)


def assert_sc_parity(got, st):
    psi, state, rho, v = got
    assert rel(psi, st.psi) < 1e-10
    assert rel(rho, st.rho_g) < 1e-10
    assert rel(v, st.vh) < 1e-10
    for k, ref_v in ((0, st.A_ind), (3, st.Adot), (6, st.Jbar)):
        assert np.abs(state[k:k + 3] - ref_v).max() <= 1e-10 * max(np.abs(ref_v).max(), 1.0), (k, state, ref_v)


@pytest.mark.parametrize("name,steps,flags,n_corr", [("P0", 20, ALL, 1), ("P0", 10, ALL, 0), ("P0", 8, 1 | 4, 3),
                                                     ("P1", 10, ALL, 1), ("P2z", 6, 2 | 4, 1)])
def test_sc_parity(name, steps, flags, n_corr):
    w = workload(name)
    x = make_inputs(w, seed=61)
    assert_sc_parity(_gpu(w, x, steps, flags, n_corr), _ref(w, x, steps, flags, n_corr))


@pytest.mark.parametrize("name,n_corr", [("P0", 1), ("C3", 2)])
def test_sc_parity_int8_gemms(name, n_corr):
    """the self-consistent step with both nonlocal GEMMs on the int8-digit tensor-core path (forced on these
    small grids): the out-of-place first factor S = N(Psi(t_n)), the exponent handshake across sweeps"""
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    w = workload(name).with_(vnoise=0.02) if name == "C3" else workload(name)
    x = make_inputs(w, seed=63)
    steps = 2 if name == "C3" else 12
    assert_sc_parity(_gpu(w, x, steps, ALL, n_corr, ctx_flags=lfd.LFD_FLAG_NL_I8), _ref(w, x, steps, ALL, n_corr))


def test_sc_parity_c3_eight_domains():
    """C3: 8 domains of 24^3 tiling the 48^3 global grid of the 2x2x2 supercell (v_H couples them)."""
    w = workload("C3").with_(vnoise=0.02)
    x = make_inputs(w, seed=62)
    assert_sc_parity(_gpu(w, x, 2, ALL, 1), _ref(w, x, 2, ALL, 1))


def test_sc_parity_exact_nl_many_projectors_chunked():
    """Exactly unitary nonlocal factor, 65 projectors (> one 64-wide tile), 3 corrector sweeps, the run
    split over three lfd_sc_step calls, through a 1-rank NCCL communicator (the all-reduce path)."""
    w = workload("P3")
    x = make_inputs(w, seed=63)
    got = _gpu(w, x, 5, ALL, 3, exact=True, chunks=(2, 1, 2), nccl=True)
    assert_sc_parity(got, _ref(w, x, 5, ALL, 3, exact=True))


def test_sc_without_couplings_is_the_plain_step_bitwise():
    """flags = 0: v_loc = v_ion, A = A_ext(midpoint) -- every sweep equals set_potential + set_vector_potential
    + lfd_step(1) bit for bit (the Psi copy / projection-carry snapshot of the corrector is exact)."""
    import torch
    from paper_conf_ipps_razakhllknvn24_b200 import Context
    w = workload("P0")
    x = make_inputs(w, seed=64)
    steps = 6
    got = _gpu(w, x, steps, 0, 2)
    dev = torch.device("cuda:0")
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    ctx = Context(psi, torch.from_numpy(x.proj).to(dev), x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc)
    ctx.set_potential(torch.from_numpy(x.vloc.copy()).to(dev))
    A = aext_half(w, steps)
    for n in range(steps):
        ctx.set_vector_potential(np.tile(A[2 * n + 1], (w.ndom, 1)))
        ctx.step(1)
    ctx.sync()
    assert np.array_equal(got[0], psi.cpu().numpy())
    ctx.close()


def test_sc_errors():
    import torch
    from paper_conf_ipps_razakhllknvn24_b200 import Context, LFDError, lfd
    w = workload("P1")
    x = make_inputs(w, seed=65)
    dev = torch.device("cuda:0")
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    ctx = Context(psi, torch.from_numpy(x.proj).to(dev), x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt)
    with pytest.raises(LFDError) as e:
        lfd.lfd_sc_step(ctx.ctx, np.zeros((3, 3)))
    assert e.value.status == -4  # ESTATE: no sc_init
    offs, gd = domain_tiling(w.ndom, (w.nx, w.ny, w.nz))
    for bad in (dict(n_corr=17), dict(flags=8), dict(gdims=(gd[0] + 2, gd[1], gd[2])),
                dict(offs=np.zeros_like(offs))):
        cfg, _k = lfd.make_sc_config(bad.get("flags", ALL), bad.get("n_corr", 1), bad.get("gdims", gd),
                                     bad.get("offs", offs))
        with pytest.raises(LFDError) as e:
            lfd.lfd_sc_workspace_size(ctx.ctx, cfg)
        assert e.value.status == -1
    cfg, _k = lfd.make_sc_config(ALL, 1, gd, offs, nranks=2, rank=0)
    ws = torch.empty(1 << 24, dtype=torch.uint8, device=dev)
    with pytest.raises(LFDError) as e:
        lfd.lfd_sc_init(ctx.ctx, cfg, None, ws, (0.0, 0.0, 0.0))
    assert e.value.status == -4  # nranks > 1 without a communicator
    cfg, _k = lfd.make_sc_config(ALL, 1, gd, offs)
    with pytest.raises(LFDError) as e:
        lfd.lfd_sc_init(ctx.ctx, cfg, None, ws[:64], (0.0, 0.0, 0.0))
    assert e.value.status == -2  # ENOMEM
    ctx.close()
