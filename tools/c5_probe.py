"""Probe the (norb, nproj) = (512, 64) nonlocal factor accuracy at several grid sizes: per-column / per-row-block
error pattern of one factor (lfd_step_prologue) against torch complex128 matmuls."""
import sys
import numpy as np
import torch
sys.path.insert(0, ".")
from paper_conf_ipps_razakhllknvn24_b200 import Context, lfd
from lfd_workloads.configs import workload

w = workload("C2")
for (nx, ny, nz, no, npj) in [(70, 70, 72, 512, 64), (70, 70, 72, 448, 64), (70, 70, 72, 512, 32), (70, 70, 72, 384, 64), (70, 70, 72, 512, 96), (40, 40, 40, 512, 64), (20, 20, 20, 512, 64)]:
    ng = nx * ny * nz
    g = torch.Generator(device="cuda").manual_seed(no * 7919 + npj)
    shape = (1, nx, ny, nz)
    psi = torch.randn(shape + (no,), dtype=torch.complex128, device="cuda", generator=g) * (1.0 / (w.dV * ng)) ** 0.5
    proj = torch.randn(shape + (npj,), dtype=torch.complex128, device="cuda", generator=g) * (1.0 / (w.dV * ng)) ** 0.5
    ctx = Context(psi, proj, np.full((1, npj), 0.07), np.full((1, no), 2.0), (w.hx, w.hy, w.hz), w.dt)
    path = lfd.lfd_nl_path(ctx.ctx)
    before = psi.clone()
    lfd.lfd_step_prologue(ctx.ctx)
    ctx.sync()
    P = before.reshape(ng, no)
    B = proj.reshape(ng, npj)
    C = w.dV * (B.mH @ P)
    R = P + B @ ((-0.5j * w.dt * 0.07) * C)
    nfac = torch.linalg.vector_norm(P, dim=0) / torch.linalg.vector_norm(R, dim=0)
    R = R * nfac
    got = psi.reshape(ng, no)
    E = (got - R).abs()
    upd = (R - P).abs().mean()
    acc = float(torch.linalg.vector_norm(got - R) / torch.linalg.vector_norm(R - P))
    colerr = (E.mean(0) / upd).cpu().numpy()
    rowerr = (E.reshape(-1, 64 if ng % 64 == 0 else 1, no).mean((1, 2)) / upd).cpu().numpy() if ng % 64 == 0 else None
    bad = np.nonzero(colerr > 1e-8)[0]
    # column scale check: got vs P column norms
    gn = torch.linalg.vector_norm(got, dim=0) / torch.linalg.vector_norm(P, dim=0)
    print(f"{nx}x{ny}x{nz} norb {no} nproj {npj} path {path} acc {acc:.2e} badcols {len(bad)} {bad[:12]} "
          f"norm-ratio dev {float((gn - 1).abs().max()):.2e}", flush=True)
    if len(bad):
        # the error of the bad columns: is it a scale (n) error or an update error?
        b0 = int(bad[0])
        d = got[:, b0] - R[:, b0]
        s = (d.conj() @ R[:, b0]) / (R[:, b0].conj() @ R[:, b0])
        print("   col", b0, "err", float(colerr[b0]), "scale-like component", complex(s), flush=True)
        rel_r = (d.abs() / (R[:, b0] - P[:, b0]).abs().clamp_min(1e-300)).cpu().numpy()
        big = np.nonzero(rel_r > 1e-6)[0]
        print("   rows with rel err > 1e-6:", len(big), "of", ng, big[:8], big[-4:] if len(big) else "", "median rel", float(np.median(rel_r)), flush=True)
        if rowerr is not None:
            rb = np.nonzero(rowerr > 1e-8)[0]
            print("   bad row blocks", len(rb), rb[:10], rb[-5:], flush=True)
    ctx.close()
    del psi, proj, before, P, B, C, R, got, E
    torch.cuda.empty_cache()
