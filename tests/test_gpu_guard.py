"""Bounds checks of our own (the GPU pool refuses compute-sanitizer): every caller buffer the library touches --
Psi, B, the workspace, rho, j, J, the energies, the remap output -- is a view into a larger allocation whose guard
bands before and after are filled with a sentinel bit pattern; after steps, the merged-factor sequence, the density,
the energy and remap_occ on the tiny shapes of tools/sanitize_drive.py (every kernel variant: periodic / zero BC,
nproj 0 / < 64 / not a multiple of 4 / > 64, the int8-digit tcgen05 GEMMs forced incl. the fused first factor, the
SP variant) the guards must be bitwise unchanged and Psi finite. An out-of-bounds write of any kernel into a
neighbouring allocation lands in a guard band here. Reads past the end are not detected by this test; the parity
tests catch reads of wrong data."""
import numpy as np
import pytest
import torch

from lfd_workloads import make_inputs, workload
from lfd_workloads.generate import midpoint_A
from paper_conf_ipps_razakhllknvn24_b200 import lfd

pytestmark = pytest.mark.gpu
GB = 4096  # guard bytes on each side (a multiple of 1024: the views keep the allocation's alignment)


class Guarded:
    """A byte buffer [guard | payload | guard]; payload views of any dtype; check() compares the guards."""

    def __init__(self, nbytes, dev, fill=0xA5):
        self.n = int(nbytes)
        self.raw = torch.full((self.n + 2 * GB,), fill, dtype=torch.uint8, device=dev)
        self.fill = fill

    def view(self, dtype, shape):
        return self.raw[GB:GB + self.n].view(dtype).view(shape)

    def check(self, what):
        lo, hi = self.raw[:GB], self.raw[GB + self.n:]
        bad = int((lo != self.fill).sum()) + int((hi != self.fill).sum())
        assert bad == 0, f"{what}: {bad} guard bytes overwritten"


def _nbytes(shape, dtype):
    return int(np.prod(shape)) * torch.empty((), dtype=dtype).element_size()


def _shapes(mode):
    if mode == "i8":
        return [workload("P0"), workload("P1"), workload("P0").with_(nx=8, ny=8, nz=70, norb=64, nocc=32, nproj=64),
                workload("P0").with_(nx=70, ny=4, nz=6, norb=64, nocc=32, nproj=64)]
    return [workload("P0"), workload("P2z"), workload("P3").with_(nx=6, ny=6, nz=8), workload("P1"),
            workload("P0").with_(nproj=0), workload("P0").with_(nz=90, nproj=7)]


@pytest.mark.parametrize("mode", ["dmma", "i8", "sp"])
def test_guard_bands_untouched(mode):
    dev = torch.device("cuda:0")
    cdt = torch.complex64 if mode == "sp" else torch.complex128
    ncdt = np.complex64 if mode == "sp" else np.complex128
    flags = lfd.LFD_FLAG_NL_I8 if mode == "i8" else 0
    if mode == "sp":
        flags |= lfd.LFD_FLAG_SP
    for w in _shapes(mode):
        x = make_inputs(w, seed=5)
        shp = (w.ndom, w.nx, w.ny, w.nz)
        bufs = {}
        bufs["psi"] = Guarded(_nbytes(shp + (w.norb,), cdt), dev)
        psi = bufs["psi"].view(cdt, shp + (w.norb,))
        psi.copy_(torch.from_numpy(x.psi0.astype(ncdt)))
        proj = None
        if w.nproj:
            bufs["proj"] = Guarded(_nbytes(shp + (w.nproj,), cdt), dev)
            proj = bufs["proj"].view(cdt, shp + (w.nproj,))
            proj.copy_(torch.from_numpy(x.proj.astype(ncdt)))
        nref = w.norb + w.nproj
        cfg = lfd.make_config(w.ndom, w.nx, w.ny, w.nz, w.hx, w.hy, w.hz, w.bc, w.norb, w.nproj, w.dt,
                              device=0, nref_max=nref, flags=flags)
        ws = lfd.lfd_workspace_size(cfg)
        bufs["workspace"] = Guarded(max(ws, 1), dev)
        wsv = bufs["workspace"].view(torch.uint8, (max(ws, 1),))
        bufs["vloc"] = Guarded(_nbytes(shp, torch.float64), dev)
        vloc = bufs["vloc"].view(torch.float64, shp)
        vloc.copy_(torch.from_numpy(x.vloc))
        ctx = lfd.lfd_init(cfg, psi, proj, x.dnl if w.nproj else None, x.occ, wsv)
        try:
            if mode == "i8" and w.nproj:
                assert lfd.lfd_nl_path(ctx) == 1, w
            lfd.lfd_set_potential(ctx, vloc)
            for n in range(3):
                lfd.lfd_set_vector_potential(ctx, midpoint_A(w, n))
                lfd.lfd_step(ctx, 1)
            if w.nproj:
                lfd.lfd_step_sequence(ctx, np.stack([midpoint_A(w, n) for n in range(3)]))
            bufs["rho"] = Guarded(_nbytes(shp, torch.float64), dev)
            bufs["j"] = Guarded(_nbytes((w.ndom, 3) + shp[1:], torch.float64), dev)
            bufs["J"] = Guarded(_nbytes((w.ndom, 3), torch.float64), dev)
            lfd.lfd_density_current(ctx, bufs["rho"].view(torch.float64, shp),
                                    bufs["j"].view(torch.float64, (w.ndom, 3) + shp[1:]),
                                    bufs["J"].view(torch.float64, (w.ndom, 3)))
            bufs["E"] = Guarded(_nbytes((w.ndom, 4), torch.float64), dev)
            lfd.lfd_energy(ctx, bufs["E"].view(torch.float64, (w.ndom, 4)))
            basis = np.concatenate([x.psi0, x.proj], axis=-1) if w.nproj else x.psi0
            nb = basis.shape[-1]
            bufs["ref"] = Guarded(_nbytes(shp + (nb,), cdt), dev)
            ref = bufs["ref"].view(cdt, shp + (nb,))
            ref.copy_(torch.from_numpy(np.ascontiguousarray(basis.astype(ncdt))))
            bufs["occ_out"] = Guarded(_nbytes((w.ndom, nb), torch.float64), dev)
            lfd.lfd_remap_occ(ctx, ref, bufs["occ_out"].view(torch.float64, (w.ndom, nb)))
            lfd.lfd_sync(ctx)
        finally:
            lfd.lfd_destroy(ctx)
        torch.cuda.synchronize()
        assert torch.isfinite(torch.view_as_real(psi)).all(), (mode, w.name)
        for k, b in bufs.items():
            b.check(f"{mode} {w.name} {k}")
