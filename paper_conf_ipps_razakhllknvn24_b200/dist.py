"""Multi-GPU plumbing of the LFD step.

DC domains are independent inside a step, so they are partitioned across ranks (one process per GPU)
with no data-path collective. The one real exchange is the DC recombination of the density and the
macroscopic current that feed the global Hartree / Maxwell updates (reading R18): every rank
packs [rho of its domains | J of its domains] and one NCCL all-gather gives every rank all of them.
Domain cores tile the global grid (buffer b = 0), so the global density is an exact assembly.
"""
from __future__ import annotations

import numpy as np


def partition(ndom_total: int, rank: int, world: int) -> range:
    """Contiguous block of domains owned by `rank` (rank r owns [r*n/P, (r+1)*n/P))."""
    lo = rank * ndom_total // world
    hi = (rank + 1) * ndom_total // world
    return range(lo, hi)


def tiling_offsets(dom_grid: tuple, dom_shape: tuple) -> np.ndarray:
    """Offsets [ndom, 3] of domain cores tiling a global grid of dom_grid domains (x-major order)."""
    gx, gy, gz = dom_grid
    nx, ny, nz = dom_shape
    off = [(i * nx, j * ny, k * nz) for i in range(gx) for j in range(gy) for k in range(gz)]
    return np.asarray(off, dtype=np.int32)


def pack_size(ndom_local: int, ngrid: int) -> int:
    return ndom_local * (ngrid + 3)


def assemble_global(gathered, counts, dom_shape, offsets, gdims):
    """Build the global density [GX, GY, GZ] and J [ndom_total, 3] from the all-gathered buffer.

    gathered: 1-D tensor/array = concatenation over ranks of [rho (ndom_r * ng) | J (ndom_r * 3)],
    each rank's block padded to the largest block (all_gather needs equal sizes). counts[r] = domains of
    rank r. offsets: [ndom_total, 3] tiling offsets."""
    import torch
    nx, ny, nz = dom_shape
    ng = nx * ny * nz
    blk = max(counts) * (ng + 3)
    rho_g = torch.zeros(tuple(int(g) for g in gdims), dtype=torch.float64, device=gathered.device)
    Jall = []
    d = 0
    for r, c in enumerate(counts):
        base = r * blk
        rho = gathered[base: base + c * ng].reshape(c, nx, ny, nz)
        J = gathered[base + c * ng: base + c * ng + 3 * c].reshape(c, 3)
        for i in range(c):
            ox, oy, oz = (int(v) for v in offsets[d])
            rho_g[ox: ox + nx, oy: oy + ny, oz: oz + nz] = rho[i]
            Jall.append(J[i])
            d += 1
    return rho_g, torch.stack(Jall) if Jall else torch.zeros((0, 3), dtype=torch.float64)


def gather(send, world: int, group=None):
    """One all-gather of every rank's packed [rho | J] block (NCCL on GPUs, gloo on CPU tensors)."""
    import torch
    import torch.distributed as dist
    recv = torch.empty(world * send.numel(), dtype=send.dtype, device=send.device)
    dist.all_gather_into_tensor(recv, send, group=group)
    return recv
