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


class OverlappedGather:
    """The per-step DC recombination (all-gather of every rank's packed [rho | J]) on a side stream, double
    buffered, so it overlaps the next step's first nonlocal factor (lfd_step_prologue: it needs only Psi, B
    and D, not the v / A the gathered density feeds).

    Per step k:  slot = g.slot(k)  -> the density kernel writes g.send[slot] on the main stream;
                 g.start(k)        -> the all-gather of g.send[slot] into g.recv[slot] on the side stream;
                 ... main stream: lfd_step_prologue (overlaps the collective) ...
                 g.wait(k)         -> the main stream waits for it (before anything reads recv[slot]).
    A send slot is rewritten two steps later; start() makes the side stream, and slot() the main stream, wait
    for the previous user of that slot. On CPU tensors (gloo) there are no streams: start() is synchronous."""

    def __init__(self, numel: int, world: int, device, dtype=None, group=None):
        import torch
        dtype = dtype or torch.float64
        self.world, self.group = world, group
        self.send = [torch.empty(numel, dtype=dtype, device=device) for _ in range(2)]
        self.recv = [torch.empty(world * numel, dtype=dtype, device=device) for _ in range(2)]
        self.cuda = torch.device(device).type == "cuda"
        if self.cuda:
            self.side = torch.cuda.Stream(device=device)
            self.done = [None, None]

    @staticmethod
    def slot(k: int) -> int:
        return k & 1

    def before_write(self, k: int):
        """The main stream must not overwrite send[slot] while the gather that read it two steps ago runs."""
        if self.cuda and self.done[self.slot(k)] is not None:
            import torch
            torch.cuda.current_stream().wait_event(self.done[self.slot(k)])

    def start(self, k: int):
        import torch
        import torch.distributed as dist
        s = self.slot(k)
        if not self.cuda:
            dist.all_gather_into_tensor(self.recv[s], self.send[s], group=self.group)
            return
        ready = torch.cuda.Event()
        ready.record(torch.cuda.current_stream())
        self.side.wait_event(ready)
        with torch.cuda.stream(self.side):
            dist.all_gather_into_tensor(self.recv[s], self.send[s], group=self.group)
            ev = torch.cuda.Event()
            ev.record(self.side)
        self.done[s] = ev

    def wait(self, k: int):
        if self.cuda and self.done[self.slot(k)] is not None:
            import torch
            torch.cuda.current_stream().wait_event(self.done[self.slot(k)])
        return self.recv[self.slot(k)]


def allgather_occupations(occ_local, counts, group=None, device="cpu"):
    """The per-MD-step occupation handshake across ranks (only the occupation numbers f cross
    between QXMD and LFD): every rank contributes f of its domains [ndom_r][norb] and receives
    f of all domains [ndom_total][norb] (rank-major, i.e. global domain order of `partition`). Blocks are
    padded to the largest rank's (all-gather needs equal sizes). Returns a host float64 array."""
    import torch
    import torch.distributed as dist
    occ_local = np.ascontiguousarray(occ_local, dtype=np.float64)
    world = len(counts)
    norb = occ_local.shape[1]
    blk = max(counts) * norb
    send = torch.zeros(blk, dtype=torch.float64, device=device)
    send[: occ_local.size] = torch.from_numpy(occ_local.reshape(-1)).to(device)
    recv = torch.empty(world * blk, dtype=torch.float64, device=device)
    dist.all_gather_into_tensor(recv, send, group=group)
    r = recv.cpu().numpy()
    return np.concatenate([r[i * blk: i * blk + counts[i] * norb].reshape(counts[i], norb) for i in range(world)])
