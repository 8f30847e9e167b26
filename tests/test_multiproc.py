"""World-size-2 gloo tests (CPU) of the N > 1 host logic: domain partitioning, packing, the all-gather
DC recombination and the global-grid assembly. The assembled global density must equal
the single-process assembly exactly."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_razakhllknvn24_b200 import dist as ldist


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def fake_rho(dom, shape):
    rng = np.random.default_rng(100 + dom)
    return torch.from_numpy(rng.random(shape))


def _worker(rank, world, port, ndom, shape, dom_grid, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    mine = ldist.partition(ndom, rank, world)
    counts = [len(ldist.partition(ndom, r, world)) for r in range(world)]
    ng = int(np.prod(shape))
    blk = max(counts) * (ng + 3)
    send = torch.zeros(blk, dtype=torch.float64)
    for i, d in enumerate(mine):
        send[i * ng:(i + 1) * ng] = fake_rho(d, shape).reshape(-1)
    for i, d in enumerate(mine):
        send[len(mine) * ng + 3 * i: len(mine) * ng + 3 * i + 3] = torch.tensor([d, -d, 0.5 * d], dtype=torch.float64)
    recv = ldist.gather(send, world)
    off = ldist.tiling_offsets(dom_grid, shape)
    gd = [dom_grid[i] * shape[i] for i in range(3)]
    rho_g, J = ldist.assemble_global(recv, counts, shape, off, gd)
    q.put((rank, rho_g.numpy(), J.numpy()))
    dist.destroy_process_group()


@pytest.mark.parametrize("ndom,dom_grid", [(8, (2, 2, 2)), (3, (3, 1, 1))])
def test_gather_assembly_two_ranks(ndom, dom_grid):
    shape = (4, 3, 2)
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, ndom, shape, dom_grid, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    off = ldist.tiling_offsets(dom_grid, shape)
    want = np.zeros([dom_grid[i] * shape[i] for i in range(3)])
    for d in range(ndom):
        ox, oy, oz = off[d]
        want[ox:ox + 4, oy:oy + 3, oz:oz + 2] = fake_rho(d, shape).numpy()
    for _, rho_g, J in res:
        assert np.array_equal(rho_g, want)
        assert np.array_equal(J[:, 0], np.arange(ndom)) and np.array_equal(J[:, 2], 0.5 * np.arange(ndom))


def test_partition_covers_all_domains():
    for n in (1, 7, 8, 13):
        for w in (1, 2, 3, 8):
            got = [d for r in range(w) for d in ldist.partition(n, r, w)]
            assert got == list(range(n))
