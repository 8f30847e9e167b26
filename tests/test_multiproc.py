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


def _sc_worker(rank, world, port, q):
    """One rank of a 2-rank self-consistent run (SURVEY §8(e) + §8(f) rank 2): it owns half of the domains,
    writes their density cores into a zeroed global grid and its share sum_dom J_dom * ng / GN of the
    macroscopic current, and one SUM all-reduce assembles both -- the host-side decomposition lfd_sc_step
    performs with NCCL (api.cu sc_density), here with gloo around the oracle's step."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import dataclasses

    from oracle import sc
    from lfd_workloads import domain_tiling
    obj = [bytes(range(128)) if rank == 0 else None]  # the NCCL unique-id handshake of bench.py / sc_init
    dist.broadcast_object_list(obj, src=0)
    assert obj[0] == bytes(range(128))
    full = _sc_problem()
    nd = full.cfg.ndom // world
    mine = slice(rank * nd, (rank + 1) * nd)
    offs_all, gd = domain_tiling(full.cfg.ndom, (full.cfg.nx, full.cfg.ny, full.cfg.nz))
    p = dataclasses.replace(full, cfg=dataclasses.replace(full.cfg, ndom=nd), occ=full.occ[mine],
                            vion=full.vion[mine], offsets=offs_all[mine], gdims=gd)
    GN = int(np.prod(gd))

    def dist_density(pp, psi, A):
        from oracle import ref
        Ad = np.tile(np.asarray(A, np.float64), (pp.cfg.ndom, 1))
        rho, _, J = ref.density_current(pp.cfg, psi, pp.occ, Ad, want_j=False)
        pack = np.zeros(GN + 3)
        pack[:GN] = sc.assemble(pp.cfg, rho, pp.offsets, pp.gdims).reshape(-1)
        pack[GN:] = J.sum(axis=0) * (pp.cfg.ngrid / GN)
        t = torch.from_numpy(pack)
        dist.all_reduce(t)
        return t[:GN].numpy().reshape(gd), t[GN:].numpy().copy()

    sc._density = dist_density
    sc.check_tiling = lambda *a: None  # each rank holds only its own cores
    psi0 = _sc_psi0(full)[mine].copy()
    A = np.outer(np.sin(np.arange(7) * 0.02), [10.0, 0.0, 5.0])
    st = sc.sc_init(p, psi0, A[0], Adot0=(1.0, -1.0, 0.5))
    sc.sc_step(p, st, A, 3)
    q.put((rank, st.psi, st.A_ind, st.Adot, st.rho_g))
    dist.destroy_process_group()


def _sc_problem():
    from oracle import ref, sc
    from lfd_workloads import domain_tiling
    ndom, dims, h, norb = 4, (4, 4, 6), (0.35, 0.3, 0.4), 2
    cfg = ref.RefConfig(ndom, *dims, *h, 0, norb, 0, 0.04)
    offs, gd = domain_tiling(ndom, dims)
    rng = np.random.default_rng(9)
    vion = -0.3 * rng.random((ndom, int(np.prod(dims))))
    return sc.SCProblem(cfg, None, None, np.full((ndom, norb), 2.0), vion, offs, gd, n_corr=1)


def _sc_psi0(p):
    from lfd_workloads.generate import _mgs
    rng = np.random.default_rng(10)
    out = np.empty((p.cfg.ndom, p.cfg.nx, p.cfg.ny, p.cfg.nz, p.cfg.norb), complex)
    for d in range(p.cfg.ndom):
        X = rng.standard_normal((p.cfg.ngrid, p.cfg.norb)) + 1j * rng.standard_normal((p.cfg.ngrid, p.cfg.norb))
        out[d] = _mgs(X, p.cfg.dV).reshape(out.shape[1:])
    return out


def test_sc_two_ranks_equal_one_process():
    from oracle import sc
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_sc_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=300) for _ in range(world)], key=lambda t: t[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    full = _sc_problem()
    A = np.outer(np.sin(np.arange(7) * 0.02), [10.0, 0.0, 5.0])
    st = sc.sc_init(full, _sc_psi0(full), A[0], Adot0=(1.0, -1.0, 0.5))
    sc.sc_step(full, st, A, 3)
    psi = np.concatenate([r[1] for r in res])
    assert np.abs(psi - st.psi).max() < 1e-13
    for r in res:
        assert np.abs(r[2] - st.A_ind).max() < 1e-12 and np.abs(r[3] - st.Adot).max() < 1e-12
        assert np.abs(r[4] - st.rho_g).max() < 1e-13


def _occ_worker(rank, world, port, ndom, norb, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    mine = ldist.partition(ndom, rank, world)
    counts = [len(ldist.partition(ndom, r, world)) for r in range(world)]
    occ = np.array([[2.0 - 0.01 * (d * norb + s) for s in range(norb)] for d in mine]).reshape(len(mine), norb)
    got = ldist.allgather_occupations(occ, counts)
    # the overlapped (double-buffered) density gather on CPU tensors: two steps, slots alternate
    g = ldist.OverlappedGather(4, world, "cpu")
    outs = []
    for k in range(3):
        s = g.slot(k)
        g.before_write(k)
        g.send[s].copy_(torch.arange(4, dtype=torch.float64) + 10 * rank + 100 * k)
        g.start(k)
        outs.append(g.wait(k).clone().numpy())
    q.put((rank, got, outs))
    dist.destroy_process_group()


@pytest.mark.parametrize("ndom", [2, 5])
def test_occupation_handshake_and_overlapped_gather_two_ranks(ndom):
    """The per-MD-step occupation all-gather gives every rank f of all domains in global order,
    and the double-buffered side-stream density gather returns each step's blocks of both ranks."""
    world, norb = 2, 3
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_occ_worker, args=(r, world, port, ndom, norb, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    want = np.array([[2.0 - 0.01 * (d * norb + s) for s in range(norb)] for d in range(ndom)])
    for _, got, outs in res:
        assert np.array_equal(got, want)
        for k, o in enumerate(outs):
            assert np.array_equal(o, np.concatenate([np.arange(4) + 100 * k, np.arange(4) + 10 + 100 * k]))
