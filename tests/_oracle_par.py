"""Oracle runs on column subsets in worker processes (tests only).

Under Eq. 6 every orbital evolves on its own: the nonlocal factor acts column by column (C_us, the
update and the renormalisation of column s involve only column s, P:65 / P:210) and the local factor is
linear and pointwise in the orbital index. So the oracle's result for a set of columns is exactly those
columns of a full-width run, and independent column sets can run in parallel processes. Each worker
regenerates the seeded inputs (no large arrays are pickled) and calls only `oracle/`.
"""
from __future__ import annotations

import os
from concurrent.futures import ProcessPoolExecutor
import multiprocessing as mp

import numpy as np


def _columns(args):
    name, overrides, seed, cols, steps, dnl_scale = args
    from lfd_workloads import make_inputs, workload
    from lfd_workloads.generate import midpoint_A
    from oracle import ref
    w = workload(name).with_(**overrides)
    x = make_inputs(w, seed=seed)
    cfg = ref.RefConfig(w.ndom, w.nx, w.ny, w.nz, w.hx, w.hy, w.hz, w.bc, len(cols), w.nproj, w.dt)
    p = np.ascontiguousarray(x.psi0[..., list(cols)])
    dnl = np.ascontiguousarray(x.dnl * dnl_scale)
    A = np.zeros((w.ndom, 3))
    for n in range(steps):
        A = midpoint_A(w, n)
        ref.step(cfg, p, x.proj if w.nproj else None, dnl if w.nproj else None, x.vloc, A, 1)
    return p, A


def oracle_columns(name, seed, cols, steps, overrides=None, dnl_scale=1.0, workers=None):
    """Psi of the given orbital columns after `steps` oracle steps (per-step laser midpoints), and the A
    of the last step. Columns are spread over `workers` spawned processes."""
    cols = list(cols)
    workers = workers or min(len(cols), max(1, (os.cpu_count() or 2) - 1))
    groups = [cols[i::workers] for i in range(workers)]
    groups = [g for g in groups if g]
    ctx = mp.get_context("spawn")
    with ProcessPoolExecutor(max_workers=len(groups), mp_context=ctx) as ex:
        res = list(ex.map(_columns, [(name, overrides or {}, seed, g, steps, dnl_scale) for g in groups]))
    out = None
    A = res[0][1]
    for g, (p, _) in zip(groups, res):
        if out is None:
            out = np.zeros(p.shape[:-1] + (len(cols),), dtype=np.complex128)
        for k, c in enumerate(g):
            out[..., cols.index(c)] = p[..., k]
    return out, A
