"""Shape sweep of the y-marching density kernel on C2 (A/B only; needs a build with LFD_NVCC_DEFINES=-DLFD_TUNING_KNOBS):
for each combination of the tuning knobs
(LFD_DENS_ZC, LFD_DENS_PX, LFD_DENS_YC, LFD_DENS_OWN, LFD_DENS_XP, read at lfd_init; a combination the shape
search rejects falls back to its best admissible shape), the device time per density call.
  python tools/dens_sweep.py [--sp]"""
import itertools
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from lfd_workloads import make_inputs, workload  # noqa: E402
from paper_conf_ipps_razakhllknvn24_b200 import Context, lfd  # noqa: E402

sp = "--sp" in sys.argv
w = workload("C2")
x = make_inputs(w, seed=1)
dev = torch.device("cuda:0")
dt = np.complex64 if sp else np.complex128
psi = torch.from_numpy(x.psi0.astype(dt)).to(dev)
proj = torch.from_numpy(x.proj.astype(dt)).to(dev)
rho = torch.empty((1, w.ngrid), dtype=torch.float64, device=dev)
J = torch.empty((1, 3), dtype=torch.float64, device=dev)
grid = {"LFD_DENS_ZC": [8, 12, 24, 36], "LFD_DENS_PX": [1, 2], "LFD_DENS_YC": [1, 2, 4], "LFD_DENS_OWN": [3, 4, 5],
        "LFD_DENS_XP": [2, 3]}
keys = list(grid)
for vals in itertools.product(*[grid[k] for k in keys]):
    for k, v in zip(keys, vals):
        os.environ[k] = str(v)
    ctx = Context(psi, proj, x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt)
    for _ in range(5):
        lfd.lfd_density_current(ctx.ctx, rho, None, J)
    s = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    for _ in range(40):
        lfd.lfd_density_current(ctx.ctx, rho, None, J)
    e1.record(s)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 40
    print(json.dumps({**dict(zip(keys, vals)), "ms": round(ms, 5)}), flush=True)
    ctx.close()
