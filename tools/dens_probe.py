"""Cold-L2 density timing on C2 (A/B only): one density call after an L2 flush (a 300 MB memset), median of 20,
for 32 and 64 active orbitals -- whether reading half of each 1 KB point row costs DRAM efficiency.
  python tools/dens_probe.py [--sp]"""
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
flush = torch.empty(300 * 2**20, dtype=torch.uint8, device=dev)
ctx = Context(psi, proj, x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt)
for nact in (32, 64, 16):
    occ = np.zeros((1, w.norb))
    occ[0, :nact] = 2.0
    ctx.set_occupations(occ)
    s = torch.cuda.current_stream()
    ts = []
    for it in range(22):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        lfd.lfd_density_current(ctx.ctx, rho, None, J)
        e1.record(s)
        torch.cuda.synchronize()
        if it >= 2:
            ts.append(e0.elapsed_time(e1))
    ms = float(np.median(ts))
    gb = (nact * (8 if sp else 16) + 8) * w.ngrid / 1e9
    print(json.dumps({"nact": nact, "sp": sp, "ms": round(ms, 5), "GBps": round(gb / ms * 1e3, 1)}), flush=True)
ctx.close()
