"""Drive a few C2 steps (the fused first-factor kernel) for the role-wait printf instrumentation build
(LFD_NVCC_DEFINES=-DLFD_FX_TIMING).   python tools/fx_timing.py [steps]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from lfd_workloads import make_inputs, workload  # noqa: E402
from paper_conf_ipps_razakhllknvn24_b200 import Context  # noqa: E402

w = workload(sys.argv[2] if len(sys.argv) > 2 else "C2")
x = make_inputs(w, seed=1)
dev = torch.device("cuda:0")
psi = torch.from_numpy(x.psi0).to(dev)
ctx = Context(psi, torch.from_numpy(x.proj).to(dev), x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc)
ctx.set_potential(torch.from_numpy(x.vloc).to(dev))
for _ in range(int(sys.argv[1]) if len(sys.argv) > 1 else 3):
    ctx.step(1)
ctx.sync()
ctx.close()
