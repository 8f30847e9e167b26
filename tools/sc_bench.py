"""A few self-consistent steps (lfd_sc_step, Hartree + exchange + Maxwell) on C2, for the ncu launch list."""
import argparse
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=2)
    ap.add_argument("--config", default="C2")
    args = ap.parse_args()
    import torch
    from lfd_workloads import domain_tiling, make_inputs, workload
    from lfd_workloads.generate import laser_A
    from paper_conf_ipps_razakhllknvn24_b200 import Context
    w = workload(args.config)
    x = make_inputs(w, seed=1)
    dev = torch.device("cuda:0")
    psi = torch.from_numpy(x.psi0).to(dev)
    ctx = Context(psi, torch.from_numpy(x.proj).to(dev), x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc)
    offs, gd = domain_tiling(w.ndom, (w.nx, w.ny, w.nz))
    Ah = np.stack([laser_A(w, 0.5 * k * w.dt)[0] for k in range(2 * args.steps + 1)])
    ctx.sc_init(gd, offs, torch.from_numpy(x.vloc).to(dev), Aext0=Ah[0])
    ctx.sc_step(Ah)
    ctx.sync()
    ctx.close()
    print("ok")


if __name__ == "__main__":
    main()
