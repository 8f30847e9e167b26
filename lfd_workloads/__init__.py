"""Seeded synthetic workloads for the LFD step (shared by the oracle tests, the GPU tests and bench.py).

This package holds ONLY input recipes (shapes, a PbTiO3-shaped local potential, orthonormal initial
orbitals and projectors, occupations, the laser vector potential). It contains none of the method's
arithmetic (no propagator, no projection, no density) -- see DESIGN.md §5 for the recipe and its
citations.
"""
from .configs import WORKLOADS, Workload, domain_tiling, workload  # noqa: F401
from .generate import Inputs, laser_A, make_inputs  # noqa: F401
