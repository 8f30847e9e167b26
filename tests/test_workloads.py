"""The synthetic workloads match the paper's printed shapes (tests/golden/paper_facts.json) and the
generator's outputs have the structure the method assumes (orthonormal Psi(0) and B, B orthogonal to
Psi(0), periodic-ready even meshes)."""
import json
import os

import numpy as np
import pytest

from lfd_workloads import laser_A, make_inputs, workload

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "paper_facts.json")))


def test_c2_is_paper_benchmark_shape():
    w = workload("C2")
    assert [w.nx, w.ny, w.nz] == GOLD["benchmark_mesh"]["value"]
    assert w.norb == GOLD["benchmark_orbitals"]["value"]
    assert 5 * np.prod(w.cells) == GOLD["atoms_per_rank"]["value"]
    # Delta_QD = 1 as in atomic units of time (2.4188843e-17 s)
    assert abs(w.dt * 2.4188843265857e-17 - GOLD["time_step_orders"]["dt_qd_s"]) < 1e-21


@pytest.mark.parametrize("name", ["C1", "P0", "P1", "P2z", "P3"])
def test_generated_orbitals_orthonormal(name):
    w = workload(name)
    x = make_inputs(w, seed=1)
    for dm in range(w.ndom):
        Q = x.psi0[dm].reshape(-1, w.norb)
        assert np.abs(w.dV * Q.conj().T @ Q - np.eye(w.norb)).max() < 1e-12
        if w.nproj:
            B = x.proj[dm].reshape(-1, w.nproj)
            assert np.abs(w.dV * B.conj().T @ B - np.eye(w.nproj)).max() < 1e-12
            assert np.abs(w.dV * B.conj().T @ Q).max() < 1e-12
    assert np.all((x.occ == 0) | (x.occ == 2))


def test_generator_is_deterministic():
    w = workload("P0")
    a, b = make_inputs(w, seed=5), make_inputs(w, seed=5)
    assert np.array_equal(a.psi0, b.psi0) and np.array_equal(a.vloc, b.vloc)


def test_laser_midpoint_values():
    w = workload("C2")
    A = laser_A(w, 0.0)
    # A0 = c E0 / omega; A(0) = A0 sin(pi/3) along z
    assert abs(A[0, 2] - 137.035999084 * 0.005 / 0.057 * np.sin(np.pi / 3)) < 1e-12
    assert A[0, 0] == 0 and A[0, 1] == 0
    assert np.all(laser_A(workload("C1"), 1.0) == 0)
