"""Pins of the solver oracle (oracle/cg.py) against things other than itself (CPU only)."""
import numpy as np
import pytest
import scipy.sparse as sp

import fieldgen
import oracle
from oracle import cg as ocg
from tests import bruteforce


def coords(dims):
    lx, ly, lz, lt = dims
    return np.meshgrid(np.arange(lt), np.arange(lz), np.arange(ly), np.arange(lx), indexing="ij")[::-1]


@pytest.mark.parametrize("parity", [0, 1])
def test_normal_operator_vs_bruteforce(parity):
    """A_p = m^2 - P_p M P_{1-p} M P_p with M the shift-matrix operator (tests/bruteforce.py)."""
    dims = (8, 8, 8, 8)
    fat, lng = fieldgen.workload_links(dims)
    x = fieldgen.vector(dims, 61)
    m = 0.3
    M = bruteforce.operator(fat, lng)
    on = np.repeat(oracle.parity_mask(dims).reshape(-1) == bool(parity), 3)
    Pp = sp.diags(on.astype(float))
    Pq = sp.diags((~on).astype(float))
    A = m * m * Pp - Pp @ M @ Pq @ M @ Pp
    ref = (A @ x.reshape(-1)).reshape(x.shape)
    got = ocg.normal_apply(fat, lng, x, parity, m)
    assert oracle.normwise_error(got, ref) < 1e-14


def test_normal_operator_hermitian_positive():
    dims = (4, 4, 4, 6)
    fat, lng = fieldgen.workload_links(dims)
    u = fieldgen.vector(dims, 62)
    v = fieldgen.vector(dims, 63)
    m = 0.2
    au = ocg.normal_apply(fat, lng, u, 0, m)
    av = ocg.normal_apply(fat, lng, v, 0, m)
    even = (~oracle.parity_mask(dims))[..., None]
    ue, ve = u * even, v * even
    assert abs(np.vdot(ve, au) - np.vdot(av, ue)) < 1e-13 * np.linalg.norm(au) * np.linalg.norm(v)
    assert np.vdot(ue, au).real >= m * m * np.vdot(ue, ue).real * (1 - 1e-14)


@pytest.mark.parametrize("parity", [0, 1])
def test_cg_solves_bruteforce_system(parity):
    dims = (8, 8, 8, 8)
    fat, lng = fieldgen.workload_links(dims)
    b = fieldgen.vector(dims, 64)
    m = 0.5
    x, it = ocg.cg(fat, lng, b, parity, m, rel_tol=1e-12)
    M = bruteforce.operator(fat, lng)
    on = np.repeat(oracle.parity_mask(dims).reshape(-1) == bool(parity), 3)
    Pp = sp.diags(on.astype(float))
    Pq = sp.diags((~on).astype(float))
    A = m * m * Pp - Pp @ M @ Pq @ M @ Pp
    bp = b.reshape(-1) * on
    res = np.linalg.norm(A @ x.reshape(-1) - bp) / np.linalg.norm(bp)
    assert res < 1e-11
    assert 1 < it < 500


@pytest.mark.parametrize("n", [(1, 0, 0, 0), (1, 2, 3, 4)])
def test_cg_free_field_closed_form(n):
    """Phased free field (pin P5): A_p psi = (m^2 + 4 sum_mu (c1 sin p + c3 sin 3p)^2) psi, so the
    solution of A_p x = psi is psi / lambda, and CG on one eigenvector converges in 1 step."""
    dims = (8, 10, 12, 14)
    c1, c3, m = 9 / 8, -1 / 24, 0.1
    X = coords(dims)
    lx, ly, lz, lt = dims
    fat = np.zeros((lt, lz, ly, lx, 4, 3, 3), np.complex128)
    lng = np.zeros_like(fat)
    for mu in range(4):
        eta = (-1.0) ** (sum(X[nu] for nu in range(mu)) if mu else 0 * X[0])
        fat[..., mu, :, :] = (c1 * eta)[..., None, None] * np.eye(3)
        lng[..., mu, :, :] = (c3 * eta)[..., None, None] * np.eye(3)
    p = [2 * np.pi * n[k] / dims[k] for k in range(4)]
    psi = np.exp(1j * sum(p[k] * X[k] for k in range(4)))[..., None] * np.array([1.0, 0.5j, -0.25])
    even = (~oracle.parity_mask(dims))[..., None]
    lam = m * m + 4 * sum((c1 * np.sin(p[k]) + c3 * np.sin(3 * p[k])) ** 2 for k in range(4))
    x, it = ocg.cg(fat, lng, psi, 0, m, rel_tol=1e-13)
    assert oracle.normwise_error(x[even[..., 0]], (psi / lam)[even[..., 0]]) < 1e-13
    assert it == 1
