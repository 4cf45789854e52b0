"""Pins of the CPU oracle against things other than itself (P1-P9).

Every test here is CPU-only.  Each one is chosen so that a plausible bug in the
oracle (a dropped term, a wrong sign, a +3/-1 hop swap, a transposed link, a
missing conjugate, a wrong axis order) fails at least one of them:

  P1 brute-force operator from shift permutation matrices (hop geometry, +-3 via S^3)
  P2 free-field plane-wave eigenvalue, closed form (signs of all four terms, Naik)
  P3 anti-Hermiticity: oracle matrix D^dag = -D bitwise; <chi, D psi> = -<D chi, psi>
  P4 gauge covariance (which end of each link multiplies which psi)
  P5 phased free field D_oe D_eo closed form (two-parity composition)
  P6 point source, exact integers (axis order, lex/cb layout)
  P7 parity structure (output independent of same-parity input)
  P8 flop accounting vs the paper's 600.8 M (L278)
  P9 linearity
"""
import json
import os

import numpy as np
import pytest

import fieldgen
import oracle
from tests import bruteforce

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "paper_constants.json")
AXIS = bruteforce.AXIS

# (Lx, Ly, Lz, Lt); every extent >= 8 in the last two so +3 and -1 never alias (Z13)
LATTICES = [(4, 4, 4, 4), (8, 8, 8, 8), (8, 10, 12, 14)]


def coords(dims):
    lx, ly, lz, lt = dims
    return np.meshgrid(np.arange(lt), np.arange(lz), np.arange(ly), np.arange(lx), indexing="ij")[::-1]


def const_links(dims, c):
    lx, ly, lz, lt = dims
    u = np.zeros((lt, lz, ly, lx, 4, 3, 3), np.complex128)
    u[..., :, :] = c * np.eye(3)
    return u


# ---------------------------------------------------------------- P1
@pytest.mark.parametrize("dims", LATTICES)
@pytest.mark.parametrize("kind", ["su3", "gauss"])
@pytest.mark.parametrize("parity", [0, 1])
def test_P1_bruteforce_operator(dims, kind, parity):
    fat = fieldgen.links(dims, 11, kind)
    lng = fieldgen.links(dims, 12, kind, scale=-1.0 / 24 if kind == "su3" else 0.5)
    psi = fieldgen.vector(dims, 13)
    M = bruteforce.operator(fat, lng)
    ref = bruteforce.apply(M, psi)
    chi = oracle.dslash(fat, lng, psi, parity)
    on = oracle.parity_mask(dims) == bool(parity)
    assert oracle.normwise_error(chi[on], ref[on]) < 1e-14
    assert np.all(chi[~on] == 0)


def test_P1_bruteforce_catches_hop_swap():
    """Sanity of the pin itself: an operator whose long links hop by 1 instead of 3
    (indistinguishable from the right one on small aliasing lattices) is rejected at L>=8."""
    dims = (8, 10, 12, 14)
    fat = fieldgen.links(dims, 11)
    lng = fieldgen.links(dims, 12)
    psi = fieldgen.vector(dims, 13)
    M_good = bruteforce.operator(fat, lng)
    V = np.prod(dims)
    import scipy.sparse as sp
    M_bad = sp.csr_matrix((3 * V, 3 * V), dtype=np.complex128)
    I3 = sp.identity(3, format="csr")
    for mu in range(4):
        S = sp.kron(bruteforce.shift(dims, mu), I3, format="csr")
        F = bruteforce.blockdiag(fat.reshape(V, 4, 3, 3)[:, mu])
        N = bruteforce.blockdiag(lng.reshape(V, 4, 3, 3)[:, mu])
        M_bad = M_bad + F @ S - S.T @ F.conj().T + N @ S - S.T @ N.conj().T
    chi = oracle.dslash(fat, lng, psi, 0)
    on = oracle.parity_mask(dims) == False  # noqa: E712
    assert oracle.normwise_error(chi[on], bruteforce.apply(M_good, psi)[on]) < 1e-14
    assert oracle.normwise_error(chi[on], bruteforce.apply(M_bad, psi)[on]) > 1e-2


def test_P1_P7_dense_structure():
    """Dense M at 4^4: anti-Hermitian bitwise, same-parity blocks exactly zero."""
    dims = (4, 4, 4, 4)
    M = bruteforce.operator(fieldgen.links(dims, 21), fieldgen.links(dims, 22, scale=-1 / 24)).toarray()
    assert np.array_equal(M.conj().T, -M)
    odd = np.repeat(oracle.parity_mask(dims).reshape(-1), 3)
    assert np.all(M[np.ix_(odd, odd)] == 0) and np.all(M[np.ix_(~odd, ~odd)] == 0)


# ---------------------------------------------------------------- P2
@pytest.mark.parametrize("dims", [(8, 8, 8, 8), (8, 10, 12, 14)])
@pytest.mark.parametrize("n", [(1, 0, 0, 0), (0, 2, 1, 0), (1, 3, 2, 5), (3, 1, 4, 1)])
@pytest.mark.parametrize("parity", [0, 1])
def test_P2_free_field_plane_wave(dims, n, parity):
    c1, c3 = 0.7, -0.3
    p = [2 * np.pi * n[m] / dims[m] for m in range(4)]
    X = coords(dims)
    phase = np.exp(1j * sum(p[m] * X[m] for m in range(4)))
    v = np.array([1.0 + 0.5j, -0.25 + 2j, 0.75 - 1j])
    psi = phase[..., None] * v
    chi = oracle.dslash(const_links(dims, c1), const_links(dims, c3), psi, parity)
    lam = 2j * sum(c1 * np.sin(p[m]) + c3 * np.sin(3 * p[m]) for m in range(4))
    on = oracle.parity_mask(dims) == bool(parity)
    assert oracle.normwise_error(chi[on], (lam * psi)[on]) < 1e-13


def test_P2_naik_improvement():
    """c1 = 9/8, c3 = -1/24 (the Naik/asqtad coefficients) cancel the O(p^3) error:
    lambda / 2i = p - 0.075 p^5 + O(p^7) for a wave along x."""
    dims = (64, 2, 2, 2)
    p = 2 * np.pi / 64
    X = coords(dims)
    psi = np.exp(1j * p * X[0])[..., None] * np.array([1.0, 0.0, 0.0])
    chi = oracle.dslash(const_links(dims, 9 / 8), const_links(dims, -1 / 24), psi, 0)
    on = ~oracle.parity_mask(dims)
    lam_half = (chi[on][:, 0] / psi[on][:, 0] / 2j)
    # the y, z, t directions have p = 0 (sin 0 = 0): only x contributes
    assert np.allclose(lam_half, 9 / 8 * np.sin(p) - 1 / 24 * np.sin(3 * p), rtol=0, atol=1e-14)
    assert np.allclose(lam_half, p - 0.075 * p ** 5, rtol=0, atol=1e-8)   # O(p^7) ~ 1.6e-9
    assert abs(lam_half.real.mean() - p) < 1e-6           # O(p^3) term is absent
    assert abs(lam_half.real.mean() - np.sin(p)) > 1e-5   # unimproved operator would be sin p


# ---------------------------------------------------------------- P3
@pytest.mark.parametrize("dims", [(4, 4, 4, 4), (4, 6, 4, 8)])
def test_P3_oracle_matrix_antihermitian_bitwise(dims):
    fat = fieldgen.links(dims, 31, "gauss")
    lng = fieldgen.links(dims, 32, "gauss")
    V = int(np.prod(dims))
    D = np.zeros((3 * V, 3 * V), np.complex128)
    lt, lz, ly, lx = dims[::-1]
    for col in range(3 * V):
        e = np.zeros(3 * V, np.complex128)
        e[col] = 1.0
        e = e.reshape(lt, lz, ly, lx, 3)
        D[:, col] = (oracle.dslash(fat, lng, e, 0) + oracle.dslash(fat, lng, e, 1)).reshape(-1)
    assert np.array_equal(D.conj().T, -D)


@pytest.mark.parametrize("dims", LATTICES)
def test_P3_inner_product_antisymmetry(dims):
    fat, lng = fieldgen.workload_links(dims)
    on_e = ~oracle.parity_mask(dims)
    psi = fieldgen.vector(dims, 41) * (~on_e)[..., None]   # odd source
    chi = fieldgen.vector(dims, 42) * on_e[..., None]      # even vector
    d_psi = oracle.dslash(fat, lng, psi, 0)                 # D_eo psi_o
    d_chi = oracle.dslash(fat, lng, chi, 1)                 # D_oe chi_e
    lhs = np.vdot(chi, d_psi)
    rhs = -np.vdot(d_chi, psi)
    scale = np.linalg.norm(chi) * np.linalg.norm(d_psi)
    assert abs(lhs - rhs) < 1e-14 * scale
    assert abs(lhs) > 1e-3 * scale  # the identity is not trivially 0 = 0


# ---------------------------------------------------------------- P4
def site_mul(g, u):
    return np.einsum("...ij,...jk->...ik", g, u)


@pytest.mark.parametrize("dims", [(8, 8, 8, 8), (8, 10, 12, 14)])
@pytest.mark.parametrize("parity", [0, 1])
def test_P4_gauge_covariance(dims, parity):
    fat = fieldgen.links(dims, 51, "gauss")
    lng = fieldgen.links(dims, 52, "gauss")
    psi = fieldgen.vector(dims, 53)
    g = fieldgen.matrices(dims, fieldgen.SEED_GAUGE, nper=1)[..., 0, :, :]
    fat2 = np.empty_like(fat)
    lng2 = np.empty_like(lng)
    for mu in range(4):
        g1 = np.roll(g, -1, axis=AXIS[mu]).conj().swapaxes(-1, -2)   # g(x+mu)^dag
        g3 = np.roll(g, -3, axis=AXIS[mu]).conj().swapaxes(-1, -2)   # g(x+3mu)^dag
        fat2[..., mu, :, :] = site_mul(site_mul(g, fat[..., mu, :, :]), g1)
        lng2[..., mu, :, :] = site_mul(site_mul(g, lng[..., mu, :, :]), g3)
    psi2 = np.einsum("...ij,...j->...i", g, psi)
    lhs = oracle.dslash(fat2, lng2, psi2, parity)
    rhs = np.einsum("...ij,...j->...i", g, oracle.dslash(fat, lng, psi, parity))
    assert oracle.normwise_error(lhs, rhs) < 1e-13


def test_P4_detects_wrong_orientation():
    """Transforming with g(x-mu) instead of g(x+mu) must break covariance (pin sanity)."""
    dims = (8, 8, 8, 8)
    fat = fieldgen.links(dims, 51, "gauss")
    lng = fieldgen.links(dims, 52, "gauss")
    psi = fieldgen.vector(dims, 53)
    g = fieldgen.matrices(dims, fieldgen.SEED_GAUGE, nper=1)[..., 0, :, :]
    fat2 = np.empty_like(fat)
    lng2 = np.empty_like(lng)
    for mu in range(4):
        gm = np.roll(g, +1, axis=AXIS[mu]).conj().swapaxes(-1, -2)
        fat2[..., mu, :, :] = site_mul(site_mul(g, fat[..., mu, :, :]), gm)
        lng2[..., mu, :, :] = site_mul(site_mul(g, lng[..., mu, :, :]), gm)
    psi2 = np.einsum("...ij,...j->...i", g, psi)
    lhs = oracle.dslash(fat2, lng2, psi2, 0)
    rhs = np.einsum("...ij,...j->...i", g, oracle.dslash(fat, lng, psi, 0))
    assert oracle.normwise_error(lhs, rhs) > 1e-2


# ---------------------------------------------------------------- P5
@pytest.mark.parametrize("dims", [(8, 8, 8, 8), (8, 10, 12, 14)])
@pytest.mark.parametrize("n", [(1, 0, 0, 0), (1, 2, 3, 4), (2, 1, 1, 3)])
def test_P5_phased_free_field_two_parity(dims, n):
    c1, c3 = 9 / 8, -1 / 24
    X = coords(dims)
    lx, ly, lz, lt = dims
    fat = np.zeros((lt, lz, ly, lx, 4, 3, 3), np.complex128)
    lng = np.zeros_like(fat)
    for mu in range(4):
        eta = (-1.0) ** (sum(X[nu] for nu in range(mu)) if mu else 0 * X[0])
        fat[..., mu, :, :] = (c1 * eta)[..., None, None] * np.eye(3)
        lng[..., mu, :, :] = (c3 * eta)[..., None, None] * np.eye(3)
    p = [2 * np.pi * n[m] / dims[m] for m in range(4)]
    psi = np.exp(1j * sum(p[m] * X[m] for m in range(4)))[..., None] * np.array([1.0, -2.0j, 0.5])
    even = ~oracle.parity_mask(dims)
    psi_e = psi * even[..., None]
    chi_o = oracle.dslash(fat, lng, psi_e, 1)            # D_oe psi_e
    res_e = oracle.dslash(fat, lng, chi_o, 0)            # D_eo D_oe psi_e
    lam = -4 * sum((c1 * np.sin(p[m]) + c3 * np.sin(3 * p[m])) ** 2 for m in range(4))
    assert oracle.normwise_error(res_e[even], (lam * psi)[even]) < 1e-13


# ---------------------------------------------------------------- P6
@pytest.mark.parametrize("x0", [(0, 0, 0, 0), (3, 7, 5, 11), (7, 9, 11, 13), (2, 1, 10, 2)])
def test_P6_point_source_exact(x0):
    dims = (8, 10, 12, 14)
    lx, ly, lz, lt = dims
    fat = const_links(dims, 1.0)
    lng = const_links(dims, 2.0)
    v = np.array([1 + 2j, -3 + 0j, 4 - 5j])
    psi = np.zeros((lt, lz, ly, lx, 3), np.complex128)
    psi[x0[3], x0[2], x0[1], x0[0]] = v
    parity = 1 - (sum(x0) & 1)
    chi = oracle.dslash(fat, lng, psi, parity)
    expect = np.zeros_like(psi)
    for mu in range(4):
        for h, coef in ((-1, +1.0), (+1, -1.0), (-3, +2.0), (+3, -2.0)):
            c = list(x0)
            c[mu] = (c[mu] + h) % dims[mu]
            expect[c[3], c[2], c[1], c[0]] += coef * v
    assert np.array_equal(chi, expect)
    assert np.count_nonzero(np.abs(chi).sum(-1)) == 16
    # the same result read back through the library's cb layout convention (Z8: cb = lex // 2)
    cb = oracle.full_to_cb(chi, parity)
    lex = x0[0] - 1 + lx * (x0[1] + ly * (x0[2] + lz * x0[3])) if x0[0] > 0 else \
        (lx - 1) + lx * (x0[1] + ly * (x0[2] + lz * x0[3]))
    assert np.array_equal(cb[:, lex // 2], v)   # site x0 - x^ carries +v


# ---------------------------------------------------------------- P7
@pytest.mark.parametrize("parity", [0, 1])
def test_P7_same_parity_input_ignored(parity):
    dims = (8, 10, 12, 14)
    fat, lng = fieldgen.workload_links(dims)
    psi = fieldgen.vector(dims, 71)
    junk = fieldgen.vector(dims, 72)
    same = (oracle.parity_mask(dims) == bool(parity))[..., None]
    a = oracle.dslash(fat, lng, psi, parity)
    b = oracle.dslash(fat, lng, np.where(same, junk, psi), parity)
    assert np.array_equal(a, b)


# ---------------------------------------------------------------- P8
def test_P8_flop_accounting_matches_paper():
    g = json.load(open(GOLDEN))
    L = g["L"]["value"]
    vh = L ** 4 // 2
    cmul, cadd = 6, 2                       # real flops per complex multiply / add
    matvec = 9 * cmul + 6 * cadd            # 3x3 complex matrix times 3-vector
    per_site = 16 * matvec + 15 * 3 * cadd  # 16 matvecs, 15 vector additions
    assert per_site == oracle.FLOP_PER_SITE == 1146
    assert round(per_site * vh / 1e6, 1) == g["flop_per_apply"]["value"] / 1e6
    assert 4 * 4 == g["matrices_per_target_site"]["value"]
    assert 4 * 4 * 3 * 3 == g["complex_mults_per_target_site"]["value"]
    wi = g["work_items_millions"]["value"]
    for name, mult in (("1LP", 1), ("2LP", 3), ("3LP", 12), ("4LP", 48)):
        assert round(vh * mult / 1e6, 1) == pytest.approx(wi[name], abs=0.051)
    assert round(768 * 16 / 1e3, 1) == g["local_memory_kbyte_3LP_768"]["value"]


# ---------------------------------------------------------------- P9
def test_P9_linearity():
    dims = (8, 10, 12, 14)
    fat, lng = fieldgen.workload_links(dims)
    psi = fieldgen.vector(dims, 91)
    phi = fieldgen.vector(dims, 92)
    a, b = 0.3 - 1.7j, -2.1 + 0.4j
    lhs = oracle.dslash(fat, lng, a * psi + b * phi, 0)
    rhs = a * oracle.dslash(fat, lng, psi, 0) + b * oracle.dslash(fat, lng, phi, 0)
    assert oracle.normwise_error(lhs, rhs) < 1e-14


# ---------------------------------------------------------------- sampled entry point
def test_sites_entry_matches_full():
    dims = (8, 10, 12, 14)
    fat, lng = fieldgen.workload_links(dims)
    psi = fieldgen.vector(dims, 93)
    full = oracle.dslash(fat, lng, psi, 1).reshape(-1, 3)
    sites = oracle.lex_sites_of_parity(dims, 1)[::37]
    assert np.array_equal(oracle.dslash_sites(fat, lng, psi, sites), full[sites])


def test_threads_do_not_change_result():
    dims = (8, 10, 12, 14)
    fat, lng = fieldgen.workload_links(dims)
    psi = fieldgen.vector(dims, 94)
    assert np.array_equal(oracle.dslash(fat, lng, psi, 0, 1), oracle.dslash(fat, lng, psi, 0, 0))
