"""GPU: the normal operator and CG against the oracle (oracle/cg.py)."""
import numpy as np
import pytest

import fieldgen
import oracle
from oracle import cg as ocg

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    torch.cuda.set_device(0)
    return torch


@pytest.mark.parametrize("kernel", ["dir2", "site"])
@pytest.mark.parametrize("parity", [0, 1])
@pytest.mark.parametrize("mask", [0, 0xC])
def test_normal_apply_vs_oracle(torch_cuda, kernel, parity, mask):
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 10, 12, 14) if mask == 0 else (8, 8, 8, 12)
    fat, lng = fieldgen.workload_links(dims)
    x = fieldgen.vector(dims, 71)
    m = 0.37
    ref = oracle.full_to_cb(ocg.normal_apply(fat, lng, x, parity, m), parity)
    with Dslash(dims, kernel=kernel, force_halo=mask) as D:
        D.load_links(fat, lng)
        xin = torch.from_numpy(oracle.full_to_cb(x, parity)).cuda()
        out = D.normal_apply(D.empty_vector(), xin, parity, m)
        torch.cuda.synchronize()
    assert oracle.normwise_error(out.cpu().numpy(), ref) <= 1e-12


@pytest.mark.parametrize("parity", [0, 1])
@pytest.mark.parametrize("precision", ["f64", "mixed"])
def test_cg_vs_oracle(torch_cuda, parity, precision):
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 10, 12, 14)
    fat, lng = fieldgen.workload_links(dims)
    b = fieldgen.vector(dims, 72)
    m, tol = 0.25, 1e-10
    bcb = oracle.full_to_cb(b, parity)
    with Dslash(dims, precision=precision) as D:
        D.load_links(fat, lng)
        x = D.empty_vector()
        ok, it, res = D.cg(x, torch.from_numpy(bcb).cuda(), parity, m, rel_tol=tol, max_iter=500)
        xg = x.cpu().numpy()
    assert ok and res <= 2 * tol and it > 1
    # the GPU solution solves the ORACLE's system (to the operator's precision)
    ax = oracle.full_to_cb(ocg.normal_apply(fat, lng, oracle.cb_to_full(xg, dims, parity), parity, m), parity)
    true_res = np.linalg.norm(ax - bcb) / np.linalg.norm(bcb)
    assert true_res <= (2 * tol if precision == "f64" else 1e-5)
    xo, ito = ocg.cg(fat, lng, b, parity, m, rel_tol=tol)
    if precision == "f64":
        assert abs(it - ito) <= 2
        assert oracle.normwise_error(xg, oracle.full_to_cb(xo, parity)) < 1e-8


def test_cg_self_halo_bitwise(torch_cuda):
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 8, 8, 12)
    fat, lng = fieldgen.workload_links(dims)
    b = torch.from_numpy(fieldgen.vector_cb(dims, 73, 0)).cuda()
    sols = []
    # unpartitioned; self-halo by device copies; self-halo through NCCL send/recv to this rank
    # with the dot products through a one-rank ncclAllReduce (DSLASH_OPT_SELF_NCCL)
    for mask, self_nccl in ((0, False), (0xC, False), (0xC, True)):
        with Dslash(dims, force_halo=mask, self_nccl=self_nccl) as D:
            D.load_links(fat, lng)
            x = D.empty_vector()
            ok, it, res = D.cg(x, b, 0, 0.3, rel_tol=1e-10)
            sols.append((x.cpu(), it, res))
    for k in (1, 2):
        assert torch.equal(sols[0][0], sols[k][0]) and sols[0][1] == sols[k][1], k


def test_cg_free_field_closed_form(torch_cuda):
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 10, 12, 14)
    c1, c3, m = 9 / 8, -1 / 24, 0.1
    lx, ly, lz, lt = dims
    X = np.meshgrid(np.arange(lt), np.arange(lz), np.arange(ly), np.arange(lx), indexing="ij")[::-1]
    fat = np.zeros((lt, lz, ly, lx, 4, 3, 3), np.complex128)
    lng = np.zeros_like(fat)
    for mu in range(4):
        eta = (-1.0) ** (sum(X[nu] for nu in range(mu)) if mu else 0 * X[0])
        fat[..., mu, :, :] = (c1 * eta)[..., None, None] * np.eye(3)
        lng[..., mu, :, :] = (c3 * eta)[..., None, None] * np.eye(3)
    n = (1, 2, 3, 4)
    p = [2 * np.pi * n[k] / dims[k] for k in range(4)]
    psi = np.exp(1j * sum(p[k] * X[k] for k in range(4)))[..., None] * np.array([1.0, 0.5j, -0.25])
    lam = m * m + 4 * sum((c1 * np.sin(p[k]) + c3 * np.sin(3 * p[k])) ** 2 for k in range(4))
    with Dslash(dims) as D:
        D.load_links(fat, lng)
        x = D.empty_vector()
        ok, it, res = D.cg(x, torch.from_numpy(oracle.full_to_cb(psi, 0)).cuda(), 0, m, rel_tol=1e-13)
    # converges in one iteration; the host learns it one iteration late (lagged check), so the
    # solver may run one more, which must leave the exact solution in place
    assert ok and it <= 2
    assert oracle.normwise_error(x.cpu().numpy(), oracle.full_to_cb(psi / lam, 0)) < 1e-13


def test_cg_not_converged_and_errors(torch_cuda):
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash, _abi
    dims = (8, 8, 8, 8)
    fat, lng = fieldgen.workload_links(dims)
    with Dslash(dims) as D:
        D.load_links(fat, lng)
        b = torch.from_numpy(fieldgen.vector_cb(dims, 74, 0)).cuda()
        x = D.empty_vector()
        ok, it, res = D.cg(x, b, 0, 0.05, rel_tol=1e-14, max_iter=3)
        assert not ok and it == 3 and res > 1e-14
        y = D(b, 0)                                    # the handle is still usable
        with pytest.raises(_abi.DslashError):
            D.cg(x, b, 0, 0.0)                         # zero mass
    with Dslash(dims, parity_mask=_abi.DSLASH_EVEN) as D:
        D.load_links(fat, lng)
        with pytest.raises(_abi.DslashError) as e:
            D.cg(D.empty_vector(), torch.from_numpy(fieldgen.vector_cb(dims, 74, 0)).cuda(), 0, 0.3)
        assert e.value.status == _abi.DSLASH_ERR_ARG


@pytest.mark.parametrize("parity", [0, 1])
@pytest.mark.parametrize("recon", [18, 12])
def test_cg_mixed_vs_oracle(torch_cuda, parity, recon):
    """Mixed-precision CG (fp32 inner solves on fp32 links, fp64 defect correction): the answer
    solves the ORACLE's fp64 system to rel_tol (true residual), and matches the oracle CG's x."""
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 10, 12, 14)
    fat, lng = fieldgen.workload_links(dims)
    b = fieldgen.vector(dims, 72)
    m, tol = 0.25, 1e-10
    bcb = oracle.full_to_cb(b, parity)
    with Dslash(dims, recon=recon) as D:
        D.load_links(fat, lng)
        x = D.empty_vector()
        ok, it, outer, res = D.cg_mixed(x, torch.from_numpy(bcb).cuda(), parity, m, rel_tol=tol, inner_tol=1e-4)
        xg = x.cpu().numpy()
    assert ok and res <= tol and outer >= 2 and it > outer
    ax = oracle.full_to_cb(ocg.normal_apply(fat, lng, oracle.cb_to_full(xg, dims, parity), parity, m), parity)
    assert np.linalg.norm(ax - bcb) / np.linalg.norm(bcb) <= 2 * tol
    xo, _ = ocg.cg(fat, lng, b, parity, m, rel_tol=tol)
    assert oracle.normwise_error(xg, oracle.full_to_cb(xo, parity)) < 1e-8


def test_cg_mixed_halo_paths_bitwise(torch_cuda):
    """The same mixed-precision solve through the self-halo paths (device copies, NCCL to self,
    P2P): bitwise equal, since every fp32 apply, BLAS pass and dot product is deterministic and
    partition-independent on one rank."""
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 8, 8, 12)
    fat, lng = fieldgen.workload_links(dims)
    b = torch.from_numpy(fieldgen.vector_cb(dims, 74, 1)).cuda()
    sols = []
    for kw in ({}, {"force_halo": 0xC}, {"force_halo": 0x8, "self_nccl": True}, {"force_halo": 0xC, "transport": "p2p"}):
        with Dslash(dims, **kw) as D:
            D.load_links(fat, lng)
            x = D.empty_vector()
            ok, it, outer, res = D.cg_mixed(x, b, 1, 0.3, rel_tol=1e-11, inner_tol=1e-3)
            assert ok and res <= 1e-11
            sols.append((x.cpu(), it, outer))
    for k in range(1, len(sols)):
        assert torch.equal(sols[0][0], sols[k][0]) and sols[0][1:] == sols[k][1:], k


def test_cg_mixed_reload_links_and_errors(torch_cuda):
    """load_links invalidates the fp32 copies: a second solve uses the new links."""
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash, DslashError
    dims = (8, 8, 8, 8)
    fat, lng = fieldgen.workload_links(dims)
    fat2 = fieldgen.links(dims, 91)
    b = fieldgen.vector(dims, 75)
    bcb = torch.from_numpy(oracle.full_to_cb(b, 0)).cuda()
    with Dslash(dims) as D:
        D.load_links(fat, lng)
        x = D.empty_vector()
        assert D.cg_mixed(x, bcb, 0, 0.4, rel_tol=1e-10)[0]
        D.load_links(fat2, lng)
        ok, it, outer, res = D.cg_mixed(x, bcb, 0, 0.4, rel_tol=1e-10)
        assert ok
        xo, _ = ocg.cg(fat2, lng, b, 0, 0.4, rel_tol=1e-10)
        assert oracle.normwise_error(x.cpu().numpy(), oracle.full_to_cb(xo, 0)) < 1e-8
        with pytest.raises(DslashError):
            D.cg_mixed(x, bcb, 0, 0.4, inner_tol=1.5)
    with Dslash(dims, precision="f32") as D:
        D.load_links(fat, lng)
        x = D.empty_vector()
        with pytest.raises(DslashError):
            D.cg_mixed(x, torch.zeros_like(x), 0, 0.4)
