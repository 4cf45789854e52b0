"""GPU: CG for several systems sharing each link pass (dslash_cg_multi_blocked; SURVEY §8(f)-3 on the
§8(f)-4 multi-RHS stencil), against the oracle's normal operator and CG (oracle/cg.py) and against
dslash_cg solving each system alone."""
import numpy as np
import pytest

import fieldgen
import oracle
from oracle import cg as ocg

pytestmark = pytest.mark.gpu

DIMS = (8, 8, 8, 12)      # Vh = 3072 = 192 blocks of 16


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    torch.cuda.set_device(0)
    return torch


def _blocked_b(torch, D, parity, seeds):
    planar = torch.stack([torch.from_numpy(oracle.full_to_cb(fieldgen.vector(DIMS, s), parity)) for s in seeds])
    planar = planar.contiguous().cuda()
    return planar, D.to_blocked(torch.empty_like(planar), planar)


@pytest.mark.parametrize("parity", [0, 1])
@pytest.mark.parametrize("nrhs", [1, 3, 8])
def test_cg_multi_vs_oracle_and_single(torch_cuda, parity, nrhs):
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    fat, lng = fieldgen.workload_links(DIMS)
    m, tol = 0.25, 1e-10
    seeds = [120 + k for k in range(nrhs)]
    with Dslash(DIMS) as D:
        D.load_links(fat, lng)
        planar_b, bb = _blocked_b(torch, D, parity, seeds)
        xb = torch.empty_like(bb)
        ok, its, res = D.cg_multi_blocked(xb, bb, parity, m, rel_tol=tol, max_iter=500)
        x = D.from_blocked(torch.empty_like(xb), xb).cpu().numpy()
        singles = []
        for k in range(nrhs):
            xs = D.empty_vector()
            oks, its_k, _ = D.cg(xs, planar_b[k].contiguous(), parity, m, rel_tol=tol, max_iter=500)
            assert oks
            singles.append((xs.cpu().numpy(), its_k))
    assert ok and all(r <= 2 * tol for r in res) and all(i > 1 for i in its)
    for k, s in enumerate(seeds):
        bcb = oracle.full_to_cb(fieldgen.vector(DIMS, s), parity)
        # the solution solves the ORACLE's system
        ax = oracle.full_to_cb(ocg.normal_apply(fat, lng, oracle.cb_to_full(x[k], DIMS, parity), parity, m), parity)
        assert np.linalg.norm(ax - bcb) / np.linalg.norm(bcb) <= 2 * tol
        # same recurrences as dslash_cg on that system alone (its arithmetic rounds differently):
        # iterations within 2, solutions at the tolerance's level
        xs, its_k = singles[k]
        assert abs(its[k] - its_k) <= 2, (k, its[k], its_k)
        assert np.linalg.norm(x[k] - xs) / np.linalg.norm(xs) <= 1e-8
    xo, ito = ocg.cg(fat, lng, fieldgen.vector(DIMS, seeds[0]), parity, m, rel_tol=tol)
    assert abs(its[0] - ito) <= 2


def test_cg_multi_frozen_systems(torch_cuda):
    """Systems converge at different iterations (a zero right-hand side at once, a scaled copy at the
    same iteration as its original); the frozen ones keep their solution exactly."""
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    fat, lng = fieldgen.workload_links(DIMS)
    m, tol, parity = 0.5, 1e-11, 0
    with Dslash(DIMS, precision="mixed") as D:
        D.load_links(fat, lng)
        b0 = torch.from_numpy(oracle.full_to_cb(fieldgen.vector(DIMS, 130), parity)).cuda()
        b1 = torch.from_numpy(oracle.full_to_cb(fieldgen.vector(DIMS, 131), parity)).cuda()
        planar = torch.stack([b0, torch.zeros_like(b0), b1, b0 * 1024.0]).contiguous()
        bb = D.to_blocked(torch.empty_like(planar), planar)
        xb = torch.empty_like(bb)
        ok, its, res = D.cg_multi_blocked(xb, bb, parity, m, rel_tol=tol, max_iter=1000)
        x = D.from_blocked(torch.empty_like(xb), xb)
        torch.cuda.synchronize()
    assert ok
    assert its[1] == 0 and res[1] == 0.0 and torch.count_nonzero(x[1]) == 0
    assert its[0] == its[3]                         # the same Krylov sequence, scaled by 2^10
    assert torch.equal(x[3], x[0] * 1024.0)
    assert all(r <= 2 * tol for k, r in enumerate(res) if k != 1)


def test_cg_multi_errors(torch_cuda):
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash, _abi
    fat, lng = fieldgen.workload_links(DIMS)
    with Dslash(DIMS, precision="f32") as D:
        D.load_links(fat, lng)
        v = torch.zeros((2, 3, D.vh), dtype=D.dtype, device="cuda")
        with pytest.raises(_abi.DslashError) as e:
            D.cg_multi_blocked(torch.empty_like(v), v, 0, 0.5)
        assert e.value.status == _abi.DSLASH_ERR_UNSUPPORTED
    with Dslash(DIMS) as D:
        D.load_links(fat, lng)
        v = torch.zeros((9, 3, D.vh), dtype=D.dtype, device="cuda")
        with pytest.raises(_abi.DslashError) as e:            # more than 8 systems
            D.cg_multi_blocked(torch.empty_like(v), v, 0, 0.5)
        assert e.value.status == _abi.DSLASH_ERR_ARG
        v = torch.zeros((2, 3, D.vh), dtype=D.dtype, device="cuda")
        with pytest.raises(_abi.DslashError) as e:            # mass 0: A is not positive definite
            D.cg_multi_blocked(torch.empty_like(v), v, 0, 0.0)
        assert e.value.status == _abi.DSLASH_ERR_ARG
