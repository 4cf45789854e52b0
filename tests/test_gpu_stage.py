"""GPU parity of the neighbour-staged kernel (DSLASH_OPT_STAGE): per block, a tile of TY full
x-rows at one (z, t); the TMA engine copies the source rows y0-3 .. y0+TY+2 into shared memory
(cp.async.bulk + mbarrier) and the x / y hops read them there (the 3LP-1
local-memory staging).

The staged kernel visits z/t before x/y, a different summation order from the unstaged kernel:
it must match the oracle within the fp64 tolerance, and, among its own launch
shapes (halo split, multi-RHS, repeated applies), it must be bitwise reproducible.
"""
import numpy as np
import pytest

import fieldgen
import oracle

pytestmark = pytest.mark.gpu

TOL = 1e-12


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    torch.cuda.set_device(0)
    return torch


def _apply(torch, dims, fat, lng, src_cb, parity, **kw):
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    with Dslash(dims, **kw) as D:
        D.load_links(fat, lng)
        out = D(torch.from_numpy(src_cb).to(D.dtype).cuda(), parity)
        torch.cuda.synchronize()
        return out.cpu().numpy().astype(np.complex128)


# Lx = 2 (one site per row), odd lxh (6x.., 10x..), Ly < TY + 6 (rows wrap several times), 4^4 aliasing,
# Ly with few divisors (14), the benchmark shape
DIMS = [(4, 4, 4, 4), (2, 4, 6, 8), (6, 8, 10, 12), (8, 10, 12, 14), (10, 14, 4, 6), (16, 16, 16, 16),
        (32, 32, 32, 32)]


@pytest.mark.parametrize("kernel", ["site", "dir2"])
@pytest.mark.parametrize("dims", DIMS)
@pytest.mark.parametrize("parity", [0, 1])
def test_stage_vs_oracle(torch_cuda, kernel, dims, parity):
    if dims == (32, 32, 32, 32) and parity == 1:
        pytest.skip("one parity at full size is enough")
    fat, lng = fieldgen.workload_links(dims)
    psi = fieldgen.vector(dims, fieldgen.SEED_PSI)
    ref = oracle.full_to_cb(oracle.dslash(fat, lng, psi, parity), parity)
    got = _apply(torch_cuda, dims, fat, lng, fieldgen.vector_cb(dims, fieldgen.SEED_PSI, 1 - parity), parity,
                 kernel=kernel, stage=True)
    assert oracle.normwise_error(got, ref) <= TOL


@pytest.mark.parametrize("kernel", ["site", "dir2"])
def test_stage_gaussian_links_and_point_source(torch_cuda, kernel):
    """Non-unitary links (Z14), and an integer point source that must come out exactly (P6 shape)."""
    dims = (8, 10, 12, 14)
    fat = fieldgen.links(dims, 101, "gauss")
    lng = fieldgen.links(dims, 102, "gauss", scale=0.3)
    psi = fieldgen.vector(dims, 103)
    for parity in (0, 1):
        ref = oracle.full_to_cb(oracle.dslash(fat, lng, psi, parity), parity)
        got = _apply(torch_cuda, dims, fat, lng, oracle.full_to_cb(psi, 1 - parity), parity, kernel=kernel,
                     stage=True)
        assert oracle.normwise_error(got, ref) <= TOL
    # identity-like integer links: every product is exact, so any summation order gives the oracle's bits
    one = np.zeros(dims[::-1] + (4, 3, 3), np.complex128)
    one[..., 0, 0] = one[..., 1, 1] = one[..., 2, 2] = 1.0
    src = np.zeros(dims[::-1] + (3,), np.complex128)
    src[3, 4, 5, 5, 1] = 1.0                                   # (x, y, z, t) = (5, 5, 4, 3): parity 1
    ref = oracle.full_to_cb(oracle.dslash(one, 2 * one, src, 0), 0)
    got = _apply(torch_cuda, dims, one, 2 * one, oracle.full_to_cb(src, 1), 0, kernel=kernel, stage=True)
    assert np.array_equal(got, ref)
    assert np.count_nonzero(np.abs(got).sum(axis=0)) == 16


@pytest.mark.parametrize("kernel", ["site", "dir2"])
@pytest.mark.parametrize("mask", [0x8, 0x4, 0xC])
def test_stage_self_halo_bitwise(torch_cuda, kernel, mask):
    """Interior + boundary (ghost-aware staged kernel) equals the unpartitioned staged apply bitwise."""
    dims = (8, 8, 8, 12)
    fat, lng = fieldgen.workload_links(dims)
    src = fieldgen.vector_cb(dims, 7, 0)
    base = _apply(torch_cuda, dims, fat, lng, src, 1, kernel=kernel, stage=True)
    for overlap in (True, False):
        halo = _apply(torch_cuda, dims, fat, lng, src, 1, kernel=kernel, stage=True, force_halo=mask,
                      overlap=overlap)
        assert np.array_equal(base, halo), overlap


@pytest.mark.parametrize("kernel", ["site", "dir2"])
@pytest.mark.parametrize("nrhs", [2, 3, 4, 8, 11])
def test_stage_multi_rhs(torch_cuda, kernel, nrhs):
    """Several right-hand sides per tile: bitwise equal to single staged applies, and to the oracle."""
    import torch
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 10, 12, 14)
    fat, lng = fieldgen.workload_links(dims)
    parity = 0
    src = torch.stack([torch.from_numpy(fieldgen.vector_cb(dims, 140 + r, 1)) for r in range(nrhs)]).cuda()
    with Dslash(dims, kernel=kernel, stage=True) as D:
        D.load_links(fat, lng)
        out = torch.empty_like(src)
        D.apply_multi(out, src, parity)
        singles = torch.stack([D(src[r].contiguous(), parity) for r in range(nrhs)])
        torch.cuda.synchronize()
    assert torch.equal(out, singles)
    for r in (0, nrhs - 1):
        ref = oracle.full_to_cb(oracle.dslash(fat, lng, fieldgen.vector(dims, 140 + r), parity), parity)
        assert oracle.normwise_error(out[r].cpu().numpy(), ref) <= TOL


@pytest.mark.parametrize("precision,recon,tol", [("f64", 12, 1e-12), ("f32", 18, 1e-5), ("f32", 12, 1e-5),
                                                 ("mixed", 18, 1e-5)])
def test_stage_precisions(torch_cuda, precision, recon, tol):
    dims = (8, 10, 12, 14)
    fat, lng = fieldgen.workload_links(dims)
    psi = fieldgen.vector(dims, 5)
    ref = oracle.full_to_cb(oracle.dslash(fat, lng, psi, 1), 1)
    for kernel in ("site", "dir2"):
        got = _apply(torch_cuda, dims, fat, lng, oracle.full_to_cb(psi, 0), 1, kernel=kernel, stage=True,
                     precision=precision, recon=recon)
        err = oracle.normwise_error(got, ref)
        assert err <= tol
        if precision != "f64":
            assert err > 1e-12


def test_stage_repeat_and_pdl_chain_bitwise(torch_cuda):
    """Back-to-back staged applies (PDL: the next grid's blocks start while this one drains) over
    chained inputs give the same bits as applies separated by synchronisation."""
    import torch
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (16, 16, 16, 16)
    fat, lng = fieldgen.workload_links(dims)
    x0 = torch.from_numpy(fieldgen.vector_cb(dims, 9, 1)).cuda()
    chains = []
    for pdl in (True, False):
        with Dslash(dims, stage=True, pdl=pdl) as D:
            D.load_links(fat, lng)
            v, outs = x0, []
            for k in range(6):
                v = D(v, k % 2)            # target parity alternates with the source
                outs.append(v.clone())
                if not pdl:
                    torch.cuda.synchronize()
            torch.cuda.synchronize()
            chains.append(torch.stack(outs).cpu())
    assert torch.equal(chains[0], chains[1])


def test_stage_option_errors(torch_cuda):
    from paper_conf_sc_dufekgaad024_b200 import Dslash, DslashError, _abi
    with pytest.raises(DslashError) as e:
        Dslash((8, 8, 8, 8), kernel="dir4", stage=True)
    assert e.value.status == _abi.DSLASH_ERR_UNSUPPORTED
    with pytest.raises(DslashError) as e:
        Dslash((6, 8, 8, 8), precision="f32", stage=True)      # Lx/2 = 3: rows not 16-byte multiples
    assert e.value.status == _abi.DSLASH_ERR_UNSUPPORTED
    with Dslash((8, 8, 8, 8), stage=True) as D:
        with pytest.raises(DslashError):
            _abi.dslash_set_option(D.h, _abi.DSLASH_OPT_KERNEL, _abi.DSLASH_KERNEL_DIR4)


def test_stage_cg_mixed_odd_half_row_refused(torch_cuda):
    """dslash_cg_mixed runs an F64 handle's kernels as F32 ones (SloppyScope).  With the staged
    kernel and Lx/2 odd the fp32 rows are not 16-byte multiples, so cp.async.bulk would fault:
    the launch refuses with DSLASH_ERR_UNSUPPORTED before any copy is issued, and the context
    stays usable (an unstaged solve on a fresh handle still converges)."""
    from paper_conf_sc_dufekgaad024_b200 import Dslash, DslashError, _abi
    torch = torch_cuda
    dims = (6, 8, 8, 8)                                          # Lx/2 = 3
    fat, lng = fieldgen.workload_links(dims)
    b = torch.from_numpy(fieldgen.vector_cb(dims, 4, 0)).cuda()
    with Dslash(dims, stage=True) as D:                          # fp64 rows (48 B): allowed
        D.load_links(fat, lng)
        with pytest.raises(DslashError) as e:
            D.cg_mixed(D.empty_vector(), b, 0, 0.5, rel_tol=1e-10)
        assert e.value.status == _abi.DSLASH_ERR_UNSUPPORTED
    with Dslash(dims) as D:
        D.load_links(fat, lng)
        ok, it, outer, res = D.cg_mixed(D.empty_vector(), b, 0, 0.5, rel_tol=1e-10)
        assert ok and res <= 2e-10
