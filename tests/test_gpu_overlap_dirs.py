"""GPU parity of the split-by-direction overlap (DSLASH_OPT_OVERLAP = DSLASH_OVERLAP_DIRS): a local
pass over every site skips the hops into ghost faces while the faces are in flight; the ghost
pass then adds exactly those hops to the boundary sites' stored partial sums.

Interior sites (no ghost hop) run the unpartitioned arithmetic and must come out bitwise equal
to the unpartitioned apply; boundary sites sum their terms in another order and must agree
within the fp64 tolerance, and the whole field must match the oracle.
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


def _interior_mask(dims, parity, halo_mask):
    """Target sites of `parity` (cb order) none of whose 16 sources is in a ghost face."""
    lx, ly, lz, lt = dims
    lex = oracle.lex_sites_of_parity(dims, parity)
    z = (lex // (lx * ly)) % lz
    t = lex // (lx * ly * lz)
    inside = np.ones(lex.shape, bool)
    if halo_mask & 0x8:
        inside &= (t >= 3) & (t < lt - 3)
    if halo_mask & 0x4:
        inside &= (z >= 3) & (z < lz - 3)
    return inside


@pytest.mark.parametrize("kernel", ["site", "dir2", "dir4"])
@pytest.mark.parametrize("dims,mask", [((8, 8, 8, 12), 0x8), ((8, 8, 12, 8), 0x4), ((8, 8, 8, 8), 0xC),
                                       ((8, 10, 12, 14), 0xC), ((6, 8, 10, 6), 0x8), ((4, 4, 4, 4), 0xC)])
@pytest.mark.parametrize("parity", [0, 1])
def test_dirs_vs_oracle_and_unpartitioned(torch_cuda, kernel, dims, mask, parity):
    fat, lng = fieldgen.workload_links(dims)
    psi = fieldgen.vector(dims, 11)
    src = oracle.full_to_cb(psi, 1 - parity)
    ref = oracle.full_to_cb(oracle.dslash(fat, lng, psi, parity), parity)
    base = _apply(torch_cuda, dims, fat, lng, src, parity, kernel=kernel)
    got = _apply(torch_cuda, dims, fat, lng, src, parity, kernel=kernel, force_halo=mask, overlap="dirs")
    assert oracle.normwise_error(got, ref) <= TOL
    assert oracle.normwise_error(got, base) <= 1e-14
    inside = _interior_mask(dims, parity, mask)
    assert np.array_equal(got[:, inside], base[:, inside])


@pytest.mark.parametrize("precision,recon,tol", [("f32", 18, 1e-5), ("f32", 12, 1e-5), ("mixed", 18, 1e-5),
                                                 ("f64", 12, 1e-12)])
@pytest.mark.parametrize("kernel", ["site", "dir2"])
def test_dirs_precisions(torch_cuda, precision, recon, tol, kernel):
    """fp32 links use the paired layout, where a kind's forward and backward matrix share loads:
    the local / ghost passes skip them per hop."""
    dims = (8, 10, 12, 14)
    fat, lng = fieldgen.workload_links(dims)
    psi = fieldgen.vector(dims, 12)
    ref = oracle.full_to_cb(oracle.dslash(fat, lng, psi, 0), 0)
    got = _apply(torch_cuda, dims, fat, lng, oracle.full_to_cb(psi, 1), 0, kernel=kernel, precision=precision,
                 recon=recon, force_halo=0xC, overlap="dirs")
    assert oracle.normwise_error(got, ref) <= tol


@pytest.mark.parametrize("kernel", ["site", "dir2"])
@pytest.mark.parametrize("nrhs", [2, 4, 8, 3])
def test_dirs_multi_rhs_bitwise(torch_cuda, kernel, nrhs):
    """apply_multi through both passes equals single applies in the same mode bitwise."""
    import torch
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 8, 8, 12)
    fat, lng = fieldgen.workload_links(dims)
    src = torch.stack([torch.from_numpy(fieldgen.vector_cb(dims, 70 + r, 0)) for r in range(nrhs)]).cuda()
    with Dslash(dims, kernel=kernel, force_halo=0xC, overlap="dirs") as D:
        D.load_links(fat, lng)
        out = torch.empty_like(src)
        for _ in range(2):
            D.apply_multi(out, src, 1)
        singles = torch.stack([D(src[r].contiguous(), 1) for r in range(nrhs)])
        torch.cuda.synchronize()
    assert torch.equal(out, singles)
    ref = oracle.full_to_cb(oracle.dslash(fat, lng, fieldgen.vector(dims, 70), 1), 1)
    assert oracle.normwise_error(out[0].cpu().numpy(), ref) <= TOL


@pytest.mark.parametrize("transport", ["p2p", "nccl-self"])
def test_dirs_transports_and_repeat(torch_cuda, transport):
    """Both halo transports feed the ghost pass; several epochs through the same ghosts."""
    import torch
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 8, 8, 12)
    fat, lng = fieldgen.workload_links(dims)
    srcs = [torch.from_numpy(fieldgen.vector_cb(dims, 80 + r, 1)).cuda() for r in range(3)]
    kw = {"transport": "p2p"} if transport == "p2p" else {"self_nccl": True}
    with Dslash(dims, force_halo=0xC, overlap="dirs", **kw) as D:
        D.load_links(fat, lng)
        first = [D(s, 0).cpu() for s in srcs]
        for _ in range(2):
            for r, s in enumerate(srcs):
                assert torch.equal(D(s, 0).cpu(), first[r])
    for r in range(3):
        ref = oracle.full_to_cb(oracle.dslash(fat, lng, fieldgen.vector(dims, 80 + r), 0), 0)
        assert oracle.normwise_error(first[r].numpy(), ref) <= TOL


def test_dirs_full_size_weak_scaling_shape(torch_cuda):
    """32^4 local with the t halo (the weak-scaling per-GPU volume) against the unpartitioned
    apply: interior bitwise, all within 1e-14."""
    dims = (32, 32, 32, 32)
    fat, lng = fieldgen.workload_links(dims)
    src = fieldgen.vector_cb(dims, fieldgen.SEED_PSI, 1)
    base = _apply(torch_cuda, dims, fat, lng, src, 0)
    got = _apply(torch_cuda, dims, fat, lng, src, 0, force_halo=0x8, overlap="dirs")
    inside = _interior_mask(dims, 0, 0x8)
    assert np.array_equal(got[:, inside], base[:, inside])
    assert oracle.normwise_error(got, base) <= 1e-14


def test_dirs_staged_kernel_and_cg(torch_cuda):
    """The staged kernel runs both passes too; CG through the split-by-direction applies solves the
    system (same iterations within 2 of the unpartitioned solve)."""
    import torch
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 8, 8, 12)
    fat, lng = fieldgen.workload_links(dims)
    psi = fieldgen.vector(dims, 13)
    ref = oracle.full_to_cb(oracle.dslash(fat, lng, psi, 1), 1)
    got = _apply(torch_cuda, dims, fat, lng, oracle.full_to_cb(psi, 0), 1, stage=True, force_halo=0xC,
                 overlap="dirs")
    assert oracle.normwise_error(got, ref) <= TOL
    b = torch.from_numpy(fieldgen.vector_cb(dims, 73, 0)).cuda()
    res = []
    for kw in ({}, {"force_halo": 0xC, "overlap": "dirs"}):
        with Dslash(dims, **kw) as D:
            D.load_links(fat, lng)
            x = D.empty_vector()
            ok, it, rel = D.cg(x, b, 0, 0.3, rel_tol=1e-10)
            assert ok and rel <= 1e-10
            res.append((x.cpu().numpy(), it))
    assert abs(res[0][1] - res[1][1]) <= 2
    assert oracle.normwise_error(res[1][0], res[0][0]) <= 1e-9


def test_dirs_option_errors(torch_cuda):
    from paper_conf_sc_dufekgaad024_b200 import Dslash, DslashError, _abi
    with Dslash((16, 8, 8, 8)) as D:
        with pytest.raises(DslashError):
            _abi.dslash_set_option(D.h, _abi.DSLASH_OPT_OVERLAP, 3)   # the removed one-shot fused mode
