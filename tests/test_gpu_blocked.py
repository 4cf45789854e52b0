"""The site-blocked multi-RHS vector layout (dslash_apply_multi_blocked, include/hisq_dslash.h):
element (rhs r, colour c, site cb) at [cb // 16][r * 3 + c][cb % 16].

- the conversion kernels against the layout's definition (a torch permutation written here);
- blocked applies are bitwise the planar dslash_apply_multi (same per-thread arithmetic and
  summation order; the planar path is oracle-checked in test_gpu_parity / test_gpu_full_size), for
  every precision, recon and right-hand-side count, and match the oracle directly;
- with a halo (self-halo t / t + z through every transport; P2P ranks in test_gpu_multiproc) the
  faces are exchanged as whole 16-site blocks, bitwise;
- the unsupported cases fail loudly (Vh or a face not whole blocks, the split-by-direction overlap).
"""
import pytest

import fieldgen
import oracle

pytestmark = pytest.mark.gpu

DIMS = (8, 10, 12, 14)    # Vh = 6720 = 420 blocks of 16; several tiles and the periodic wrap


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    torch.cuda.set_device(0)
    return torch


def _blocked_ref(torch, planar):
    """the layout's definition: (nrhs, 3, Vh) -> flat [Vh / 16][nrhs * 3][16]"""
    nrhs, _, vh = planar.shape
    return planar.reshape(nrhs * 3, vh // 16, 16).permute(1, 0, 2).contiguous().reshape(-1)


@pytest.mark.parametrize("precision", ["f64", "f32"])
@pytest.mark.parametrize("nrhs", [1, 3, 8])
def test_conversion_matches_definition(torch_cuda, precision, nrhs):
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    with Dslash(DIMS, precision=precision) as D:
        g = torch.Generator().manual_seed(7)
        planar = torch.randn((nrhs, 3, D.vh), dtype=D.dtype, generator=g).cuda()
        blocked = D.to_blocked(torch.empty_like(planar), planar)
        back = D.from_blocked(torch.empty_like(planar), blocked)
        torch.cuda.synchronize()
    assert torch.equal(blocked.reshape(-1), _blocked_ref(torch, planar))
    assert torch.equal(back, planar)


@pytest.mark.parametrize("precision,recon", [("f64", 18), ("f64", 12), ("f64", 9), ("f32", 18), ("f32", 12),
                                             ("f32", 9), ("mixed", 18), ("mixed", 12), ("mixed", 9)])
@pytest.mark.parametrize("nrhs", [1, 2, 5, 8, 11])
def test_blocked_bitwise_planar(torch_cuda, precision, recon, nrhs):
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    fat, lng = fieldgen.workload_links(DIMS)
    parity = nrhs & 1
    with Dslash(DIMS, precision=precision, recon=recon, kernel="site") as D:
        D.load_links(fat, lng)
        src = torch.stack([torch.from_numpy(fieldgen.vector_cb(DIMS, 60 + r, 1 - parity)) for r in range(nrhs)])
        src = src.to(D.dtype).contiguous().cuda()
        planar = D.apply_multi(torch.empty_like(src), src, parity)
        bsrc = D.to_blocked(torch.empty_like(src), src)
        bout = D.apply_multi_blocked(torch.empty_like(src), bsrc, parity)
        got = D.from_blocked(torch.empty_like(src), bout)
        torch.cuda.synchronize()
    assert torch.equal(got, planar)


@pytest.mark.parametrize("precision,tol", [("f64", 1e-12), ("f32", 1e-5)])
def test_blocked_vs_oracle(torch_cuda, precision, tol):
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    fat, lng = fieldgen.workload_links(DIMS)
    parity, nrhs = 0, 8
    with Dslash(DIMS, precision=precision) as D:
        D.load_links(fat, lng)
        src = torch.stack([torch.from_numpy(fieldgen.vector_cb(DIMS, 80 + r, 1)) for r in range(nrhs)])
        src = src.to(D.dtype).contiguous().cuda()
        bout = D.apply_multi_blocked(torch.empty_like(src), D.to_blocked(torch.empty_like(src), src), parity)
        got = D.from_blocked(torch.empty_like(src), bout).cpu().numpy()
    for r in range(nrhs):
        ref = oracle.full_to_cb(oracle.dslash(fat, lng, fieldgen.vector(DIMS, 80 + r), parity), parity)
        assert oracle.normwise_error(got[r].astype("complex128"), ref) <= tol


@pytest.mark.parametrize("halo,kw", [(8, {}), (12, {}), (8, {"transport": "p2p"}), (12, {"transport": "p2p"}),
                                     (12, {"overlap": False}), (8, {"self_nccl": True}),
                                     (12, {"precision": "f32"}), (12, {"precision": "mixed", "recon": 12}),
                                     (8, {"kernel": "dir2"})])
def test_blocked_self_halo_bitwise(torch_cuda, halo, kw):
    """With a self-halo (t: 8, t + z: 12; device copies, P2P copies, NCCL to self, one launch after
    the exchange) the blocked apply exchanges whole 16-site blocks and equals the planar apply
    without a halo bitwise."""
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 8, 12, 12)          # Vh 4608; t face 3 x 384 sites, z faces 3 x 32 per t-slice
    fat, lng = fieldgen.workload_links(dims)
    kernel = kw.pop("kernel", "site")
    plain_kw = {k: v for k, v in kw.items() if k in ("precision", "recon")}
    with Dslash(dims, kernel=kernel, **plain_kw) as D:
        D.load_links(fat, lng)
        src = torch.stack([torch.from_numpy(fieldgen.vector_cb(dims, 90 + r, 1)) for r in range(8)])
        src = src.to(D.dtype).contiguous().cuda()
        ref = D.apply_multi(torch.empty_like(src), src, 0)
        torch.cuda.synchronize()
    with Dslash(dims, kernel=kernel, force_halo=halo, **kw) as D:
        D.load_links(fat, lng)
        bsrc = D.to_blocked(torch.empty_like(src), src)
        bout = torch.empty_like(src)
        for _ in range(3):                        # several epochs through the same ghosts
            D.apply_multi_blocked(bout, bsrc, 0)
        got = D.from_blocked(torch.empty_like(src), bout)
        torch.cuda.synchronize()
    assert torch.equal(got, ref)


def test_blocked_unsupported(torch_cuda):
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash, _abi
    dims = (8, 8, 12, 12)
    with Dslash(dims, force_halo=8, overlap="dirs") as D:   # split by direction: planar partial sums
        D.load_links(*fieldgen.workload_links(dims))
        v = torch.zeros((8, 3, D.vh), dtype=D.dtype, device="cuda")
        with pytest.raises(_abi.DslashError) as e:
            D.apply_multi_blocked(torch.empty_like(v), v, 0)
        assert e.value.status == _abi.DSLASH_ERR_UNSUPPORTED
    dims = (6, 6, 6, 6)                           # Vh = 648, not a multiple of 16
    with Dslash(dims) as D:
        D.load_links(*fieldgen.workload_links(dims))
        v = torch.zeros((2, 3, D.vh), dtype=D.dtype, device="cuda")
        for call in (lambda: D.apply_multi_blocked(torch.empty_like(v), v, 0),
                     lambda: D.to_blocked(torch.empty_like(v), v)):
            with pytest.raises(_abi.DslashError) as e:
                call()
            assert e.value.status == _abi.DSLASH_ERR_UNSUPPORTED
    dims = (8, 6, 8, 8)                           # t face 3 x 192 sites is whole blocks, z face 3 x 24 per t is not
    with Dslash(dims, force_halo=4) as D:
        D.load_links(*fieldgen.workload_links(dims))
        v = torch.zeros((2, 3, D.vh), dtype=D.dtype, device="cuda")
        with pytest.raises(_abi.DslashError) as e:
            D.apply_multi_blocked(torch.empty_like(v), v, 0)
        assert e.value.status == _abi.DSLASH_ERR_UNSUPPORTED
