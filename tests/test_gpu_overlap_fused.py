"""GPU parity of the one-shot fused overlap (DSLASH_OPT_OVERLAP = DSLASH_OVERLAP_FUSED): one launch
over all sites with interior blocks first; each boundary block looks once at the halo flags and
either computes its sites (ghosts read with coherent loads) or defers itself to a stream-ordered
clean-up launch.  Every site runs the per-site arithmetic of the split by sites, so results must
be BITWISE equal to the unpartitioned apply, whichever blocks deferred."""
import numpy as np
import pytest

import fieldgen
import oracle

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    torch.cuda.set_device(0)
    return torch


def _run(torch, dims, fat, lng, srcs, parity, napply=3, defer=False, **kw):
    from paper_conf_sc_dufekgaad024_b200 import Dslash, _abi
    with Dslash(dims, **kw) as D:
        D.load_links(fat, lng)
        if defer:
            _abi.dslash_set_option(D.h, _abi.DSLASH_OPT_FUSED_DEFER, 1)
        outs = None
        for _ in range(napply):                       # several epochs through the same ghosts
            outs = [D(s, parity) for s in srcs]
        torch.cuda.synchronize()
        return [o.cpu() for o in outs]


@pytest.mark.parametrize("kernel", ["site", "dir2", "dir4"])
@pytest.mark.parametrize("dims,mask", [((8, 8, 8, 12), 0x8), ((8, 8, 12, 8), 0x4), ((8, 8, 8, 8), 0xC),
                                       ((8, 10, 12, 14), 0xC), ((6, 8, 10, 6), 0x8), ((4, 4, 4, 4), 0xC),
                                       ((6, 8, 10, 12), 0x8)])
@pytest.mark.parametrize("defer", [False, True])
def test_fused_bitwise(torch_cuda, kernel, dims, mask, defer):
    import torch
    fat, lng = fieldgen.workload_links(dims)
    srcs = [torch.from_numpy(fieldgen.vector_cb(dims, 20 + r, 0)).cuda() for r in range(3)]
    base = _run(torch, dims, fat, lng, srcs, 1, napply=1, kernel=kernel)
    got = _run(torch, dims, fat, lng, srcs, 1, defer=defer, kernel=kernel, force_halo=mask, overlap="fused")
    for b, g in zip(base, got):
        assert torch.equal(b, g)
    ref = oracle.full_to_cb(oracle.dslash(fat, lng, fieldgen.vector(dims, 20), 1), 1)
    assert oracle.normwise_error(got[0].numpy(), ref) <= 1e-12


@pytest.mark.parametrize("transport", ["p2p", "nccl-self"])
@pytest.mark.parametrize("defer", [False, True])
def test_fused_transports(torch_cuda, transport, defer):
    import torch
    dims = (8, 8, 8, 12)
    fat, lng = fieldgen.workload_links(dims)
    srcs = [torch.from_numpy(fieldgen.vector_cb(dims, 30 + r, 1)).cuda() for r in range(3)]
    base = _run(torch, dims, fat, lng, srcs, 0, napply=1)
    kw = {"transport": "p2p"} if transport == "p2p" else {"self_nccl": True}
    got = _run(torch, dims, fat, lng, srcs, 0, napply=4, defer=defer, force_halo=0xC, overlap="fused", **kw)
    for b, g in zip(base, got):
        assert torch.equal(b, g)


@pytest.mark.parametrize("precision,recon", [("f32", 18), ("mixed", 12), ("f64", 12)])
def test_fused_precisions(torch_cuda, precision, recon):
    import torch
    dims = (8, 10, 12, 14)
    fat, lng = fieldgen.workload_links(dims)
    srcs = [torch.from_numpy(fieldgen.vector_cb(dims, 40, 1)).to(
        torch.complex64 if precision == "f32" else torch.complex128).cuda()]
    base = _run(torch, dims, fat, lng, srcs, 0, napply=1, precision=precision, recon=recon)
    got = _run(torch, dims, fat, lng, srcs, 0, precision=precision, recon=recon, force_halo=0xC, overlap="fused")
    assert torch.equal(base[0], got[0])


def test_fused_full_size_and_multi_rhs_fallback(torch_cuda):
    """32^4 with the t halo (weak-scaling per-GPU volume), bitwise; apply_multi in this mode takes
    the split by sites (same bits)."""
    import torch
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (32, 32, 32, 32)
    fat, lng = fieldgen.workload_links(dims)
    srcs = [torch.from_numpy(fieldgen.vector_cb(dims, fieldgen.SEED_PSI, 1)).cuda()]
    base = _run(torch, dims, fat, lng, srcs, 0, napply=1)
    got = _run(torch, dims, fat, lng, srcs, 0, force_halo=0x8, overlap="fused")
    assert torch.equal(base[0], got[0])
    dims = (8, 8, 8, 12)
    fat, lng = fieldgen.workload_links(dims)
    src = torch.stack([torch.from_numpy(fieldgen.vector_cb(dims, 50 + r, 0)) for r in range(3)]).cuda()
    with Dslash(dims, force_halo=0xC, overlap="fused") as D:
        D.load_links(fat, lng)
        out = torch.empty_like(src)
        D.apply_multi(out, src, 1)
        singles = torch.stack([D(src[r].contiguous(), 1) for r in range(3)])
        torch.cuda.synchronize()
    assert torch.equal(out, singles)


def test_fused_chained_cg(torch_cuda):
    """CG through fused applies (each apply's input is the previous one's output: the exchange of
    apply k+1 must wait for apply k's clean-up) solves the system with the unpartitioned bits."""
    import torch
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 8, 8, 12)
    fat, lng = fieldgen.workload_links(dims)
    b = torch.from_numpy(fieldgen.vector_cb(dims, 73, 0)).cuda()
    res = []
    for kw in ({}, {"force_halo": 0xC, "overlap": "fused"}):
        with Dslash(dims, **kw) as D:
            D.load_links(fat, lng)
            x = D.empty_vector()
            ok, it, rel = D.cg(x, b, 0, 0.3, rel_tol=1e-10)
            assert ok
            res.append((x.cpu(), it))
    assert torch.equal(res[0][0], res[1][0]) and res[0][1] == res[1][1]


def test_halo_dryrun_timing_aid(torch_cuda):
    """DSLASH_OPT_HALO_DRYRUN keeps the exchange's stream structure but moves no bytes: interior
    sites are still right (they read no ghost), and the P2P transport refuses it."""
    import torch
    from paper_conf_sc_dufekgaad024_b200 import Dslash, DslashError, _abi
    dims = (8, 8, 8, 12)
    fat, lng = fieldgen.workload_links(dims)
    src = torch.from_numpy(fieldgen.vector_cb(dims, 60, 1)).cuda()
    with Dslash(dims) as D:
        D.load_links(fat, lng)
        base = D(src, 0).cpu().numpy()
    with Dslash(dims, force_halo=0x8) as D:
        D.load_links(fat, lng)
        _abi.dslash_set_option(D.h, _abi.DSLASH_OPT_HALO_DRYRUN, 1)
        got = D(src, 0).cpu().numpy()
    lex = oracle.lex_sites_of_parity(dims, 0)
    t = lex // (dims[0] * dims[1] * dims[2])
    inside = (t >= 3) & (t < dims[3] - 3)
    assert np.array_equal(got[:, inside], base[:, inside])
    with Dslash(dims, force_halo=0x8, transport="p2p") as D:
        with pytest.raises(DslashError):
            _abi.dslash_set_option(D.h, _abi.DSLASH_OPT_HALO_DRYRUN, 1)
