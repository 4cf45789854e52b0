"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Tolerance (reading Z11): normwise  max|chi - chi_ref| / max|chi_ref|
<= 1e-12 in fp64; summation order and FMA differ from the oracle, so bit equality with the
oracle is not expected.  Bitwise equality IS required between the unpartitioned apply and
the self-halo (interior + boundary) apply, and between repeated applies.
"""
import numpy as np
import pytest

import fieldgen
import oracle

pytestmark = pytest.mark.gpu

TOL = 1e-12
KERNELS = ["site", "dir2", "dir4"]


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    torch.cuda.set_device(0)
    return torch


def _gpu_apply(torch, dims, fat, lng, src_cb, parity, **kw):
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    with Dslash(dims, **kw) as D:
        D.load_links(fat, lng)
        out = D(torch.from_numpy(src_cb).cuda(), parity)
        torch.cuda.synchronize()
        return out.cpu().numpy()


# ragged: 6x8x10x12 has Vh = 2880 (not a multiple of the block); 4^4 aliases +3 with -1
SMALL = [(4, 4, 4, 4), (8, 8, 8, 8), (8, 10, 12, 14), (6, 8, 10, 12), (2, 4, 6, 8), (16, 16, 16, 16)]


@pytest.mark.parametrize("kernel", KERNELS)
@pytest.mark.parametrize("dims", SMALL)
@pytest.mark.parametrize("parity", [0, 1])
def test_parity_vs_oracle(torch_cuda, kernel, dims, parity):
    fat, lng = fieldgen.workload_links(dims)
    psi = fieldgen.vector(dims, fieldgen.SEED_PSI)
    ref = oracle.full_to_cb(oracle.dslash(fat, lng, psi, parity), parity)
    got = _gpu_apply(torch_cuda, dims, fat, lng, fieldgen.vector_cb(dims, fieldgen.SEED_PSI, 1 - parity), parity,
                     kernel=kernel)
    assert oracle.normwise_error(got, ref) <= TOL


@pytest.mark.parametrize("kernel", KERNELS)
def test_parity_gaussian_links(torch_cuda, kernel):
    """Non-unitary links: nothing in the kernel may assume SU(3) (reading Z14)."""
    dims = (8, 10, 12, 14)
    fat = fieldgen.links(dims, 101, "gauss")
    lng = fieldgen.links(dims, 102, "gauss", scale=0.3)
    psi = fieldgen.vector(dims, 103)
    for parity in (0, 1):
        ref = oracle.full_to_cb(oracle.dslash(fat, lng, psi, parity), parity)
        got = _gpu_apply(torch_cuda, dims, fat, lng, fieldgen.vector_cb(dims, 103, 1 - parity), parity, kernel=kernel)
        assert oracle.normwise_error(got, ref) <= TOL


@pytest.mark.parametrize("kernel", KERNELS)
def test_point_source_exact(torch_cuda, kernel):
    """P6 on the GPU: identity-scaled links and a point source give exact integers (bitwise)."""
    dims = (8, 10, 12, 14)
    lx, ly, lz, lt = dims
    fat = np.zeros((lt, lz, ly, lx, 4, 3, 3), np.complex128)
    lng = np.zeros_like(fat)
    fat[...] = np.eye(3)
    lng[...] = 2 * np.eye(3)
    x0 = (3, 7, 5, 11)
    psi = np.zeros((lt, lz, ly, lx, 3), np.complex128)
    psi[x0[3], x0[2], x0[1], x0[0]] = [1 + 2j, -3, 4 - 5j]
    parity = 1 - (sum(x0) & 1)
    ref = oracle.full_to_cb(oracle.dslash(fat, lng, psi, parity), parity)
    got = _gpu_apply(torch_cuda, dims, fat, lng, oracle.full_to_cb(psi, 1 - parity), parity, kernel=kernel)
    assert np.array_equal(got, ref)


@pytest.mark.parametrize("kernel", KERNELS)
@pytest.mark.parametrize("dims,mask", [((8, 8, 8, 8), 0x8), ((8, 8, 8, 8), 0x4), ((8, 8, 8, 8), 0xC),
                                       ((8, 10, 12, 14), 0xC), ((4, 4, 4, 4), 0xC), ((6, 8, 10, 12), 0x8)])
@pytest.mark.parametrize("overlap", [True, False])
def test_self_halo_bitwise(torch_cuda, kernel, dims, mask, overlap):
    """The halo path with neighbour = self (ghost faces; separate interior/boundary launches, or
    one launch after the exchange) must give the unpartitioned result bit for bit (same per-site
    device function), and match the oracle."""
    fat, lng = fieldgen.workload_links(dims)
    psi = fieldgen.vector(dims, fieldgen.SEED_PSI)
    for parity in (0, 1):
        src = fieldgen.vector_cb(dims, fieldgen.SEED_PSI, 1 - parity)
        plain = _gpu_apply(torch_cuda, dims, fat, lng, src, parity, kernel=kernel)
        halo = _gpu_apply(torch_cuda, dims, fat, lng, src, parity, kernel=kernel, force_halo=mask, overlap=overlap)
        assert np.array_equal(plain, halo)
        ref = oracle.full_to_cb(oracle.dslash(fat, lng, psi, parity), parity)
        assert oracle.normwise_error(halo, ref) <= TOL


@pytest.mark.parametrize("kernel", KERNELS)
@pytest.mark.parametrize("minb,block", [(2, 64), (3, 96), (4, 256), (2, 256)])
def test_launch_configs_agree(torch_cuda, kernel, minb, block):
    """Every register budget and block size gives the same bits for a given mapping (the
    mapping fixes the summation order), and the mappings agree to rounding."""
    dims = (16, 16, 16, 16)
    fat, lng = fieldgen.workload_links(dims)
    src = fieldgen.vector_cb(dims, 7, 1)
    base = _gpu_apply(torch_cuda, dims, fat, lng, src, 0, kernel=kernel)
    other = _gpu_apply(torch_cuda, dims, fat, lng, src, 0, kernel=kernel, min_blocks=minb, block=block)
    assert np.array_equal(base, other)
    ref = _gpu_apply(torch_cuda, dims, fat, lng, src, 0, kernel="site")
    assert oracle.normwise_error(base, ref) < 1e-14


@pytest.mark.parametrize("kernel", KERNELS)
def test_full_size_32(torch_cuda, kernel):
    """The benchmark size (32^4) in the bench's launch configuration, whole output vs the oracle."""
    dims = (32, 32, 32, 32)
    fat, lng = fieldgen.workload_links(dims)
    psi = fieldgen.vector(dims, fieldgen.SEED_PSI)
    parity = 0
    ref = oracle.full_to_cb(oracle.dslash(fat, lng, psi, parity), parity)
    got = _gpu_apply(torch_cuda, dims, fat, lng, fieldgen.vector_cb(dims, fieldgen.SEED_PSI, 1), parity,
                     kernel=kernel)
    assert oracle.normwise_error(got, ref) <= TOL


def test_sampled_48(torch_cuda):
    """48^4 (strong-scaling global lattice) on one GPU: 4096 sampled sites vs the oracle, one by one."""
    dims = (48, 48, 48, 48)
    fat, lng = fieldgen.workload_links(dims)
    psi = fieldgen.vector(dims, fieldgen.SEED_PSI)
    parity = 1
    got = _gpu_apply(torch_cuda, dims, fat, lng, fieldgen.vector_cb(dims, fieldgen.SEED_PSI, 0), parity)
    lex = oracle.lex_sites_of_parity(dims, parity)
    rng = np.random.default_rng(48)
    pick = np.sort(rng.choice(lex.size, 4096, replace=False))
    pick = np.concatenate([[0, 1, lex.size - 1], pick])          # first/last sites (wrap in every dim)
    ref = oracle.dslash_sites(fat, lng, psi, lex[pick])           # (n, 3)
    assert oracle.normwise_error(got[:, pick].T, ref) <= TOL


@pytest.mark.parametrize("mask", [0x8, 0xC])
def test_full_size_32_halo_path(torch_cuda, mask):
    """The per-GPU launch configuration of the weak-scaling bench (local 32^4, t-halo; plus z):
    interior + boundary kernels on two streams with the self-halo, bitwise equal to the
    unpartitioned apply at full size."""
    import torch
    from paper_conf_sc_dufekgaad024_b200 import Dslash, _abi
    dims = (32, 32, 32, 32)
    fat, lng = fieldgen.workload_links(dims)
    src = torch.from_numpy(fieldgen.vector_cb(dims, fieldgen.SEED_PSI, 1)).cuda()
    outs = []
    for m, ov in ((0, True), (mask, True), (mask, False)):
        with Dslash(dims, parity_mask=_abi.DSLASH_EVEN, force_halo=m, overlap=ov) as D:
            D.load_links(fat, lng)
            o = D.empty_vector()
            for _ in range(3):                       # repeated applies reuse the ghost buffers
                D.apply(o, src, 0)
            torch.cuda.synchronize()
            outs.append(o.cpu())
    assert torch.equal(outs[0], outs[1]) and torch.equal(outs[0], outs[2])


@pytest.mark.parametrize("recon", [18, 9])
def test_large_lattice_64x64x64x32(torch_cuda, recon):
    """A large local volume (Vh = 4.2M, 9.7 GB of links per parity): 64-bit indexing and grid
    sizes; 2048 sampled sites vs the oracle (first/last sites included).  recon-9 too: its load
    check must accept the 33 M long links of a random lattice (the rebuild's worst-link error grows
    with the lattice, DESIGN.md §12 f-2b)."""
    import torch
    from paper_conf_sc_dufekgaad024_b200 import Dslash, _abi
    dims = (64, 64, 64, 32)
    fat, lng = fieldgen.workload_links(dims)
    psi = fieldgen.vector(dims, fieldgen.SEED_PSI)
    parity = 0
    with Dslash(dims, parity_mask=_abi.DSLASH_EVEN, recon=recon, kernel="site" if recon == 9 else "dir2") as D:
        D.load_links(fat, lng)
        out = D(torch.from_numpy(fieldgen.vector_cb(dims, fieldgen.SEED_PSI, 1)).cuda(), parity)
        torch.cuda.synchronize()
        got = out.cpu().numpy()
    lex = oracle.lex_sites_of_parity(dims, parity)
    pick = np.concatenate([[0, 1, lex.size - 2, lex.size - 1],
                           np.sort(np.random.default_rng(64).choice(lex.size, 2048, replace=False))])
    ref = oracle.dslash_sites(fat, lng, psi, lex[pick])
    assert oracle.normwise_error(got[:, pick].T, ref) <= TOL


def test_antihermitian_gpu(torch_cuda):
    """P3 through the library: <chi_e, D_eo psi_o> = -<D_oe chi_e, psi_o>."""
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    torch = torch_cuda
    dims = (8, 10, 12, 14)
    fat, lng = fieldgen.workload_links(dims)
    with Dslash(dims) as D:
        D.load_links(fat, lng)
        psi_o = torch.from_numpy(fieldgen.vector_cb(dims, 5, 1)).cuda()
        chi_e = torch.from_numpy(fieldgen.vector_cb(dims, 6, 0)).cuda()
        d_psi = D(psi_o, 0)
        d_chi = D(chi_e, 1)
        lhs = torch.vdot(chi_e.reshape(-1), d_psi.reshape(-1)).item()
        rhs = -torch.vdot(d_chi.reshape(-1), psi_o.reshape(-1)).item()
        scale = (chi_e.norm() * d_psi.norm()).item()
        assert abs(lhs - rhs) < 1e-13 * scale


def test_apply_host_and_determinism(torch_cuda):
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    torch = torch_cuda
    dims = (8, 8, 8, 16)
    fat, lng = fieldgen.workload_links(dims)
    with Dslash(dims) as D:
        D.load_links(fat, lng)
        src = torch.from_numpy(fieldgen.vector_cb(dims, 3, 1))
        a = D(src.cuda(), 0)
        b = D(src.cuda(), 0)
        hout = torch.empty_like(src).pin_memory()
        D.apply_host(hout, src.pin_memory(), 0)
        torch.cuda.synchronize()
        assert torch.equal(a, b)
        assert torch.equal(a.cpu(), hout)


def test_apply_host_batch(torch_cuda):
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    torch = torch_cuda
    dims = (8, 8, 8, 16)
    fat, lng = fieldgen.workload_links(dims)
    with Dslash(dims, force_halo=0x8) as D:
        D.load_links(fat, lng)
        ins = [torch.from_numpy(fieldgen.vector_cb(dims, 30 + i, 0)).pin_memory() for i in range(7)]
        outs = [torch.empty_like(ins[0]).pin_memory() for _ in range(7)]
        D.apply_host_batch(outs, ins, 1)
        torch.cuda.synchronize()
        for i in range(7):
            assert torch.equal(outs[i], D(ins[i].cuda(), 1).cpu())
        D.apply_host_batch([], [], 1)          # empty batch is a no-op


def test_device_links_equal_host_links(torch_cuda):
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    torch = torch_cuda
    dims = (8, 8, 8, 8)
    fat, lng = fieldgen.workload_links(dims)
    src = torch.from_numpy(fieldgen.vector_cb(dims, 3, 0)).cuda()
    with Dslash(dims) as D:
        D.load_links(fat, lng)
        a = D(src, 1)
        D.load_links(torch.from_numpy(fat).cuda(), torch.from_numpy(lng).cuda())
        b = D(src, 1)
        torch.cuda.synchronize()
        assert torch.equal(a, b)


@pytest.mark.parametrize("precision,tol", [("f32", 1e-5), ("mixed", 1e-5)])
@pytest.mark.parametrize("kernel", KERNELS)
@pytest.mark.parametrize("dims", [(8, 10, 12, 14), (4, 4, 4, 4), (6, 8, 10, 12)])
def test_reduced_precision_vs_fp64_oracle(torch_cuda, precision, tol, kernel, dims):
    """§8(f)-1: fp32 and mixed paths against the fp64 oracle on the fp64 inputs, normwise 1e-5
    (north star).  The fp32 input vector is the fp64 one rounded."""
    import torch
    fat, lng = fieldgen.workload_links(dims)
    psi = fieldgen.vector(dims, fieldgen.SEED_PSI)
    for parity in (0, 1):
        ref = oracle.full_to_cb(oracle.dslash(fat, lng, psi, parity), parity)
        src = torch.from_numpy(fieldgen.vector_cb(dims, fieldgen.SEED_PSI, 1 - parity))
        from paper_conf_sc_dufekgaad024_b200 import Dslash
        with Dslash(dims, kernel=kernel, precision=precision) as D:
            D.load_links(fat, lng)
            out = D(src.to(D.dtype).cuda(), parity)
            torch.cuda.synchronize()
            got = out.cpu().numpy().astype(np.complex128)
        err = oracle.normwise_error(got, ref)
        assert err <= tol
        assert err > 1e-12          # it really ran in reduced precision


@pytest.mark.parametrize("precision", ["f32", "mixed"])
def test_reduced_precision_self_halo_bitwise(torch_cuda, precision):
    import torch
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 8, 8, 12)
    fat, lng = fieldgen.workload_links(dims)
    outs = []
    for mask in (0, 0xC):
        with Dslash(dims, precision=precision, force_halo=mask) as D:
            D.load_links(fat, lng)
            src = torch.from_numpy(fieldgen.vector_cb(dims, 3, 0)).to(D.dtype).cuda()
            outs.append(D(src, 1).cpu())
    assert torch.equal(outs[0], outs[1])


@pytest.mark.parametrize("kernel", KERNELS)
@pytest.mark.parametrize("precision,tol", [("f64", 1e-12), ("mixed", 1e-5), ("f32", 1e-5)])
@pytest.mark.parametrize("dims", [(8, 10, 12, 14), (4, 4, 4, 4)])
def test_recon12_vs_oracle(torch_cuda, kernel, precision, tol, dims):
    """§8(f)-2: long links stored as two rows, row 2 rebuilt as conj(r0 x r1)/s in registers."""
    import torch
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    fat, lng = fieldgen.workload_links(dims)
    psi = fieldgen.vector(dims, fieldgen.SEED_PSI)
    for parity in (0, 1):
        ref = oracle.full_to_cb(oracle.dslash(fat, lng, psi, parity), parity)
        src = torch.from_numpy(fieldgen.vector_cb(dims, fieldgen.SEED_PSI, 1 - parity))
        with Dslash(dims, kernel=kernel, precision=precision, recon=12) as D:
            D.load_links(fat, lng)
            got = D(src.to(D.dtype).cuda(), parity).cpu().numpy().astype(np.complex128)
        assert oracle.normwise_error(got, ref) <= tol


def test_recon12_self_halo_and_scale(torch_cuda):
    """recon-12 through the halo path is bitwise the unpartitioned recon-12 result; a long-link
    scale other than -1/24 is found from det(N) = s^3."""
    import torch
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 8, 8, 12)
    fat = fieldgen.links(dims, 1)
    lng = fieldgen.links(dims, 2, scale=0.37)
    psi = fieldgen.vector(dims, 3)
    src = torch.from_numpy(fieldgen.vector_cb(dims, 3, 0)).cuda()
    outs = []
    for mask in (0, 0xC):
        with Dslash(dims, recon=12, force_halo=mask) as D:
            D.load_links(fat, lng)
            outs.append(D(src, 1).cpu())
    assert torch.equal(outs[0], outs[1])
    ref = oracle.full_to_cb(oracle.dslash(fat, lng, psi, 1), 1)
    assert oracle.normwise_error(outs[0].numpy(), ref) <= 1e-12


def test_recon12_rejects_non_su3_long_links(torch_cuda):
    from paper_conf_sc_dufekgaad024_b200 import Dslash, _abi
    dims = (8, 8, 8, 8)
    fat = fieldgen.links(dims, 1)
    with Dslash(dims, recon=12) as D:
        with pytest.raises(_abi.DslashError) as e:
            D.load_links(fat, fieldgen.links(dims, 2, "gauss"))          # not unitary
        assert e.value.status == _abi.DSLASH_ERR_ARG
    lng = fieldgen.links(dims, 2, scale=-1 / 24)
    lng[1, 2, 3, 4, 2] *= -1                                              # one link with the other sign
    with Dslash(dims, recon=12) as D:
        with pytest.raises(_abi.DslashError) as e:
            D.load_links(fat, lng)
        assert e.value.status == _abi.DSLASH_ERR_ARG


@pytest.mark.parametrize("kernel", KERNELS)
@pytest.mark.parametrize("nrhs", [1, 2, 3, 5, 8, 11])
@pytest.mark.parametrize("mask", [0, 0xC])
def test_multi_rhs_bitwise_and_oracle(torch_cuda, kernel, nrhs, mask):
    """§8(f)-4: one link pass for nrhs vectors gives, for every right-hand side, the bits of the
    single-vector apply (same per-thread arithmetic) and matches the oracle."""
    import torch
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 10, 12, 14) if mask == 0 else (8, 8, 8, 12)
    fat, lng = fieldgen.workload_links(dims)
    parity = 1
    src = torch.stack([torch.from_numpy(fieldgen.vector_cb(dims, 40 + r, 0)) for r in range(nrhs)]).cuda()
    with Dslash(dims, kernel=kernel, force_halo=mask) as D:
        D.load_links(fat, lng)
        out = torch.empty_like(src)
        D.apply_multi(out, src, parity)
        singles = torch.stack([D(src[r].contiguous(), parity) for r in range(nrhs)])
        torch.cuda.synchronize()
    assert torch.equal(out, singles)
    for r in (0, nrhs - 1):
        psi = fieldgen.vector(dims, 40 + r)
        ref = oracle.full_to_cb(oracle.dslash(fat, lng, psi, parity), parity)
        assert oracle.normwise_error(out[r].cpu().numpy(), ref) <= TOL


@pytest.mark.parametrize("precision,recon", [("f32", 18), ("mixed", 12), ("f64", 12)])
def test_multi_rhs_precisions(torch_cuda, precision, recon):
    import torch
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 10, 12, 14)
    fat, lng = fieldgen.workload_links(dims)
    with Dslash(dims, precision=precision, recon=recon) as D:
        D.load_links(fat, lng)
        src = torch.stack([torch.from_numpy(fieldgen.vector_cb(dims, 50 + r, 1)) for r in range(4)]).to(D.dtype).cuda()
        out = torch.empty_like(src)
        D.apply_multi(out, src, 0)
        singles = torch.stack([D(src[r].contiguous(), 0) for r in range(4)])
        torch.cuda.synchronize()
    assert torch.equal(out, singles)


def test_error_paths(torch_cuda):
    from paper_conf_sc_dufekgaad024_b200 import Dslash, _abi
    torch = torch_cuda
    dims = (8, 8, 8, 8)
    D = Dslash(dims, parity_mask=_abi.DSLASH_EVEN)
    v = D.empty_vector()
    w = D.empty_vector()
    with pytest.raises(_abi.DslashError) as e:
        D.apply(v, w, 0)
    assert e.value.status == _abi.DSLASH_ERR_STATE
    fat, lng = fieldgen.workload_links(dims)
    D.load_links(fat, lng)
    with pytest.raises(_abi.DslashError) as e:
        _abi.dslash_apply(D.h, v.data_ptr(), v.data_ptr(), 0, 0)         # in == out
    assert e.value.status == _abi.DSLASH_ERR_ARG
    with pytest.raises(_abi.DslashError) as e:
        D.apply(v, w, 1)                                                  # parity not prepared
    assert e.value.status == _abi.DSLASH_ERR_ARG
    with pytest.raises(_abi.DslashError) as e:
        _abi.dslash_apply(D.h, v.data_ptr(), w.data_ptr(), 2, 0)         # bad parity
    assert e.value.status == _abi.DSLASH_ERR_ARG
    with pytest.raises(_abi.DslashError) as e:
        _abi.dslash_apply(D.h, v.data_ptr() + 8, w.data_ptr(), 0, 0)     # misaligned
    assert e.value.status == _abi.DSLASH_ERR_ARG
    with pytest.raises(_abi.DslashError) as e:
        _abi.dslash_set_option(D.h, _abi.DSLASH_OPT_KERNEL, _abi.DSLASH_KERNEL_DIR4)  # after load_links
    assert e.value.status == _abi.DSLASH_ERR_STATE
    D.close()
    with pytest.raises(_abi.DslashError) as e:
        Dslash((8, 8, 8, 8), proc_grid=(1, 1, 1, 2))                       # nranks mismatch
    assert e.value.status == _abi.DSLASH_ERR_ARG


def test_kernel_timing_records(torch_cuda):
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    torch = torch_cuda
    dims = (8, 8, 8, 16)
    fat, lng = fieldgen.workload_links(dims)
    with Dslash(dims, timing=True, force_halo=0x8) as D:
        D.load_links(fat, lng)
        src = torch.from_numpy(fieldgen.vector_cb(dims, 3, 1)).cuda()
        out = D.empty_vector()
        for _ in range(3):
            D.apply(out, src, 0)
        for _ in range(40):        # enough timed launches to grow the event pool repeatedly
            D.apply(out, src, 0)
        ms, n = D.kernel_timing()
        assert n == 86 and ms > 0  # interior + boundary per apply
        assert D.kernel_timing(0)[1] == 43 and D.kernel_timing(1)[1] == 43
        span_ms, n_span = D.kernel_timing(3)
        assert n_span == 43 and span_ms > 0
        D.kernel_timing_reset()
        assert D.kernel_timing()[1] == 0


@pytest.mark.parametrize("mask", [0x8, 0x4, 0xC])
def test_p2p_transport_self_halo(torch_cuda, mask):
    """The P2P transport (copy-engine face puts + stream-memory epoch flags) with neighbour =
    self: several epochs through the same ghosts, single and multi-RHS, bitwise equal to the
    unpartitioned apply."""
    import torch
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 8, 8, 12)
    fat, lng = fieldgen.workload_links(dims)
    srcs = torch.stack([torch.from_numpy(fieldgen.vector_cb(dims, 60 + r, 0)) for r in range(3)]).cuda()
    with Dslash(dims) as D:
        D.load_links(fat, lng)
        ref = torch.stack([D(srcs[r].contiguous(), 1) for r in range(3)]).cpu()
    with Dslash(dims, force_halo=mask, transport="p2p") as D:
        D.load_links(fat, lng)
        for it in range(4):
            for r in range(3):
                out = D(srcs[r].contiguous(), 1)
                assert torch.equal(out.cpu(), ref[r]), (it, r)
        multi = torch.empty_like(srcs)
        D.apply_multi(multi, srcs, 1)
        torch.cuda.synchronize()
        assert torch.equal(multi.cpu(), ref)


@pytest.mark.parametrize("mask", [0x8, 0xC])
def test_p2p_epochs_across_modes(torch_cuda, mask):
    """The P2P epoch counter is one monotonic sequence whatever launches an exchange: multi-RHS
    applies, split-by-sites, split-by-direction and no-overlap applies interleaved, each with a
    different source, every result bitwise equal to the unpartitioned apply (a stale ghost face
    from an earlier epoch would change the boundary sites)."""
    import torch
    from paper_conf_sc_dufekgaad024_b200 import Dslash, _abi
    dims = (8, 8, 8, 12)
    fat, lng = fieldgen.workload_links(dims)
    srcs = torch.stack([torch.from_numpy(fieldgen.vector_cb(dims, 70 + r, 0)) for r in range(6)]).cuda()
    with Dslash(dims) as D:
        D.load_links(fat, lng)
        ref = torch.stack([D(srcs[r].contiguous(), 1) for r in range(6)]).cpu()
    with Dslash(dims, force_halo=mask, transport="p2p") as D:
        D.load_links(fat, lng)
        multi = torch.empty_like(srcs[:2])
        D.apply_multi(multi, srcs[:2].contiguous(), 1)
        assert torch.equal(multi.cpu(), ref[:2])
        for r, mode in zip(range(2, 6), ("dirs", "none", "sites", "dirs")):
            _abi.dslash_set_option(D.h, _abi.DSLASH_OPT_OVERLAP, _abi.OVERLAPS[mode])
            out = D(srcs[r].contiguous(), 1)
            torch.cuda.synchronize()
            if mode == "dirs":   # boundary sites sum in another order: equal within rounding
                assert oracle.normwise_error(out.cpu().numpy(), ref[r].numpy()) < 1e-14, (r, mode)
            else:
                assert torch.equal(out.cpu(), ref[r]), (r, mode)


@pytest.mark.parametrize("kernel", ["site", "dir2", "dir4"])
@pytest.mark.parametrize("mask", [0, 0xC])
def test_load_links_layout_roundtrip(torch_cuda, kernel, mask):
    """Row a0 bitwise: the internal arrays hold exactly F(x,mu), F(x-mu,mu)^dag, N(x,mu) and
    N(x-3mu,mu)^dag for every target site (built here with numpy rolls of the canonical input),
    in every kernel layout, through the local and the halo-slab paths."""
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (16, 8, 8, 12)
    fat = fieldgen.links(dims, 81, "gauss")
    lng = fieldgen.links(dims, 82, "gauss")
    AX = {0: 3, 1: 2, 2: 1, 3: 0}
    dag = lambda m: np.conj(np.swapaxes(m, -1, -2))
    with Dslash(dims, kernel=kernel, force_halo=mask) as D:
        D.load_links(fat, lng)
        for parity in (0, 1):
            got = D.get_links(parity)                       # (Vh, mu, l, 3, 3)
            lex = oracle.lex_sites_of_parity(dims, parity)
            for mu in range(4):
                fb = dag(np.roll(fat[..., mu, :, :], 1, axis=AX[mu]))
                nb = dag(np.roll(lng[..., mu, :, :], 3, axis=AX[mu]))
                for l, arr in enumerate((fat[..., mu, :, :], fb, lng[..., mu, :, :], nb)):
                    assert np.array_equal(got[:, mu, l], arr.reshape(-1, 3, 3)[lex]), (parity, mu, l)


def test_c_api_demo_runs(torch_cuda):
    """examples/c_api_demo (plain C, no Python binding): create / load_links / apply_host / sync /
    destroy, anti-Hermiticity to 1e-12."""
    import os
    import subprocess
    from paper_conf_sc_dufekgaad024_b200 import build
    exe = build.build_c_demo()
    for dims in (["8", "8", "8", "16"], ["8", "10", "12", "14"]):
        r = subprocess.run([exe, *dims], capture_output=True, text=True, timeout=120)
        assert r.returncode == 0, r.stdout + r.stderr
        assert "rel.diff" in r.stdout


@pytest.mark.parametrize("kernel", ["dir2", "site", "dir4"])
def test_pdl_chained_applies_bitwise(torch_cuda, kernel):
    """Programmatic dependent launch: a chain x_{k+1} = D x_k (alternating parity, each apply
    reading the previous one's output) must give the same bits as ordinary launches; the
    kernel reads psi only after griddepcontrol.wait."""
    import torch
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (16, 16, 16, 16)
    fat, lng = fieldgen.workload_links(dims)
    x0 = torch.from_numpy(fieldgen.vector_cb(dims, 9, 1)).cuda()
    res = []
    for pdl in (False, True):
        with Dslash(dims, kernel=kernel, pdl=pdl) as D:
            D.load_links(fat, lng)
            xs = [x0] + [D.empty_vector() for _ in range(12)]
            for k in range(12):
                D.apply(xs[k + 1], xs[k], k % 2)          # x_k has parity 1 - (k % 2)
                xs[k + 1].mul_(0.05)                       # interleaved torch kernel on the stream
            torch.cuda.synchronize()
            res.append(torch.stack([x.cpu() for x in xs]))
    assert torch.equal(res[0], res[1])


@pytest.mark.parametrize("mask", [0x8, 0x4, 0xC])
@pytest.mark.parametrize("kernel", ["dir2", "site"])
def test_nccl_transport_self_halo(torch_cuda, mask, kernel):
    """The NCCL transport run for real on one GPU (DSLASH_OPT_SELF_NCCL): a one-rank
    communicator, faces and link slabs sent with ncclSend/ncclRecv to this rank in the P = 2
    message pattern (both neighbours one peer, matched in issue order).  Several epochs, single
    and multi-RHS, bitwise equal to the unpartitioned apply; the NCCL face order and the ghost
    layout are the ones a 2-rank t / z partition uses."""
    import torch
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 8, 8, 12)
    fat, lng = fieldgen.workload_links(dims)
    srcs = torch.stack([torch.from_numpy(fieldgen.vector_cb(dims, 90 + r, 1)) for r in range(3)]).cuda()
    with Dslash(dims, kernel=kernel) as D:
        D.load_links(fat, lng)
        ref = torch.stack([D(srcs[r].contiguous(), 0) for r in range(3)]).cpu()
    with Dslash(dims, kernel=kernel, force_halo=mask, self_nccl=True) as D:
        D.load_links(fat, lng)
        for it in range(3):
            for r in range(3):
                out = D(srcs[r].contiguous(), 0)
                assert torch.equal(out.cpu(), ref[r]), (it, r)
        multi = torch.empty_like(srcs)
        D.apply_multi(multi, srcs, 0)
        torch.cuda.synchronize()
        assert torch.equal(multi.cpu(), ref)
    # the oracle as well, so a consistently wrong face (both paths) cannot pass
    psi = fieldgen.vector(dims, 90)
    want = oracle.full_to_cb(oracle.dslash(fat, lng, psi, 0), 0)
    assert oracle.normwise_error(ref[0].numpy(), want) <= TOL


def test_nccl_self_option_errors(torch_cuda):
    from paper_conf_sc_dufekgaad024_b200 import Dslash, DslashError, _abi
    dims = (8, 8, 8, 12)
    with Dslash(dims, force_halo=0x8) as D:     # no communicator
        with pytest.raises(DslashError):
            _abi.dslash_set_option(D.h, _abi.DSLASH_OPT_SELF_NCCL, 1)
    fat, lng = fieldgen.workload_links(dims)
    with Dslash(dims, force_halo=0x8, self_nccl=True) as D:
        D.load_links(fat, lng)
        with pytest.raises(DslashError):           # after load_links
            _abi.dslash_set_option(D.h, _abi.DSLASH_OPT_SELF_NCCL, 0)


@pytest.mark.parametrize("mask", [0x8, 0x4, 0xC])
def test_load_links_halo_caller_slabs(torch_cuda, mask):
    """dslash_load_links_halo: the caller hands over the 3 link slices below the origin (here,
    with neighbour = self, the lattice's own top slices, host memory); the internal links equal
    those of the library's own exchange bitwise."""
    import ctypes
    from paper_conf_sc_dufekgaad024_b200 import Dslash, _abi
    dims = (8, 10, 12, 14)
    fat = fieldgen.links(dims, 91, "gauss")
    lng = fieldgen.links(dims, 92, "gauss")
    with Dslash(dims, force_halo=mask) as D:
        D.load_links(fat, lng)
        want = [D.get_links(q) for q in (0, 1)]
    keep = []
    sf, sl = [0] * 4, [0] * 4
    for d, axis in ((3, 0), (2, 1)):
        if not (mask >> d) & 1:
            continue
        for k, arr in enumerate((fat, lng)):
            top = np.ascontiguousarray(np.take(arr, range(arr.shape[axis] - 3, arr.shape[axis]), axis=axis))
            keep.append(top)
            (sf if k == 0 else sl)[d] = top.ctypes.data
    with Dslash(dims, force_halo=mask) as D:
        _abi.dslash_load_links_halo(D.h, fat.ctypes.data, lng.ctypes.data, sf, sl, 0, 0)
        got = [D.get_links(q) for q in (0, 1)]
    for q in (0, 1):
        assert np.array_equal(got[q], want[q])


@pytest.mark.parametrize("args", [["2", "8", "8", "8", "16"], ["3", "8", "10", "12", "18"], ["4", "8", "8", "8", "32"]])
def test_c_p2p_demo_runs(torch_cuda, args):
    """examples/c_p2p_demo (plain C, forked ranks, no Python in the ranks): a t-partitioned P2P
    run whose link halo and face exchanges the library does itself; the gathered result equals
    the 1-rank apply bitwise."""
    import subprocess
    from paper_conf_sc_dufekgaad024_b200 import build
    exe = build.build_c_demo("c_p2p_demo")
    r = subprocess.run([exe, *args], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stdout + r.stderr
    assert "EQUALS" in r.stdout
