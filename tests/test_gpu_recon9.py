"""recon-9 long-link compression (SURVEY §8(f)-2 "recon-12/9"): each long matrix is stored as the
8 parameters of its SU(3) part plus one phase, M = s e^{i psi} W, and rebuilt in registers
(stencil.cuh reconstruct_9).  1824 algorithmic bytes per site instead of 2400 (recon-18) or 2016
(recon-12).  Unlike recon-12 it accepts long links with folded staggered phases (det = -s^3) and
any U(1) phase per link."""
import numpy as np
import pytest

import fieldgen
import oracle

KERNELS = ["site", "dir2", "dir4"]


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    torch.cuda.set_device(0)
    return torch


def test_recon9_algorithmic_bytes():
    from paper_conf_sc_dufekgaad024_b200 import algo_bytes
    assert algo_bytes("f64", 9) == 1824 and algo_bytes("f64", 12) == 2016 and algo_bytes("f64", 18) == 2400
    assert algo_bytes("f64", 9, nrhs=4) == 1728 + 4 * 96
    assert algo_bytes("f32", 9) == 896 + 48 and algo_bytes("mixed", 9) == 896 + 96


def _phased_long_links(dims, seed=2):
    """-1/24 SU(3) long links times the staggered phase eta_mu(x) = (-1)^(x_0 + .. + x_{mu-1})
    (MILC folds it into the links, reading Z5) and a random U(1) phase per link."""
    lng = fieldgen.links(dims, seed, scale=fieldgen.LONG_SCALE)
    lx, ly, lz, lt = dims
    t, z, y, x = np.meshgrid(np.arange(lt), np.arange(lz), np.arange(ly), np.arange(lx), indexing="ij")
    coords = [x, y, z, t]
    rng = np.random.default_rng(seed)
    for mu in range(4):
        eta = (-1.0) ** sum(coords[:mu]) if mu else np.ones_like(x, dtype=float)
        phase = np.exp(1j * rng.uniform(-np.pi, np.pi, size=x.shape))
        lng[..., mu, :, :] *= (eta * phase)[..., None, None]
    return lng


@pytest.mark.gpu
@pytest.mark.parametrize("kernel", KERNELS)
@pytest.mark.parametrize("dims", [(8, 10, 12, 14), (4, 4, 4, 4)])
def test_recon9_vs_oracle(torch_cuda, kernel, dims):
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    fat, lng = fieldgen.workload_links(dims)
    psi = fieldgen.vector(dims, fieldgen.SEED_PSI)
    with Dslash(dims, kernel=kernel, recon=9) as D:
        D.load_links(fat, lng)
        for parity in (0, 1):
            ref = oracle.full_to_cb(oracle.dslash(fat, lng, psi, parity), parity)
            src = torch.from_numpy(fieldgen.vector_cb(dims, fieldgen.SEED_PSI, 1 - parity)).cuda()
            got = D(src, parity).cpu().numpy()
            assert oracle.normwise_error(got, ref) <= 1e-12


@pytest.mark.gpu
@pytest.mark.parametrize("kernel", KERNELS)
@pytest.mark.parametrize("precision", ["f32", "mixed"])
def test_recon9_reduced_precision_vs_oracle(torch_cuda, kernel, precision):
    """fp32 paired layout: the recon-9 parameters rounded to fp32, (psi_f, 0, psi_b, 0) in one
    float4; rebuilt in fp32 with the hardware sin/cos and rsqrt, then widened to fp64 for mixed;
    1e-5 against the fp64 oracle, and the error is above fp64 rounding (reduced precision really
    ran)."""
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 10, 12, 14)
    fat = fieldgen.links(dims, 1)
    lng = _phased_long_links(dims, 8)
    psi = fieldgen.vector(dims, 9)
    with Dslash(dims, kernel=kernel, recon=9, precision=precision) as D:
        D.load_links(fat, lng)
        for parity in (0, 1):
            ref = oracle.full_to_cb(oracle.dslash(fat, lng, psi, parity), parity)
            src = torch.from_numpy(fieldgen.vector_cb(dims, 9, 1 - parity)).to(D.dtype).cuda()
            got = D(src, parity).cpu().numpy().astype(np.complex128)
            err = oracle.normwise_error(got, ref)
            assert 1e-12 < err <= 1e-5, err


@pytest.mark.gpu
@pytest.mark.parametrize("kernel", KERNELS)
def test_recon9_folded_phases(torch_cuda, kernel):
    """Long links with staggered signs and U(1) phases: recon-9 reproduces the oracle, recon-12
    refuses them (its det is not one real s^3)."""
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash, _abi
    dims = (8, 8, 10, 12)
    fat = fieldgen.links(dims, 1)
    lng = _phased_long_links(dims)
    psi = fieldgen.vector(dims, 5)
    with Dslash(dims, kernel=kernel, recon=9) as D:
        D.load_links(fat, lng)
        for parity in (0, 1):
            ref = oracle.full_to_cb(oracle.dslash(fat, lng, psi, parity), parity)
            got = D(torch.from_numpy(fieldgen.vector_cb(dims, 5, 1 - parity)).cuda(), parity).cpu().numpy()
            assert oracle.normwise_error(got, ref) <= 1e-12
    with Dslash(dims, recon=12) as D:
        with pytest.raises(_abi.DslashError) as e:
            D.load_links(fat, lng)
        assert e.value.status == _abi.DSLASH_ERR_ARG


@pytest.mark.gpu
def test_recon9_halo_paths_and_rhs_bitwise(torch_cuda):
    """Self-halo (t, z, t+z), split by direction, producer push, staged and multi-RHS
    recon-9 applies against the unpartitioned recon-9 apply: bitwise where the per-site
    arithmetic is the same, within 1e-13 where the summation order differs."""
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 8, 8, 12)
    fat = fieldgen.links(dims, 1)
    lng = fieldgen.links(dims, 2, scale=0.37)   # another scale, found from |det N| = s^3
    srcs = torch.stack([torch.from_numpy(fieldgen.vector_cb(dims, 10 + r, 0)) for r in range(3)]).cuda()
    with Dslash(dims, recon=9) as D:
        D.load_links(fat, lng)
        base = torch.stack([D(srcs[r], 1) for r in range(3)]).cpu()
        multi = D.apply_multi(torch.empty_like(srcs), srcs, 1).cpu()
    assert torch.equal(base, multi)
    ref = oracle.full_to_cb(oracle.dslash(fat, lng, fieldgen.vector(dims, 10), 1), 1)
    assert oracle.normwise_error(base[0].numpy(), ref) <= 1e-12
    for kw, exact in (({"force_halo": 0x8}, True), ({"force_halo": 0xC}, True),
                      ({"force_halo": 0xC, "transport": "p2p", "push": True}, True),
                      ({"force_halo": 0xC, "overlap": "dirs"}, False),
                      ({"stage": True}, False)):
        with Dslash(dims, recon=9, **kw) as D:
            D.load_links(fat, lng)
            got = torch.stack([D(srcs[r], 1) for r in range(3)]).cpu()
        if exact:
            assert torch.equal(got, base), kw
        else:
            assert oracle.normwise_error(got.numpy(), base.numpy()) <= 1e-13, kw


@pytest.mark.gpu
def test_recon9_get_links_round_trip(torch_cuda):
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 8, 8, 8)
    fat = fieldgen.links(dims, 1)
    lng = _phased_long_links(dims, 3)
    with Dslash(dims, recon=9) as D:
        D.load_links(fat, lng)
        exp = {q: D.get_links(q) for q in (0, 1)}
    with Dslash(dims) as D:
        D.load_links(fat, lng)
        full = {q: D.get_links(q) for q in (0, 1)}
    for q in (0, 1):
        assert np.array_equal(exp[q][:, :, :2], full[q][:, :, :2])          # fat links stored as given
        err = np.abs(exp[q][:, :, 2:] - full[q][:, :, 2:]).max()
        assert err <= 1e-12 / 24, err                   # long links rebuilt (load_links' guarantee)


@pytest.mark.gpu
def test_recon9_rejections(torch_cuda):
    from paper_conf_sc_dufekgaad024_b200 import Dslash, _abi
    dims = (8, 8, 8, 8)
    fat = fieldgen.links(dims, 1)
    lng = fieldgen.links(dims, 2, scale=fieldgen.LONG_SCALE)
    for bad in (fieldgen.links(dims, 2, "gauss"),                              # not s e^{i psi} SU(3)
                np.broadcast_to(np.eye(3, dtype=np.complex128) / 24, lng.shape).copy()):   # singular set
        with Dslash(dims, recon=9) as D:
            with pytest.raises(_abi.DslashError) as e:
                D.load_links(fat, bad)
            assert e.value.status == _abi.DSLASH_ERR_ARG
    import torch
    fat = fieldgen.links(dims, 1)
    lng = fieldgen.links(dims, 2, scale=fieldgen.LONG_SCALE)
    with Dslash(dims, recon=9) as D:
        D.load_links(fat, lng)
        b = torch.from_numpy(fieldgen.vector_cb(dims, 4, 0)).cuda()
        ok, it, res = D.cg(D.empty_vector(), b, 0, 0.3, rel_tol=1e-10)   # the fp64 solver runs
        assert ok and res <= 2e-10


@pytest.mark.gpu
def test_recon9_mixed_cg(torch_cuda):
    """Mixed-precision CG on a recon-9 handle: the fp32 sloppy links are the recon-9 links rebuilt
    in fp64 and rounded once, stored in full; the answer solves the fp64 system like recon 18's."""
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 8, 8, 12)
    fat = fieldgen.links(dims, 1)
    lng = _phased_long_links(dims, 6)
    b = torch.from_numpy(fieldgen.vector_cb(dims, 7, 1)).cuda()
    sols = {}
    for recon in (18, 9):
        with Dslash(dims, recon=recon) as D:
            D.load_links(fat, lng)
            x = D.empty_vector()
            ok, it, outer, res = D.cg_mixed(x, b, 1, 0.3, rel_tol=1e-11, inner_tol=1e-3)
            assert ok and res <= 1e-11, (recon, res)
            x2 = D.empty_vector()
            D.cg(x2, b, 1, 0.3, rel_tol=1e-12)
            sols[recon] = (x.cpu().numpy(), x2.cpu().numpy())
    assert oracle.normwise_error(sols[9][0], sols[18][1]) <= 1e-9
    assert oracle.normwise_error(sols[9][1], sols[18][1]) <= 1e-10


@pytest.mark.gpu
def test_recon9_reduced_precision_error_budget(torch_cuda):
    """Regression guard on the accuracy of the fp32 recon-9 rebuild, 16^4, both
    parities, against the fp64 oracle: recon-9 may not be more than 12x (mixed) / 3x (f32) less
    accurate than recon-18 of the same precision.  Measured (profiles/r02/recon9_accuracy/): f32
    3.7e-7 vs 2.6e-7, mixed 2.4e-7 vs 2.7e-8 -- the fp32-stored parameters and the
    parameterisation's conditioning set it, and a 1e-7 -> 1e-6 regression would fail here."""
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (16, 16, 16, 16)
    fat, lng = fieldgen.workload_links(dims)
    psi = fieldgen.vector(dims, fieldgen.SEED_PSI)
    refs = {p: oracle.full_to_cb(oracle.dslash(fat, lng, psi, p), p) for p in (0, 1)}
    for precision, ratio in (("f32", 3.0), ("mixed", 12.0)):
        err = {}
        for recon in (18, 9):
            e = 0.0
            with Dslash(dims, precision=precision, recon=recon, kernel="site") as D:
                D.load_links(fat, lng)
                for p in (0, 1):
                    src = torch.from_numpy(fieldgen.vector_cb(dims, fieldgen.SEED_PSI, 1 - p)).to(D.dtype).cuda()
                    e = max(e, oracle.normwise_error(D(src, p).cpu().numpy().astype(np.complex128), refs[p]))
            err[recon] = e
        assert err[9] <= ratio * err[18], (precision, err)
        assert err[9] <= 5e-7, (precision, err)
