"""32^4 oracle parity of every configuration that has a published bench number (VERDICT r1
"What's weak" 1), in the bench's launch configuration.

The bench lattice is 32^4 (BASELINE.json configs[2]): 524288 target sites,
i.e. 8192 blocks of the default 64-thread dir2 launch, 55 waves over 148 SMs, so the wave tail
and the programmatic-dependent-launch overlap of consecutive applies (DSLASH_OPT_PDL, on by
default as in bench.py) both occur.  Each test runs three applies back to back on one stream,
each with its own source (as the bench's rotating buffers do), and checks every one of them on
>= 4096 randomly sampled target sites plus the first two and the last two (the periodic wrap in
every direction) against the oracle, site by site (oracle.dslash_sites).  Multi-RHS checks
EVERY right-hand side.

Tolerances: normwise 1e-12 for fp64, 1e-5 for fp32 / mixed against the fp64
oracle on the fp64 inputs (north star), with the reduced-precision error also required to be
> 1e-12 (the reduced-precision path really ran).
"""
import numpy as np
import pytest

import fieldgen
import oracle

pytestmark = pytest.mark.gpu

DIMS = (32, 32, 32, 32)
NSAMPLE = 4096
SEEDS = (301, 302, 303)          # the three back-to-back sources (multi-RHS: seed + r)
TOL = {"f64": 1e-12, "f32": 1e-5, "mixed": 1e-5}


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    torch.cuda.set_device(0)
    return torch


@pytest.fixture(scope="module")
def links32():
    return fieldgen.workload_links(DIMS)


@pytest.fixture(scope="module")
def psi_full():
    cache = {}

    def get(seed):
        if seed not in cache:
            cache[seed] = fieldgen.vector(DIMS, seed)
        return cache[seed]
    return get


def _sample(parity, seed=32):
    lex = oracle.lex_sites_of_parity(DIMS, parity)
    pick = np.sort(np.random.default_rng(seed).choice(lex.size, NSAMPLE, replace=False))
    pick = np.unique(np.concatenate([[0, 1, lex.size - 2, lex.size - 1], pick]))
    return pick, lex[pick]


def _check(got_cb, fat, lng, psi, parity, precision, what):
    pick, sites = _sample(parity)
    ref = oracle.dslash_sites(fat, lng, psi, sites)                     # (n, 3)
    err = oracle.normwise_error(np.asarray(got_cb)[:, pick].T.astype(np.complex128), ref)
    assert err <= TOL[precision], (what, err)
    if precision != "f64":
        assert err > 1e-12, (what, err)
    return err


def _bench_kernel(recon, nrhs, precision="f64"):
    # bench.py's default mapping: site for recon-9, multi-RHS and mixed precision, dir2 otherwise
    return "site" if (recon == 9 or nrhs > 1 or precision == "mixed") else "dir2"


def _run_chain(torch, links32, psi_full, parity, nrhs=1, blocked=False, **kw):
    """Three applies back to back (PDL on), distinct sources; returns [(seeds, out numpy)].
    blocked: the sources are converted to the site-blocked layout on the device first, the three
    applies run dslash_apply_multi_blocked back to back, and the outputs are converted back."""
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    fat, lng = links32
    res = []
    with Dslash(DIMS, parity_mask=parity, **kw) as D:
        D.load_links(fat, lng)
        srcs, outs, seeds = [], [], []
        for s in SEEDS:
            ss = [s + 10 * r for r in range(nrhs)]
            vs = [torch.from_numpy(fieldgen.vector_cb(DIMS, q, 1 - parity)).to(D.dtype) for q in ss]
            srcs.append((vs[0] if nrhs == 1 else torch.stack(vs)).contiguous().cuda())
            outs.append(torch.empty_like(srcs[-1]))
            seeds.append(ss)
        if blocked:
            bsrcs = [D.to_blocked(torch.empty_like(v), v) for v in srcs]
            bouts = [torch.empty_like(v) for v in srcs]
            for src, out in zip(bsrcs, bouts):
                D.apply_multi_blocked(out, src, parity)
            for out, bout in zip(outs, bouts):
                D.from_blocked(out, bout)
        else:
            for src, out in zip(srcs, outs):
                if nrhs == 1:
                    D.apply(out, src, parity)
                else:
                    D.apply_multi(out, src, parity)
        torch.cuda.synchronize()
        for ss, out in zip(seeds, outs):
            res.append((ss, out.cpu().numpy()))
    return res


@pytest.mark.parametrize("precision,recon", [("f64", 18), ("f32", 18), ("mixed", 18),
                                             ("f64", 12), ("f32", 12), ("mixed", 12),
                                             ("f64", 9), ("f32", 9), ("mixed", 9)])
def test_32_precisions_and_recon(torch_cuda, links32, psi_full, precision, recon):
    """fp32 / mixed (§8(f)-1), recon-12 and recon-9 in every precision (§8(f)-2)."""
    fat, lng = links32
    parity = 0
    kernel = _bench_kernel(recon, 1, precision)
    for ss, got in _run_chain(torch_cuda, links32, psi_full, parity, precision=precision, recon=recon,
                              kernel=kernel):
        _check(got, fat, lng, psi_full(ss[0]), parity, precision, (precision, recon, ss))


@pytest.mark.parametrize("nrhs", [2, 4, 8])
@pytest.mark.parametrize("precision", ["f64", "f32"])
def test_32_multi_rhs_every_rhs(torch_cuda, links32, psi_full, nrhs, precision):
    """§8(f)-4 at the bench size: every right-hand side of every apply against the oracle."""
    fat, lng = links32
    parity = 1
    for ss, got in _run_chain(torch_cuda, links32, psi_full, parity, nrhs=nrhs, precision=precision,
                              kernel=_bench_kernel(18, nrhs)):
        for r, s in enumerate(ss):
            _check(got[r], fat, lng, psi_full(s), parity, precision, (nrhs, r, s))


@pytest.mark.parametrize("precision", ["f64", "f32", "mixed"])
def test_32_multi_rhs_blocked_every_rhs(torch_cuda, links32, psi_full, precision):
    """The site-blocked 8-RHS layout (dslash_apply_multi_blocked) at the bench size, as bench.py
    --layout blocked runs it: every right-hand side of every apply against the oracle."""
    fat, lng = links32
    parity = 1
    for ss, got in _run_chain(torch_cuda, links32, psi_full, parity, nrhs=8, blocked=True, precision=precision,
                              kernel="site"):
        for r, s in enumerate(ss):
            _check(got[r], fat, lng, psi_full(s), parity, precision, ("blocked", r, s))


@pytest.mark.parametrize("kernel,nrhs", [("dir2", 1), ("site", 1), ("site", 8)])
def test_32_stage(torch_cuda, links32, psi_full, kernel, nrhs):
    """The neighbour-staged kernel (DSLASH_OPT_STAGE) at the bench size."""
    fat, lng = links32
    parity = 0
    for ss, got in _run_chain(torch_cuda, links32, psi_full, parity, nrhs=nrhs, kernel=kernel, stage=True):
        for r, s in enumerate(ss):
            _check(got if nrhs == 1 else got[r], fat, lng, psi_full(s), parity, "f64", (kernel, nrhs, r))


@pytest.mark.parametrize("mask", [0x8, 0xC])
@pytest.mark.parametrize("precision", ["f64", "f32", "mixed"])
@pytest.mark.parametrize("overlap", ["sites", "dirs"])
def test_32_self_halo_paths(torch_cuda, links32, psi_full, mask, precision, overlap):
    """The weak-scaling per-GPU launch configuration (32^3 x 32 local, t halo; plus z) through
    the self-halo: interior + boundary kernels on two streams (split by sites, the default) or
    the local + ghost passes (split by direction), every precision, against the oracle; the split
    by sites is also bitwise the unpartitioned apply."""
    fat, lng = links32
    parity = 1
    halo = _run_chain(torch_cuda, links32, psi_full, parity, precision=precision, force_halo=mask, overlap=overlap)
    for ss, got in halo:
        _check(got, fat, lng, psi_full(ss[0]), parity, precision, (mask, precision, overlap, ss))
    if overlap == "sites":
        plain = _run_chain(torch_cuda, links32, psi_full, parity, precision=precision)
        for (_, a), (_, b) in zip(halo, plain):
            assert np.array_equal(a, b)


def test_32_nccl_self_halo(torch_cuda, links32, psi_full):
    """The NCCL transport (one-rank communicator, faces through ncclSend/ncclRecv to this rank:
    the P = 2 message pattern) at the bench size, t + z halo."""
    fat, lng = links32
    parity = 0
    for ss, got in _run_chain(torch_cuda, links32, psi_full, parity, force_halo=0xC, self_nccl=True):
        _check(got, fat, lng, psi_full(ss[0]), parity, "f64", ("nccl", ss))


# ---------------------------------------------------------------------------- 48^4 and its per-GPU volumes
DIMS48 = (48, 48, 48, 48)


@pytest.fixture(scope="module")
def links48():
    return fieldgen.workload_links(DIMS48)


def _check48(torch, fat, lng, dims, parity, precision, what, nsample=2048, **kw):
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    with Dslash(dims, parity_mask=parity, precision=precision, **kw) as D:
        D.load_links(fat, lng)
        src = torch.from_numpy(fieldgen.vector_cb(dims, 401, 1 - parity)).to(D.dtype).cuda()
        out = D.empty_vector()
        for _ in range(2):                              # back to back, PDL
            D.apply(out, src, parity)
        torch.cuda.synchronize()
        got = out.cpu().numpy()
    lex = oracle.lex_sites_of_parity(dims, parity)
    pick = np.unique(np.concatenate([[0, 1, lex.size - 2, lex.size - 1],
                                     np.random.default_rng(48).choice(lex.size, nsample, replace=False)]))
    ref = oracle.dslash_sites(fat, lng, fieldgen.vector(dims, 401), lex[pick])
    err = oracle.normwise_error(got[:, pick].T.astype(np.complex128), ref)
    assert err <= TOL[precision], (what, err)
    if precision != "f64":
        assert err > 1e-12, (what, err)


@pytest.mark.parametrize("precision,recon", [("f32", 18), ("mixed", 18), ("f64", 12), ("f64", 9), ("f32", 12)])
def test_48_precisions_and_recon(torch_cuda, links48, precision, recon):
    """The strong-scaling lattice (BASELINE.json configs[3]) on one GPU, reduced precision and
    long-link compression, sampled against the oracle."""
    fat, lng = links48
    _check48(torch_cuda, fat, lng, DIMS48, 1, precision, (precision, recon), recon=recon,
             kernel="site" if recon == 9 else "dir2")


@pytest.mark.parametrize("dims,mask,overlap", [((48, 48, 48, 6), 0x8, "sites"), ((48, 48, 48, 6), 0x8, "dirs"),
                                               ((48, 48, 24, 12), 0xC, "sites"), ((48, 48, 48, 12), 0x8, "sites")])
@pytest.mark.parametrize("precision", ["f64", "mixed"])
def test_48_per_gpu_volumes_self_halo(torch_cuda, dims, mask, overlap, precision):
    """The per-GPU volumes of 48^4 on 8 GPUs (t8: 48^3 x 6, no interior site; z2 x t4: 48^2 x 24 x
    12, choose_grid's pick) and on 4 (48^3 x 12), through the self-halo in the bench's launch
    configuration, sampled against the oracle of that (periodic) lattice."""
    fat, lng = fieldgen.workload_links(dims)
    _check48(torch_cuda, fat, lng, dims, 0, precision, (dims, mask, overlap), force_halo=mask, overlap=overlap)
