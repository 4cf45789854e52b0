"""GPU: the producer push (DSLASH_OPT_PUSH).  An apply_push stores the depth-3 faces of its OUTPUT
straight into the neighbours' ghost faces from the stencil kernel's epilogue (peer memory), so
the next apply, whose source that output is, exchanges no bytes: the compute step and the
exchange that follows it in D_{p,1-p} D_{1-p,p} (the normal operator, CG) are one kernel.

Every result must be BITWISE equal to the same chain without the push: the pushed face values
are the very bits the kernel stores into `out`, and the consumer's arithmetic is unchanged.
One GPU: self-halo (neighbour = self, the push lands in this handle's own second ghost bank)
and several processes on the one device (CUDA IPC-mapped banks, stream-memory epoch flags)."""
import os
import socket

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


def _chain(D, torch, x, parity, steps, push):
    """steps x (y = D x on `parity`, x = D y on 1 - parity); returns every intermediate (CPU)."""
    outs = []
    for _ in range(steps):
        y = D.empty_vector()
        (D.apply_push if push else D.apply)(y, x, parity)
        z = D.empty_vector()
        D.apply(z, y, 1 - parity)
        outs += [y, z]
        x = z
    torch.cuda.synchronize()
    return [o.cpu() for o in outs]


@pytest.mark.parametrize("mask", [0x8, 0x4, 0xC])
@pytest.mark.parametrize("overlap", ["sites", "none", "dirs"])
def test_push_chain_self_halo_bitwise(torch_cuda, mask, overlap):
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 8, 8, 12)
    fat, lng = fieldgen.workload_links(dims)
    x = torch.from_numpy(fieldgen.vector_cb(dims, 81, 1)).cuda()
    res = {}
    for push in (False, True):
        with Dslash(dims, force_halo=mask, transport="p2p", push=push, overlap=overlap) as D:
            D.load_links(fat, lng)
            res[push] = _chain(D, torch, x, 0, 3, push)
    for a, b in zip(res[False], res[True]):
        assert torch.equal(a, b)
    # and the first link of the chain is the operator itself
    ref = oracle.full_to_cb(oracle.dslash(fat, lng, oracle.cb_to_full(x.cpu().numpy(), dims, 1), 0), 0)
    assert oracle.normwise_error(res[True][0].numpy(), ref) <= 1e-12


@pytest.mark.parametrize("kw", [{"kernel": "site"}, {"kernel": "dir4", "recon": 12}, {"precision": "mixed"},
                                {"precision": "f32"}, {"stage": True}, {"kernel": "dir2", "block": 128}])
def test_push_chain_variants_bitwise(torch_cuda, kw):
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 8, 8, 16)
    fat, lng = fieldgen.workload_links(dims)
    x = torch.from_numpy(fieldgen.vector_cb(dims, 82, 0))
    res = {}
    for push in (False, True):
        with Dslash(dims, force_halo=0xC, transport="p2p", push=push, **kw) as D:
            D.load_links(fat, lng)
            res[push] = _chain(D, torch, x.to(D.dtype).cuda(), 1, 2, push)
    for a, b in zip(res[False], res[True]):
        assert torch.equal(a, b)


def test_push_local_extent_4(torch_cuda):
    """L_t = 4: the middle slices are both bottom and top slices, pushed to both neighbours."""
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 8, 4, 4)
    fat, lng = fieldgen.workload_links(dims)
    x = torch.from_numpy(fieldgen.vector_cb(dims, 83, 0)).cuda()
    res = {}
    for push in (False, True):
        with Dslash(dims, force_halo=0xC, transport="p2p", push=push) as D:
            D.load_links(fat, lng)
            res[push] = _chain(D, torch, x, 1, 2, push)
    with Dslash(dims) as D:
        D.load_links(fat, lng)
        ref = _chain(D, torch, x, 1, 2, False)
    for a, b, c in zip(res[False], res[True], ref):
        assert torch.equal(a, b) and torch.equal(b, c)


def test_push_normal_and_cg_bitwise(torch_cuda):
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 8, 8, 12)
    fat, lng = fieldgen.workload_links(dims)
    b = torch.from_numpy(fieldgen.vector_cb(dims, 84, 0)).cuda()
    m = 0.3
    sols = []
    # unpartitioned; self-halo P2P split by sites without / with the push; split by direction
    # (boundary sites sum in another order: bitwise only against itself) without / with the push
    for kw in ({}, {"force_halo": 0xC, "transport": "p2p"}, {"force_halo": 0xC, "transport": "p2p", "push": True},
               {"force_halo": 0x8, "transport": "p2p", "overlap": "dirs"},
               {"force_halo": 0x8, "transport": "p2p", "push": True, "overlap": "dirs"}):
        with Dslash(dims, **kw) as D:
            D.load_links(fat, lng)
            q = D.normal_apply(D.empty_vector(), b, 0, m)
            q2 = D.normal_apply(D.empty_vector(), q, 0, m)
            x = D.empty_vector()
            ok, it, res = D.cg(x, b, 0, m, rel_tol=1e-10)
            assert ok and res <= 2e-10
            xm = D.empty_vector()
            okm, itm, outer, resm = D.cg_mixed(xm, b, 0, m, rel_tol=1e-10, inner_tol=1e-3)
            assert okm and resm <= 1e-10
            torch.cuda.synchronize()
            sols.append((q.cpu(), q2.cpu(), x.cpu(), it, xm.cpu(), itm, outer))
    for j, k in ((0, 1), (0, 2), (3, 4)):
        a, c = sols[j], sols[k]
        for i in (0, 1, 2, 4):
            assert torch.equal(a[i], c[i]), (k, i)
        assert a[3] == c[3] and a[5:] == c[5:], k
    assert oracle.normwise_error(sols[4][1].numpy(), sols[0][1].numpy()) <= 1e-13
    ref = oracle.full_to_cb(ocg.normal_apply(fat, lng, oracle.cb_to_full(b.cpu().numpy(), dims, 0), 0, m), 0)
    assert oracle.normwise_error(sols[2][0].numpy(), ref) <= 1e-12


def test_push_errors(torch_cuda):
    torch = torch_cuda
    from paper_conf_sc_dufekgaad024_b200 import Dslash, _abi
    dims = (8, 8, 8, 12)
    fat, lng = fieldgen.workload_links(dims)
    x = torch.from_numpy(fieldgen.vector_cb(dims, 85, 1)).cuda()
    with pytest.raises(_abi.DslashError, match="UNSUPPORTED"):   # push needs peer-mapped ghosts
        Dslash(dims, force_halo=0xC, push=True).close()
    with Dslash(dims, force_halo=0xC, transport="p2p") as D:      # apply_push without the option
        D.load_links(fat, lng)
        with pytest.raises(_abi.DslashError, match="STATE"):
            D.apply_push(D.empty_vector(), x, 0)
    with Dslash(dims, force_halo=0xC, transport="p2p", push=True) as D:
        D.load_links(fat, lng)
        with pytest.raises(_abi.DslashError, match="STATE"):     # option after load_links
            _abi.dslash_set_option(D.h, _abi.DSLASH_OPT_PUSH, 0)
        y = D.apply_push(D.empty_vector(), x, 0)
        with pytest.raises(_abi.DslashError, match="STATE"):     # the next source must be y
            D.apply(D.empty_vector(), x, 1)
    with Dslash(dims, transport="p2p", push=True) as D:            # no halo: apply_push == apply
        D.load_links(fat, lng)
        y = D.apply_push(D.empty_vector(), x, 0)
        z = D.apply(D.empty_vector(), x, 0)
        torch.cuda.synchronize()
        assert torch.equal(y, z)


# ------------------------------------------------------------------ several processes, one GPU
def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _rank_main(rank, world, port, gdims, grid, kw, q):
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_sc_dufekgaad024_b200 import Dslash
        D = Dslash(gdims, grid, rank=rank, world_size=world, transport="p2p", push=True, **kw)
        o, e = D.origin, D.local_dims
        fat, lng = fieldgen.workload_links(gdims, origin=o, extent=e)
        D.load_links(fat, lng)
        x = torch.from_numpy(fieldgen.vector_cb(gdims, 86, 1, origin=o, extent=e)).cuda()
        chain = _chain(D, torch, x, 0, 3, True)
        b = torch.from_numpy(fieldgen.vector_cb(gdims, 87, 0, origin=o, extent=e)).cuda()
        nq = D.normal_apply(D.empty_vector(), b, 0, 0.3)
        nq2 = D.normal_apply(D.empty_vector(), nq, 0, 0.3)
        torch.cuda.synchronize()
        q.put((rank, tuple(o), tuple(e), [c.numpy() for c in chain] + [nq.cpu().numpy(), nq2.cpu().numpy()],
               None))
        D.close()
    except Exception as exc:  # pragma: no cover - reported to the parent
        q.put((rank, None, None, repr(exc), None))
    finally:
        dist.destroy_process_group()


def _gather(results, gdims, k):
    lx, ly, lz, lt = gdims
    full = np.zeros((3, lt, lz, ly, lx // 2), np.complex128)
    for rank, o, e, outs, _ in results:
        assert o is not None, outs
        full[:, o[3]:o[3] + e[3], o[2]:o[2] + e[2]] = outs[k].reshape(3, e[3], e[2], e[1], e[0] // 2)
    return full.reshape(3, -1)


@pytest.mark.parametrize("gdims,grid,kw", [((8, 8, 8, 16), (1, 1, 1, 2), {}),
                                           ((8, 8, 16, 8), (1, 1, 2, 1), {}),
                                           ((8, 8, 8, 8), (1, 1, 2, 2), {}),
                                           ((8, 8, 8, 24), (1, 1, 1, 3), {"overlap": "none"}),
                                           ((8, 8, 8, 16), (1, 1, 1, 2), {"overlap": "dirs", "kernel": "site"})])
def test_push_multirank_bitwise(torch_cuda, gdims, grid, kw):
    torch = torch_cuda
    import torch.multiprocessing as mp
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    world = grid[2] * grid[3]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rank_main, args=(r, world, port, gdims, grid, kw, q)) for r in range(world)]
    for p in procs:
        p.start()
    results = [q.get(timeout=300) for _ in procs]
    for p in procs:
        p.join(timeout=120)
    fat, lng = fieldgen.workload_links(gdims)
    with Dslash(gdims, **{k: v for k, v in kw.items() if k != "overlap"}) as D:
        D.load_links(fat, lng)
        x = torch.from_numpy(fieldgen.vector_cb(gdims, 86, 1)).cuda()
        ref = _chain(D, torch, x, 0, 3, False)
        b = torch.from_numpy(fieldgen.vector_cb(gdims, 87, 0)).cuda()
        nq = D.normal_apply(D.empty_vector(), b, 0, 0.3)
        nq2 = D.normal_apply(D.empty_vector(), nq, 0, 0.3).cpu()
        nq = nq.cpu()
    for k, r in enumerate(ref + [nq, nq2]):
        got = _gather(results, gdims, k)
        if kw.get("overlap") == "dirs":   # boundary sites sum their hops in another order
            assert oracle.normwise_error(got, r.numpy()) <= 1e-13, k
        else:
            assert np.array_equal(got, r.numpy()), k
