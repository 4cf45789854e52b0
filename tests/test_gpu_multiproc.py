"""Real multi-rank runs on ONE GPU: several processes, each a rank with its own library handle,
exchanging depth-3 halos through the P2P transport (CUDA IPC-mapped ghost buffers, copy
engines, stream-memory epoch flags).  NCCL cannot put two ranks on one device, so this is how
the multi-rank data path (plan, ghost addressing, link halo, epoch protocol, interior and
boundary launches) is exercised end to end on a single B200.

The gathered N-rank result must equal the 1-rank result BITWISE (same per-site device function,
SURVEY §8(c) P11) and match the oracle."""
import os
import socket

import numpy as np
import pytest

import fieldgen
import oracle

pytestmark = pytest.mark.gpu

SEED = 3


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _rank_main(rank, world, port, gdims, grid, kw, parity, napply, nrhs, q):
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_sc_dufekgaad024_b200 import Dslash
        D = Dslash(gdims, grid, rank=rank, world_size=world, transport="p2p", **kw)
        o, e = D.origin, D.local_dims
        fat, lng = fieldgen.workload_links(gdims, origin=o, extent=e)
        D.load_links(fat, lng)
        if nrhs == 1:
            src = torch.from_numpy(fieldgen.vector_cb(gdims, SEED, 1 - parity, origin=o, extent=e)).cuda()
            out = D.empty_vector()
            for _ in range(napply):                  # several epochs through the same ghosts
                D.apply(out, src, parity)
        else:
            src = torch.stack([torch.from_numpy(fieldgen.vector_cb(gdims, SEED + r, 1 - parity, origin=o, extent=e))
                               for r in range(nrhs)]).cuda()
            out = torch.empty_like(src)
            for _ in range(napply):
                D.apply_multi(out, src, parity)
        torch.cuda.synchronize()
        q.put((rank, tuple(o), tuple(e), out.cpu().numpy()))
        D.close()
    except Exception as exc:  # pragma: no cover - reported to the parent
        q.put((rank, None, None, repr(exc)))
    finally:
        dist.destroy_process_group()


def _gather(results, gdims, nrhs):
    lx, ly, lz, lt = gdims
    full = np.zeros((nrhs, 3, lt, lz, ly, lx // 2), np.complex128)
    for rank, o, e, out in results:
        assert o is not None, out
        v = out.reshape(nrhs, 3, e[3], e[2], e[1], e[0] // 2)
        full[:, :, o[3]:o[3] + e[3], o[2]:o[2] + e[2]] = v
    return full.reshape(nrhs, 3, -1)


def _run(world, gdims, grid, kw=None, parity=0, napply=3, nrhs=1):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rank_main, args=(r, world, port, gdims, grid, kw or {}, parity, napply, nrhs, q))
             for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in procs]
    for p in procs:
        p.join(timeout=120)
    return _gather(res, gdims, nrhs)


def _single(gdims, kw, parity, nrhs=1):
    import torch
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    fat, lng = fieldgen.workload_links(gdims)
    with Dslash(gdims, **{k: v for k, v in (kw or {}).items() if k != "push"}) as D:   # push: a P2P option
        D.load_links(fat, lng)
        outs = [D(torch.from_numpy(fieldgen.vector_cb(gdims, SEED + r, 1 - parity)).cuda(), parity).cpu().numpy()
                for r in range(nrhs)]
    return np.stack(outs)


@pytest.mark.parametrize("gdims,grid", [((8, 8, 8, 16), (1, 1, 1, 2)), ((8, 8, 16, 8), (1, 1, 2, 1)),
                                        ((8, 8, 8, 8), (1, 1, 2, 2)), ((8, 8, 8, 24), (1, 1, 1, 3))])
@pytest.mark.parametrize("overlap", [True, False])
def test_multirank_p2p_bitwise(gdims, grid, overlap):   # split by sites, or one launch after the exchange
    world = grid[2] * grid[3]
    kw = {"overlap": overlap}
    for parity in (0, 1):
        got = _run(world, gdims, grid, kw, parity)
        ref = _single(gdims, kw, parity)
        assert np.array_equal(got, ref)
        fat, lng = fieldgen.workload_links(gdims)
        o = oracle.full_to_cb(oracle.dslash(fat, lng, fieldgen.vector(gdims, SEED), parity), parity)
        assert oracle.normwise_error(got[0], o) <= 1e-12


@pytest.mark.parametrize("kw", [{"kernel": "site"}, {"kernel": "dir4", "recon": 12}, {"precision": "mixed"},
                                {"kernel": "site", "recon": 9}, {"recon": 9, "push": True}])
def test_multirank_p2p_variants(kw):
    gdims, grid = (8, 8, 8, 16), (1, 1, 1, 2)
    got = _run(2, gdims, grid, kw, 1)
    assert np.array_equal(got, _single(gdims, kw, 1))


def test_multirank_p2p_multi_rhs():
    gdims, grid = (8, 8, 8, 16), (1, 1, 1, 2)
    got = _run(2, gdims, grid, {}, 0, napply=2, nrhs=3)
    assert np.array_equal(got, _single(gdims, {}, 0, nrhs=3))


def test_multirank_p2p_32_local():
    """The weak-scaling per-GPU configuration: 32^3 x 32 local, t-partitioned over 2 ranks."""
    gdims, grid = (32, 32, 32, 64), (1, 1, 1, 2)
    got = _run(2, gdims, grid, {}, 0, napply=2)
    assert np.array_equal(got, _single(gdims, {}, 0))


@pytest.mark.parametrize("gdims,grid", [((8, 8, 8, 16), (1, 1, 1, 2)), ((8, 8, 16, 8), (1, 1, 2, 1)),
                                        ((8, 8, 8, 8), (1, 1, 2, 2)), ((8, 8, 8, 18), (1, 1, 1, 3))])
def test_multirank_p2p_overlap_dirs(gdims, grid):
    """Split-by-direction overlap across real ranks (local pass during the exchange, ghost pass
    after): boundary sites sum in another order, so the gathered result matches the 1-rank apply
    and the oracle within tolerance (18 = 3 x local extent 6: no interior site at all)."""
    world = grid[2] * grid[3]
    for kw in ({"overlap": "dirs"}, {"overlap": "dirs", "kernel": "site", "precision": "mixed"}):
        got = _run(world, gdims, grid, kw, 1)
        ref = _single(gdims, {k: v for k, v in kw.items() if k != "overlap"}, 1)
        tol = 1e-14 if kw.get("precision", "f64") == "f64" else 1e-6
        assert oracle.normwise_error(got[0], ref[0]) <= tol
        fat, lng = fieldgen.workload_links(gdims)
        o = oracle.full_to_cb(oracle.dslash(fat, lng, fieldgen.vector(gdims, SEED), 1), 1)
        assert oracle.normwise_error(got[0], o) <= (1e-12 if tol == 1e-14 else 1e-5)
