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
CG_MASS = 0.1


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
    kw = dict(kw)
    mode = kw.pop("_mode", "apply")              # "apply", "cg" or "cg_mixed"
    distinct = kw.pop("_distinct", False)        # one GPU per rank (needs >= world GPUs)
    transport = kw.pop("transport", "p2p")
    dev = rank if distinct else 0
    torch.cuda.set_device(dev)
    if transport == "nccl":
        dist.init_process_group("nccl", rank=rank, world_size=world, device_id=torch.device("cuda", dev))
    else:
        dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_sc_dufekgaad024_b200 import Dslash
        D = Dslash(gdims, grid, rank=rank, world_size=world, transport=transport, **kw)
        o, e = D.origin, D.local_dims
        fat, lng = fieldgen.workload_links(gdims, origin=o, extent=e)
        D.load_links(fat, lng)
        if mode in ("cg", "cg_mixed"):
            b = torch.from_numpy(fieldgen.vector_cb(gdims, SEED, parity, origin=o, extent=e)).cuda()
            x = D.empty_vector()
            if mode == "cg":
                ok, it, res = D.cg(x, b, parity, CG_MASS, rel_tol=1e-10, max_iter=2000)
                info = (ok, it, res)
            else:
                ok, it, outer, res = D.cg_mixed(x, b, parity, CG_MASS, rel_tol=1e-10, inner_tol=1e-3, max_iter=4000)
                info = (ok, it, outer, res)
            torch.cuda.synchronize()
            q.put((rank, tuple(o), tuple(e), x.cpu().numpy(), info))
            D.close()
            return
        if mode == "blocked":                    # site-blocked multi-RHS layout
            src = torch.stack([torch.from_numpy(fieldgen.vector_cb(gdims, SEED + r, 1 - parity, origin=o, extent=e))
                               for r in range(nrhs)]).to(D.dtype).contiguous().cuda()
            bsrc = D.to_blocked(torch.empty_like(src), src)
            bout = torch.empty_like(src)
            for _ in range(napply):
                D.apply_multi_blocked(bout, bsrc, parity)
            out = D.from_blocked(torch.empty_like(src), bout)
            torch.cuda.synchronize()
            q.put((rank, tuple(o), tuple(e), out.cpu().numpy(), None))
            D.close()
            return
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
        q.put((rank, tuple(o), tuple(e), out.cpu().numpy(), None))
        D.close()
    except Exception as exc:  # pragma: no cover - reported to the parent
        q.put((rank, None, None, repr(exc), None))
    finally:
        dist.destroy_process_group()


def _gather(results, gdims, nrhs):
    lx, ly, lz, lt = gdims
    full = np.zeros((nrhs, 3, lt, lz, ly, lx // 2), np.complex128)
    for rank, o, e, out, _ in results:
        assert o is not None, out
        v = out.reshape(nrhs, 3, e[3], e[2], e[1], e[0] // 2)
        full[:, :, o[3]:o[3] + e[3], o[2]:o[2] + e[2]] = v
    return full.reshape(nrhs, 3, -1)


def _run(world, gdims, grid, kw=None, parity=0, napply=3, nrhs=1, infos=None):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rank_main, args=(r, world, port, gdims, grid, kw or {}, parity, napply, nrhs, q))
             for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=600) for _ in procs]
    for p in procs:
        p.join(timeout=120)
    if infos is not None:
        infos.extend(r[4] for r in sorted(res, key=lambda r: r[0]))
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


@pytest.mark.parametrize("gdims,grid", [((8, 8, 8, 16), (1, 1, 1, 2)), ((8, 8, 16, 8), (1, 1, 2, 1)),
                                        ((8, 8, 8, 8), (1, 1, 2, 2))])
@pytest.mark.parametrize("kw", [{"kernel": "site"}, {"precision": "mixed", "kernel": "site"}, {"overlap": False}])
def test_multirank_p2p_blocked(gdims, grid, kw):
    """The site-blocked multi-RHS layout across P2P ranks (faces = whole 16-site blocks): the
    gathered result equals the 1-rank planar apply bitwise."""
    world = grid[2] * grid[3]
    got = _run(world, gdims, grid, dict(kw, _mode="blocked"), 0, napply=2, nrhs=8)
    single_kw = {k: v for k, v in kw.items() if k != "overlap"}
    ref = _single(gdims, single_kw, 0, nrhs=8)
    assert np.array_equal(got, ref)


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



def _single_cg(gdims, parity, mixed=False, kw=None):
    import torch
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    fat, lng = fieldgen.workload_links(gdims)
    with Dslash(gdims, **(kw or {})) as D:
        D.load_links(fat, lng)
        b = torch.from_numpy(fieldgen.vector_cb(gdims, SEED, parity)).cuda()
        x = D.empty_vector()
        if mixed:
            info = D.cg_mixed(x, b, parity, CG_MASS, rel_tol=1e-10, inner_tol=1e-3, max_iter=4000)
        else:
            info = D.cg(x, b, parity, CG_MASS, rel_tol=1e-10, max_iter=2000)
        torch.cuda.synchronize()
        return x.cpu().numpy()[None], info


@pytest.mark.parametrize("gdims,grid", [((8, 8, 8, 16), (1, 1, 1, 2)), ((8, 8, 16, 8), (1, 1, 2, 1)),
                                        ((8, 8, 8, 8), (1, 1, 2, 2)), ((8, 8, 8, 24), (1, 1, 1, 3))])
@pytest.mark.parametrize("mixed", [False, True])
def test_multirank_p2p_cg_bitwise(gdims, grid, mixed):
    """§8(f)-3 across ranks without NCCL (several ranks on one GPU): the dot products' per-rank
    double-double sums meet through the ranks' IPC-mapped control blocks and every rank adds them
    in rank order (hisq_p2p_gather).  The solve is decomposition-independent: the gathered x,
    the iteration count and the true residual equal the 1-rank solve's BITWISE (plain CG and
    mixed-precision CG), and x solves the system like the oracle CG's."""
    world = grid[2] * grid[3]
    parity = 0
    infos = []
    got = _run(world, gdims, grid, {"_mode": "cg_mixed" if mixed else "cg"}, parity, infos=infos)
    ref, ref_info = _single_cg(gdims, parity, mixed)
    assert all(i[0] for i in infos), infos
    assert all(i == infos[0] for i in infos), infos                  # every rank: same counts and residual
    assert tuple(infos[0]) == tuple(ref_info), (infos[0], ref_info)
    assert np.array_equal(got, ref)
    from oracle import cg as ocg
    fat, lng = fieldgen.workload_links(gdims)
    b_full = oracle.cb_to_full(fieldgen.vector_cb(gdims, SEED, parity), gdims, parity)
    x_ref, _ = ocg.cg(fat, lng, b_full, parity, CG_MASS, rel_tol=1e-10, max_iter=2000)
    assert oracle.normwise_error(got[0], oracle.full_to_cb(x_ref, parity)) <= 1e-8


@pytest.mark.parametrize("kw", [{"recon": 9, "kernel": "site"}, {"recon": 12}, {"overlap": "dirs"}])
@pytest.mark.parametrize("mixed", [False, True])
def test_multirank_p2p_cg_variants(kw, mixed):
    """CG and mixed CG over 2 colocated ranks with compressed long links or the split-by-direction
    overlap: the same iterates as the 1-rank solve (recon-9 / recon-12 bitwise; the split by
    direction sums boundary sites in another order, so its solve is compared with the oracle)."""
    gdims, grid = (8, 8, 8, 16), (1, 1, 1, 2)
    infos = []
    got = _run(2, gdims, grid, {"_mode": "cg_mixed" if mixed else "cg", **kw}, 0, infos=infos)
    assert all(i[0] for i in infos), infos
    if kw.get("overlap") != "dirs":
        ref, ref_info = _single_cg(gdims, 0, mixed, kw)
        assert tuple(infos[0]) == tuple(ref_info), (infos[0], ref_info)
        assert np.array_equal(got, ref)
    from oracle import cg as ocg
    fat, lng = fieldgen.workload_links(gdims)
    b_full = oracle.cb_to_full(fieldgen.vector_cb(gdims, SEED, 0), gdims, 0)
    x_ref, _ = ocg.cg(fat, lng, b_full, 0, CG_MASS, rel_tol=1e-10, max_iter=2000)
    assert oracle.normwise_error(got[0], oracle.full_to_cb(x_ref, 0)) <= 1e-8


def test_multirank_p2p_cg_push():
    """CG with the producer push across 2 ranks (push in every exchange, P2P reductions)."""
    gdims, grid = (8, 8, 8, 16), (1, 1, 1, 2)
    infos = []
    got = _run(2, gdims, grid, {"_mode": "cg", "push": True}, 1, infos=infos)
    ref, ref_info = _single_cg(gdims, 1)
    assert tuple(infos[0]) == tuple(ref_info)
    assert np.array_equal(got, ref)


# ---------------------------------------------------------------------------- distinct GPUs
# The same data paths across DISTINCT devices (NVLink peers on a B200 node): NCCL send/recv
# between two GPUs, P2P copy-engine puts into another GPU's IPC-mapped ghosts, and the producer
# push storing into a peer GPU's memory from the kernel epilogue.  Collected always, run when at
# least two GPUs are visible (the driver's one-GPU boxes skip them).

def _ngpu():
    import torch
    return torch.cuda.device_count()


@pytest.mark.parametrize("transport,extra", [("nccl", {}), ("p2p", {}), ("p2p", {"push": True}),
                                             ("nccl", {"overlap": "dirs"}), ("nccl", {"precision": "mixed"})])
@pytest.mark.parametrize("gdims,grid", [((8, 8, 8, 16), (1, 1, 1, 2)), ((8, 8, 16, 8), (1, 1, 2, 1)),
                                        ((16, 16, 16, 16), (1, 1, 2, 2))])
def test_distinct_gpus_apply(transport, extra, gdims, grid):
    world = grid[2] * grid[3]
    if _ngpu() < world:
        pytest.skip(f"needs {world} GPUs, {_ngpu()} visible")
    kw = {"_distinct": True, "transport": transport, **extra}
    parity = 1
    got = _run(world, gdims, grid, kw, parity)
    single_kw = {k: v for k, v in extra.items() if k not in ("push", "overlap")}
    ref = _single(gdims, single_kw, parity)
    prec = extra.get("precision", "f64")
    if extra.get("overlap") == "dirs":
        assert oracle.normwise_error(got[0], ref[0]) <= (1e-14 if prec == "f64" else 1e-6)
    else:
        assert np.array_equal(got, ref)
    fat, lng = fieldgen.workload_links(gdims)
    o = oracle.full_to_cb(oracle.dslash(fat, lng, fieldgen.vector(gdims, SEED), parity), parity)
    assert oracle.normwise_error(got[0], o) <= (1e-12 if prec == "f64" else 1e-5)


@pytest.mark.parametrize("transport,extra", [("nccl", {}), ("p2p", {}), ("p2p", {"push": True})])
def test_distinct_gpus_cg(transport, extra):
    gdims, grid = (8, 8, 8, 16), (1, 1, 1, 2)
    if _ngpu() < 2:
        pytest.skip(f"needs 2 GPUs, {_ngpu()} visible")
    infos = []
    got = _run(2, gdims, grid, {"_mode": "cg", "_distinct": True, "transport": transport, **extra}, 0, infos=infos)
    ref, ref_info = _single_cg(gdims, 0)
    assert tuple(infos[0]) == tuple(ref_info)
    assert np.array_equal(got, ref)


def test_distinct_gpus_multi_rhs_nccl():
    gdims, grid = (8, 8, 8, 16), (1, 1, 1, 2)
    if _ngpu() < 2:
        pytest.skip(f"needs 2 GPUs, {_ngpu()} visible")
    got = _run(2, gdims, grid, {"_distinct": True, "transport": "nccl"}, 0, napply=2, nrhs=3)
    assert np.array_equal(got, _single(gdims, {}, 0, nrhs=3))


@pytest.mark.parametrize("transport", ["nccl", "p2p"])
@pytest.mark.parametrize("gdims,grid", [((8, 8, 8, 16), (1, 1, 1, 2)), ((8, 8, 16, 8), (1, 1, 2, 1))])
def test_distinct_gpus_blocked(transport, gdims, grid):
    """The site-blocked 8-RHS layout across two GPUs (faces as whole 16-site blocks over NCCL or
    NVLink peer copies): bitwise the 1-rank planar apply."""
    if _ngpu() < 2:
        pytest.skip(f"needs 2 GPUs, {_ngpu()} visible")
    got = _run(2, gdims, grid, {"_distinct": True, "transport": transport, "kernel": "site", "_mode": "blocked"}, 0,
               napply=2, nrhs=8)
    assert np.array_equal(got, _single(gdims, {"kernel": "site"}, 0, nrhs=8))


def test_two_handles_two_devices_one_process():
    """Two handles in one process on different GPUs, used interleaved while torch's current device
    is the other one: every entry point runs on its handle's device (DeviceGuard) and leaves the
    caller's current device as it was."""
    import torch
    if _ngpu() < 2:
        pytest.skip(f"needs 2 GPUs, {_ngpu()} visible")
    from paper_conf_sc_dufekgaad024_b200 import Dslash
    dims = (8, 8, 8, 16)
    fat, lng = fieldgen.workload_links(dims)
    handles = []
    for dev in (0, 1):
        torch.cuda.set_device(dev)
        D = Dslash(dims)
        D.load_links(fat, lng)
        handles.append(D)
    src = [torch.from_numpy(fieldgen.vector_cb(dims, SEED, 1)).to(f"cuda:{d}") for d in (0, 1)]
    outs = []
    for it in range(3):
        for d, D in enumerate(handles):
            torch.cuda.set_device(1 - d)                         # the OTHER device is current
            with torch.cuda.device(d):
                o = torch.empty_like(src[d])
                D.apply(o, src[d], 0, torch.cuda.current_stream(d))
            assert torch.cuda.current_device() == 1 - d
            outs.append(o)
    torch.cuda.synchronize(0)
    torch.cuda.synchronize(1)
    ref = outs[0].cpu()
    for o in outs:
        assert torch.equal(o.cpu(), ref)
    for D in handles:
        D.close()
