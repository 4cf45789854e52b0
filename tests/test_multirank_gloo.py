"""Multi-rank host logic on CPU (gloo, world size 2 and 4): the decomposition dslash_plan
computes, the face layouts include/hisq_dslash.h documents, and the NCCL issue order the
library uses (per direction: send bottom->minus, send top->plus, recv plus ghost, recv minus
ghost; messages of one pair are matched in issue order, like NCCL) deliver exactly the source
sites each rank's ghost zones must hold -- checked against the generator at global coordinates.
No Dslash arithmetic is involved."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import fieldgen
from paper_conf_sc_dufekgaad024_b200 import _abi

SEED = 77


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _faces(psi_cb, plan, mu):
    """(bottom, top) depth-3 faces of the local source field in the library's face layout."""
    L = plan.local_dims
    lxh = L[0] // 2
    v = psi_cb.reshape(3, L[3], L[2], L[1], lxh)          # [c][t][z][y][xh]
    if mu == 3:
        return v[:, :3].copy(), v[:, L[3] - 3:].copy()    # [c][d][z][y][xh]
    return v[:, :, :3].copy(), v[:, :, L[2] - 3:].copy()  # [c][t][d][y][xh]


def _expected_ghost(plan, mu, side, src_parity):
    """Generator values of the ghost slab: coordinates origin-3..origin-1 (side 0) or
    origin+L..origin+L+2 (side 1) along mu, periodic in the global lattice."""
    G, L, O = plan.global_dims, plan.local_dims, plan.origin
    lxh = L[0] // 2
    start = (O[mu] - 3) % G[mu] if side == 0 else (O[mu] + L[mu]) % G[mu]
    parts = []
    for d in range(3):
        o = list(O)
        o[mu] = (start + d) % G[mu]
        e = list(L)
        e[mu] = 1
        slab = fieldgen.vector_cb(G, SEED, src_parity, origin=o, extent=e)   # [c][one slice]
        if mu == 3:
            parts.append(slab.reshape(3, 1, L[2], L[1], lxh))
        else:
            parts.append(slab.reshape(3, L[3], 1, L[1], lxh))
    return np.concatenate(parts, axis=1 if mu == 3 else 2)


def _worker(rank, world, port, gdims, grid, src_parity, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        plan = _abi.dslash_plan(gdims, grid, rank, world)
        psi = fieldgen.vector_cb(gdims, SEED, src_parity, origin=tuple(plan.origin), extent=tuple(plan.local_dims))
        ok = []
        for mu in (3, 2):                          # the library's direction order: t then z
            if not plan.halo[mu]:
                continue
            bottom, top = _faces(psi, plan, mu)
            assert bottom.size == 3 * plan.face_vh[mu]
            ghost = [np.empty_like(bottom), np.empty_like(top)]
            minus, plus = plan.nbr_rank[mu][0], plan.nbr_rank[mu][1]
            as_t = lambda a: torch.from_numpy(np.ascontiguousarray(a).view(np.float64))
            bufs = [as_t(g) for g in ghost]
            reqs = [dist.isend(as_t(bottom), minus, tag=mu), dist.isend(as_t(top), plus, tag=mu),
                    dist.irecv(bufs[1], plus, tag=mu), dist.irecv(bufs[0], minus, tag=mu)]
            for r in reqs:
                r.wait()
            for side in (0, 1):
                got = bufs[side].numpy().view(np.complex128).reshape(ghost[side].shape)
                ok.append(np.array_equal(got, _expected_ghost(plan, mu, side, src_parity)))
        q.put((rank, all(ok), len(ok)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("gdims,grid", [((4, 6, 8, 16), (1, 1, 1, 2)), ((4, 6, 8, 8), (1, 1, 2, 1)),
                                        ((4, 2, 8, 16), (1, 1, 2, 2)), ((4, 4, 4, 24), (1, 1, 1, 4))])
@pytest.mark.parametrize("src_parity", [0, 1])
def test_halo_faces_gloo(gdims, grid, src_parity):
    world = int(np.prod(grid))
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, gdims, grid, src_parity, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    assert sorted(r for r, _, _ in res) == list(range(world))
    assert all(ok for _, ok, _ in res), res
    assert all(n > 0 for _, _, n in res)
