"""Property-based tests (hypothesis) of dslash_plan over random valid lattices and process
grids: the boxes are disjoint, cover the local lattice, keep every interior source local, and
the counts / neighbours / face sizes follow from the definitions.  Host only."""
import numpy as np
from hypothesis import given, settings
from hypothesis import strategies as st

from paper_conf_sc_dufekgaad024_b200 import _abi


@st.composite
def configs(draw):
    lx = 2 * draw(st.integers(1, 4))
    ly = 2 * draw(st.integers(1, 3))
    pz = draw(st.integers(1, 3))
    pt = draw(st.integers(1, 3))
    force = draw(st.sampled_from([0, 0x4, 0x8, 0xC]))
    # local halo extents must be even and >= 4; others even >= 2
    lz_loc = 2 * draw(st.integers(2 if (pz > 1 or force & 4) else 1, 4))
    lt_loc = 2 * draw(st.integers(2 if (pt > 1 or force & 8) else 1, 4))
    rank = draw(st.integers(0, pz * pt - 1))
    return (lx, ly, lz_loc * pz, lt_loc * pt), (1, 1, pz, pt), rank, force


@settings(max_examples=150, deadline=None)
@given(configs())
def test_plan_properties(cfg):
    dims, grid, rank, force = cfg
    n = grid[2] * grid[3]
    p = _abi.dslash_plan(dims, grid, rank, n, force)
    L = list(p.local_dims)
    assert [dims[d] // grid[d] for d in range(4)] == L
    assert p.vh_local == np.prod(L) // 2
    cover = np.zeros((L[3], L[2], L[1]), np.int32)
    boxes = [p.interior[i] for i in range(p.n_interior)] + [p.boundary[i] for i in range(p.n_boundary)]
    for b in boxes:
        assert b.lo[0] == 0 and b.hi[0] == L[0]          # x is never split
        cover[b.lo[3]:b.hi[3], b.lo[2]:b.hi[2], b.lo[1]:b.hi[1]] += 1
    assert np.all(cover == 1)                             # disjoint and complete
    halo = [bool(p.halo[d]) for d in range(4)]
    assert halo[2] == (grid[2] > 1 or bool(force & 4)) and halo[3] == (grid[3] > 1 or bool(force & 8))
    if p.n_interior:
        for d in (2, 3):
            if halo[d]:
                assert p.interior[0].lo[d] >= 3 and p.interior[0].hi[d] <= L[d] - 3   # all 16 sources local
    assert p.interior_sites + p.boundary_sites == p.vh_local
    cz, ct = rank % grid[2], rank // grid[2]
    assert tuple(p.origin) == (0, 0, cz * L[2], ct * L[3])
    for d, c, P in ((2, cz, grid[2]), (3, ct, grid[3])):
        minus, plus = p.nbr_rank[d][0], p.nbr_rank[d][1]
        cm, cp = (c - 1) % P, (c + 1) % P
        assert minus == (cm + grid[2] * ct if d == 2 else cz + grid[2] * cm)
        assert plus == (cp + grid[2] * ct if d == 2 else cz + grid[2] * cp)
        assert p.face_vh[d] == (3 * np.prod(L) // L[d] // 2 if halo[d] else 0)
