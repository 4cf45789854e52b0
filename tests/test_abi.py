"""The C ABI without a GPU: the library loads, exports every function include/hisq_dslash.h
declares, and its host-only entry points (dslash_plan, argument checks that precede any CUDA
call) behave as documented.  No compute calls here."""
import ctypes
import re

import pytest

from paper_conf_sc_dufekgaad024_b200 import _abi


def declared_functions():
    src = open(_abi.HEADER).read()
    return sorted(set(re.findall(r"^DSLASH_API\s+[\w\s\*]+?\b(dslash_\w+)\s*\(", src, flags=re.M)))


def test_header_declares_the_survey_boundary():
    names = declared_functions()
    for must in ("dslash_create", "dslash_load_links", "dslash_apply", "dslash_halo_start", "dslash_halo_wait",
                 "dslash_sync", "dslash_destroy", "dslash_error_string", "dslash_local_half_volume"):
        assert must in names


def test_library_exports_every_declared_symbol():
    names = declared_functions()
    assert len(names) >= 15
    for n in names:
        assert hasattr(_abi.lib, n), f"{n} declared in the header but not exported"
        assert n in _abi.EXPORTED, f"{n} has no Python binding"


def test_plan_single_gpu():
    p = _abi.dslash_plan((32, 32, 32, 32))
    assert p.vh_local == 32 ** 4 // 2
    assert p.n_interior == 1 and p.n_boundary == 0
    assert p.interior_sites == p.vh_local and list(p.halo) == [0, 0, 0, 0]


@pytest.mark.parametrize("grid,rank", [((1, 1, 1, 8), 3), ((1, 1, 2, 4), 5), ((1, 1, 2, 1), 1)])
def test_plan_partitioned_counts(grid, rank):
    n = grid[0] * grid[1] * grid[2] * grid[3]
    p = _abi.dslash_plan((32, 32, 32, 32 * grid[3]), grid, rank, n)
    assert p.interior_sites + p.boundary_sites == p.vh_local
    # boxes are disjoint and cover the local lattice exactly
    seen = set()
    boxes = [p.interior[i] for i in range(p.n_interior)] + [p.boundary[i] for i in range(p.n_boundary)]
    for b in boxes:
        for t in range(b.lo[3], b.hi[3]):
            for z in range(b.lo[2], b.hi[2]):
                for y in range(b.lo[1], b.hi[1]):
                    key = (y, z, t)
                    assert key not in seen
                    seen.add(key)
    L = p.local_dims
    assert len(seen) == L[1] * L[2] * L[3]
    # interior sites keep all 16 sources local: 3 <= c < L-3 along halo directions
    for d in range(4):
        if p.halo[d]:
            assert p.interior[0].lo[d] == 3 and p.interior[0].hi[d] == L[d] - 3
            assert p.face_vh[d] == 3 * (L[0] * L[1] * L[2] * L[3] // L[d]) // 2
    # neighbour ranks: rank = cz + Pz * ct
    cz, ct = rank % grid[2], rank // grid[2]
    assert (p.proc_coords[2], p.proc_coords[3]) == (cz, ct)
    assert p.nbr_rank[3][1] == cz + grid[2] * ((ct + 1) % grid[3])
    assert p.nbr_rank[3][0] == cz + grid[2] * ((ct - 1) % grid[3])
    assert p.nbr_rank[2][1] == (cz + 1) % grid[2] + grid[2] * ct
    assert p.origin[3] == ct * L[3] and p.origin[2] == cz * L[2]


def test_plan_interior_fraction_matches_survey():
    # 32^3 x 32 per GPU t-partitioned -> 81% interior; 48^4 t8 -> 0%
    p = _abi.dslash_plan((32, 32, 32, 256), (1, 1, 1, 8), 0, 8)
    assert p.interior_sites / p.vh_local == pytest.approx(26 / 32)
    p = _abi.dslash_plan((48, 48, 48, 48), (1, 1, 1, 8), 0, 8)
    assert p.interior_sites == 0 and p.boundary_sites == p.vh_local
    p = _abi.dslash_plan((48, 48, 48, 48), (1, 1, 2, 4), 0, 8)
    assert p.interior_sites / p.vh_local == pytest.approx((6 / 12) * (18 / 24))


@pytest.mark.parametrize("dims,grid,nr,code", [
    ((31, 32, 32, 32), (1, 1, 1, 1), 1, _abi.DSLASH_ERR_ARG),       # odd extent
    ((32, 32, 32, 32), (1, 1, 1, 3), 3, _abi.DSLASH_ERR_ARG),       # not divisible
    ((32, 32, 32, 12), (1, 1, 1, 6), 6, _abi.DSLASH_ERR_ARG),       # local extent 2 < 4
    ((32, 32, 32, 30), (1, 1, 1, 6), 6, _abi.DSLASH_ERR_ARG),       # local extent 5 odd
    ((32, 32, 32, 32), (1, 1, 1, 2), 1, _abi.DSLASH_ERR_ARG),       # nranks mismatch
    ((32, 32, 32, 32), (2, 1, 1, 1), 2, _abi.DSLASH_ERR_UNSUPPORTED),  # x partition
])
def test_plan_errors(dims, grid, nr, code):
    with pytest.raises(_abi.DslashError) as e:
        _abi.dslash_plan(dims, grid, 0, nr)
    assert e.value.status == code
    assert _abi.dslash_error_string(None)


def test_self_halo_plan():
    p = _abi.dslash_plan((8, 8, 8, 8), force_halo_mask=0xC)
    assert list(p.halo) == [0, 0, 1, 1]
    assert p.nbr_rank[3][0] == p.nbr_rank[3][1] == 0
    p = _abi.dslash_plan((4, 4, 4, 4), force_halo_mask=0x8)
    assert p.n_interior == 0 and p.boundary_sites == p.vh_local
    with pytest.raises(_abi.DslashError):
        _abi.dslash_plan((8, 8, 8, 8), force_halo_mask=0x1)     # x halo unsupported


def test_create_argument_errors_precede_cuda():
    h = ctypes.c_void_p()
    rc = _abi.lib.dslash_create(_abi.i4((7, 8, 8, 8)), _abi.i4((1, 1, 1, 1)), 0, 0, None, 1, 0, ctypes.byref(h))
    assert rc == _abi.DSLASH_ERR_ARG and not h.value
    rc = _abi.lib.dslash_create(_abi.i4((8, 8, 8, 8)), _abi.i4((1, 1, 1, 1)), 5, 0, None, 1, 0, ctypes.byref(h))
    assert rc == _abi.DSLASH_ERR_ARG
    rc = _abi.lib.dslash_create(_abi.i4((8, 8, 8, 8)), _abi.i4((1, 1, 1, 2)), 2, 0, None, 4, 0, ctypes.byref(h))
    assert rc == _abi.DSLASH_ERR_ARG           # prod(proc_grid) != nranks
    rc = _abi.lib.dslash_create(_abi.i4((8, 8, 8, 8)), _abi.i4((1, 1, 1, 1)), 0, 7, None, 1, 0, ctypes.byref(h))
    assert rc == _abi.DSLASH_ERR_ARG           # unknown precision
    assert _abi.lib.dslash_apply(None, None, None, 0, None) == _abi.DSLASH_ERR_ARG
    assert _abi.lib.dslash_local_half_volume(None) == -1
    assert _abi.lib.dslash_destroy(None) == _abi.DSLASH_OK
    assert _abi.dslash_ipc_blob_size() > 9 * 64          # 9 CUDA IPC handles + header


def test_c_demo_builds_and_links():
    """The boundary is a plain C ABI: examples/c_api_demo.c compiles against include/ and links
    the library with gcc (it runs on the GPU in tests/test_gpu_parity.py)."""
    import os
    from paper_conf_sc_dufekgaad024_b200 import build
    exe = build.build_c_demo()
    assert os.path.exists(exe)
