"""The shared seeded input generator (fieldgen/): determinism, partition
independence, SU(3) properties and layout consistency.  No Dslash arithmetic."""
import numpy as np
import pytest

import fieldgen
import oracle


def test_su3_links_are_special_unitary():
    u = fieldgen.links((4, 6, 4, 8), 1).reshape(-1, 3, 3)
    eye = np.einsum("nij,nkj->nik", u, u.conj())
    assert np.abs(eye - np.eye(3)).max() < 1e-14
    assert np.abs(np.linalg.det(u) - 1).max() < 1e-14


def test_su3_haar_moments():
    # Haar SU(3): E[U_ij] = 0 and E[|U_ij|^2] = 1/3
    u = fieldgen.links((8, 8, 8, 8), 5).reshape(-1, 3, 3)
    assert np.abs(u.mean(0)).max() < 0.01
    assert np.abs((np.abs(u) ** 2).mean(0) - 1 / 3).max() < 0.01


def test_long_link_scale():
    fat, lng = fieldgen.workload_links((4, 4, 4, 4))
    raw = fieldgen.links((4, 4, 4, 4), fieldgen.SEED_LONG)
    assert np.array_equal(lng, raw * fieldgen.LONG_SCALE)
    assert not np.array_equal(fat, raw)


def test_deterministic():
    a = fieldgen.vector((4, 4, 4, 6), 3)
    b = fieldgen.vector((4, 4, 4, 6), 3)
    assert np.array_equal(a, b)
    assert not np.array_equal(a, fieldgen.vector((4, 4, 4, 6), 4))


@pytest.mark.parametrize("kind", ["su3", "gauss"])
def test_partition_independent(kind):
    dims = (4, 6, 8, 12)
    full = fieldgen.links(dims, 9, kind)
    part = fieldgen.links(dims, 9, kind, origin=(0, 0, 4, 6), extent=(4, 6, 4, 6))
    assert np.array_equal(part, full[6:12, 4:8])
    v = fieldgen.vector(dims, 9)
    assert np.array_equal(fieldgen.vector(dims, 9, origin=(0, 0, 2, 3), extent=(4, 6, 2, 3)), v[3:6, 2:4])


@pytest.mark.parametrize("parity", [0, 1])
def test_vector_cb_layout(parity):
    dims = (4, 6, 8, 10)
    full = fieldgen.vector(dims, 3)
    assert np.array_equal(fieldgen.vector_cb(dims, 3, parity), oracle.full_to_cb(full, parity))
    # on a partitioned box the local cb order is the local lex order of the parity-p sites
    part = fieldgen.vector_cb(dims, 3, parity, origin=(0, 0, 4, 2), extent=(4, 6, 4, 4))
    assert np.array_equal(part, oracle.full_to_cb(full[2:6, 4:8], parity))


def test_bad_arguments():
    with pytest.raises(ValueError):
        fieldgen.vector((4, 4, 4, 4), 1, origin=(0, 0, 0, 2), extent=(4, 4, 4, 4))
    with pytest.raises(ValueError):
        fieldgen.vector_cb((3, 4, 4, 4), 1, 0)
