"""Brute-force HISQ Dslash operator built from shift permutation matrices (pin P1).

Independent of the oracle's index arithmetic: the hop x -> x+mu is a permutation
matrix obtained from ``np.roll`` of an index grid, and the third-neighbour hop is
its matrix CUBE, so a +3 / -1 confusion in either implementation cannot cancel.

    M = sum_mu [ F_mu S_mu - S_mu^T F_mu^dag + N_mu S_mu^3 - (S_mu^3)^T N_mu^dag ]

(Eq. (1), with the Naik terms of L27/L51; Z1, Z2.)
"""
import numpy as np
import scipy.sparse as sp

AXIS = {0: 3, 1: 2, 2: 1, 3: 0}  # mu -> numpy axis of a (t, z, y, x) array


def shift(dims, mu):
    """S_mu as a V x V permutation: (S psi)(x) = psi(x + mu), periodic."""
    lx, ly, lz, lt = dims
    V = lx * ly * lz * lt
    idx = np.arange(V).reshape(lt, lz, ly, lx)
    cols = np.roll(idx, -1, axis=AXIS[mu]).reshape(-1)
    return sp.csr_matrix((np.ones(V), (np.arange(V), cols)), shape=(V, V))


def blockdiag(m):
    """Block-diagonal 3V x 3V matrix from per-site 3x3 blocks m[V,3,3]."""
    V = m.shape[0]
    return sp.bsr_matrix((m, np.arange(V), np.arange(V + 1)), shape=(3 * V, 3 * V)).tocsr()


def operator(fat, lng):
    """The full (both-parity) operator M as a sparse 3V x 3V matrix."""
    lt, lz, ly, lx = fat.shape[:4]
    dims = (lx, ly, lz, lt)
    V = lx * ly * lz * lt
    I3 = sp.identity(3, format="csr")
    M = sp.csr_matrix((3 * V, 3 * V), dtype=np.complex128)
    for mu in range(4):
        S = shift(dims, mu)
        S3 = S @ S @ S
        Sk = sp.kron(S, I3, format="csr")
        S3k = sp.kron(S3, I3, format="csr")
        F = blockdiag(fat.reshape(V, 4, 3, 3)[:, mu])
        N = blockdiag(lng.reshape(V, 4, 3, 3)[:, mu])
        M = M + F @ Sk - Sk.T @ F.conj().T + N @ S3k - S3k.T @ N.conj().T
    return M


def apply(M, psi_full):
    return (M @ psi_full.reshape(-1)).reshape(psi_full.shape)
