"""CPU oracle of the single-parity HISQ Dslash -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The CUDA product path
(``paper_conf_sc_dufekgaad024_b200``) never imports it, and the two share no code;
the only shared module is the seeded input generator ``fieldgen``.

The arithmetic lives in ``hisq_oracle.c`` (plain C99 complex, fp64, -O2
-ffp-contract=off), which follows PAPER.md Eq. (1) (L45-51, §II) plus the Naik
third-neighbour terms (L27, L51); see its header and DESIGN.md for the readings
Z1-Z18.  Pins: ``tests/test_oracle_pins.py`` (P1-P9).

Layouts here are the plain full-lattice ones: links ``(Lt, Lz, Ly, Lx, 4, 3, 3)``
(forward only, canonical) and vectors ``(Lt, Lz, Ly, Lx, 3)``.
``full_to_cb`` / ``cb_to_full`` translate to and from the library's vector layout
``[3][Vh]`` (checkerboard index cb = lex // 2) so results can be compared.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "hisq_oracle.c")
_LIB = os.path.join(_HERE, "libhisq_oracle.so")

FLOP_PER_SITE = 1146  # 600.8 MFLOP per apply at L=32 -> 1146 per target site


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-std=c99", "-O2", "-ffp-contract=off", "-fopenmp", "-fPIC", "-shared",
                               "-o", _LIB, _SRC, "-lm"])
    return _LIB


_lib = None


def _get():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        i4 = ctypes.POINTER(ctypes.c_int32)
        vp = ctypes.c_void_p
        lib.oracle_dslash.argtypes = [i4, vp, vp, vp, vp, ctypes.c_int32, ctypes.c_int32]
        lib.oracle_dslash.restype = ctypes.c_int
        lib.oracle_dslash_sites.argtypes = [i4, vp, vp, vp, ctypes.c_int64, vp, vp, ctypes.c_int32]
        lib.oracle_dslash_sites.restype = ctypes.c_int
        _lib = lib
    return _lib


def _dims_of(links):
    lt, lz, ly, lx = links.shape[:4]
    return (lx, ly, lz, lt)


def _c(a):
    a = np.ascontiguousarray(a, dtype=np.complex128)
    return a


def dslash(fat, lng, psi, parity, nthreads=0):
    """chi = D psi on target parity `parity`; full-lattice arrays; chi = 0 off parity."""
    fat, lng, psi = _c(fat), _c(lng), _c(psi)
    dims = _dims_of(fat)
    assert fat.shape == lng.shape == (dims[3], dims[2], dims[1], dims[0], 4, 3, 3)
    assert psi.shape == (dims[3], dims[2], dims[1], dims[0], 3)
    chi = np.empty_like(psi)
    d = (ctypes.c_int32 * 4)(*dims)
    rc = _get().oracle_dslash(d, fat.ctypes.data, lng.ctypes.data, psi.ctypes.data, chi.ctypes.data,
                              int(parity), int(nthreads))
    if rc != 0:
        raise ValueError("oracle_dslash: bad arguments")
    return chi


def dslash_sites(fat, lng, psi, sites, nthreads=0):
    """(D psi)(x) at the given lex site indices, shape (n, 3)."""
    fat, lng, psi = _c(fat), _c(lng), _c(psi)
    dims = _dims_of(fat)
    sites = np.ascontiguousarray(sites, dtype=np.int64)
    out = np.empty((sites.size, 3), dtype=np.complex128)
    d = (ctypes.c_int32 * 4)(*dims)
    rc = _get().oracle_dslash_sites(d, fat.ctypes.data, lng.ctypes.data, psi.ctypes.data, sites.size,
                                    sites.ctypes.data, out.ctypes.data, int(nthreads))
    if rc != 0:
        raise ValueError("oracle_dslash_sites: bad arguments")
    return out


# ---- layout translation for comparisons (index bookkeeping only, no Dslash arithmetic) ----

def parity_mask(dims):
    """Boolean (Lt, Lz, Ly, Lx) array: True where (x+y+z+t) is odd."""
    lx, ly, lz, lt = dims
    t, z, y, x = np.meshgrid(np.arange(lt), np.arange(lz), np.arange(ly), np.arange(lx), indexing="ij")
    return ((x + y + z + t) & 1).astype(bool)


def lex_sites_of_parity(dims, parity):
    """Lex indices of the sites of the given parity, in increasing lex order (= cb order)."""
    odd = parity_mask(dims).reshape(-1)
    return np.nonzero(odd == bool(parity))[0]


def full_to_cb(v_full, parity):
    """(Lt,Lz,Ly,Lx,3) -> [3][Vh] on the sites of `parity`, ordered by lex (cb = lex // 2)."""
    lt, lz, ly, lx, _ = v_full.shape
    s = lex_sites_of_parity((lx, ly, lz, lt), parity)
    return np.ascontiguousarray(v_full.reshape(-1, 3)[s].T)


def cb_to_full(v_cb, dims, parity):
    """Inverse of full_to_cb; sites of the other parity are 0."""
    lx, ly, lz, lt = dims
    out = np.zeros((lx * ly * lz * lt, 3), dtype=np.complex128)
    out[lex_sites_of_parity(dims, parity)] = np.asarray(v_cb).T
    return out.reshape(lt, lz, ly, lx, 3)


def normwise_error(a, ref):
    """max |a - ref| / max |ref| (reading Z11)."""
    a = np.asarray(a)
    ref = np.asarray(ref)
    den = np.abs(ref).max()
    return float(np.abs(a - ref).max() / den) if den > 0 else float(np.abs(a).max())
