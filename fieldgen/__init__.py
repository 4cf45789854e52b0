"""Seeded counter-based synthetic fields for the HISQ Dslash (shared input generator).

This package is the only code the CPU oracle (``oracle/``) and the CUDA path
(``paper_conf_sc_dufekgaad024_b200``) have in common.  It contains no Dslash
arithmetic: it draws random numbers keyed by (seed, global site, slot, element)
and writes them in the layouts both sides consume (see ``fieldgen.c``).

Seeds of the benchmark workload: fat links 1, long links 2,
source vector 3, gauge transform 4.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "fieldgen.c")
_LIB = os.path.join(_HERE, "libfieldgen.so")

SEED_FAT, SEED_LONG, SEED_PSI, SEED_GAUGE = 1, 2, 3, 4
LONG_SCALE = -1.0 / 24.0  # Naik coefficient used for the long links of the workload


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fopenmp", "-fPIC", "-shared",
                               "-o", _LIB, _SRC, "-lm"])
    return _LIB


_lib = None


def _get():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        i4 = ctypes.POINTER(ctypes.c_int32)
        dp = ctypes.c_void_p
        lib.fg_matrices.argtypes = [i4, i4, i4, ctypes.c_uint64, ctypes.c_int32, ctypes.c_int32,
                                    ctypes.c_double, dp]
        lib.fg_matrices.restype = ctypes.c_int64
        lib.fg_vector.argtypes = [i4, i4, i4, ctypes.c_uint64, dp]
        lib.fg_vector.restype = ctypes.c_int64
        lib.fg_vector_cb.argtypes = [i4, i4, i4, ctypes.c_uint64, ctypes.c_int32, dp]
        lib.fg_vector_cb.restype = ctypes.c_int64
        _lib = lib
    return _lib


def _i4(v):
    return (ctypes.c_int32 * 4)(*[int(a) for a in v])


def _box(dims, origin, extent):
    dims = tuple(int(d) for d in dims)
    origin = (0, 0, 0, 0) if origin is None else tuple(int(o) for o in origin)
    extent = dims if extent is None else tuple(int(e) for e in extent)
    return dims, origin, extent


def matrices(dims, seed, nper=4, kind="su3", scale=1.0, origin=None, extent=None, out=None):
    """Matrix field over a local box, shape (Et, Ez, Ey, Ex, nper, 3, 3) complex128.

    With nper=4 this is the canonical link layout [t][z][y][x][mu][3][3]
    (PAPER.md L364).  kind: "su3" (Haar SU(3)) or "gauss" (complex Gaussian).
    """
    dims, origin, extent = _box(dims, origin, extent)
    shape = (extent[3], extent[2], extent[1], extent[0], nper, 3, 3)
    if out is None:
        out = np.empty(shape, dtype=np.complex128)
    assert out.shape == shape and out.dtype == np.complex128 and out.flags.c_contiguous
    k = {"su3": 0, "gauss": 1}[kind]
    n = _get().fg_matrices(_i4(dims), _i4(origin), _i4(extent), seed, nper, k, float(scale),
                           out.ctypes.data)
    if n < 0:
        raise ValueError("fieldgen: bad arguments")
    return out


def links(dims, seed, kind="su3", scale=1.0, origin=None, extent=None, out=None):
    """Canonical forward links [t][z][y][x][mu][3][3] complex128 over a local box."""
    return matrices(dims, seed, 4, kind, scale, origin, extent, out)


def vector(dims, seed, origin=None, extent=None):
    """Full-box colour vector, shape (Et, Ez, Ey, Ex, 3) complex128 (both parities)."""
    dims, origin, extent = _box(dims, origin, extent)
    out = np.empty((extent[3], extent[2], extent[1], extent[0], 3), dtype=np.complex128)
    if _get().fg_vector(_i4(dims), _i4(origin), _i4(extent), seed, out.ctypes.data) < 0:
        raise ValueError("fieldgen: bad arguments")
    return out


def vector_cb(dims, seed, parity, origin=None, extent=None, out=None):
    """The same values on one parity, in the library vector layout [3][Vh] complex128."""
    dims, origin, extent = _box(dims, origin, extent)
    vh = extent[0] * extent[1] * extent[2] * extent[3] // 2
    if out is None:
        out = np.empty((3, vh), dtype=np.complex128)
    assert out.shape == (3, vh) and out.dtype == np.complex128 and out.flags.c_contiguous
    if _get().fg_vector_cb(_i4(dims), _i4(origin), _i4(extent), seed, int(parity), out.ctypes.data) < 0:
        raise ValueError("fieldgen: bad arguments")
    return out


def workload_links(dims, origin=None, extent=None):
    """The benchmark's fat (SU(3), seed 1) and long (-1/24 SU(3), seed 2) links."""
    fat = links(dims, SEED_FAT, "su3", 1.0, origin, extent)
    lng = links(dims, SEED_LONG, "su3", LONG_SCALE, origin, extent)
    return fat, lng
