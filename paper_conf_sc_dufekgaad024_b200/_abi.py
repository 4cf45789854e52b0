"""ctypes binding of include/hisq_dslash.h -- argument marshalling only.

Every function here has the same name and arguments as the C ABI; all computation
happens inside libhisq_dslash.so (CUDA, sm_100a).  Importing this module on a
machine without the built library raises immediately: there is no fallback.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# HISQ_DSLASH_LIB: another build of the same library (A/B measurement of a compile-time variant)
LIB_PATH = os.environ.get("HISQ_DSLASH_LIB") or os.path.join(_HERE, "libhisq_dslash.so")
HEADER = os.path.join(os.path.dirname(_HERE), "include", "hisq_dslash.h")

DSLASH_OK, DSLASH_ERR_ARG, DSLASH_ERR_STATE, DSLASH_ERR_CUDA, DSLASH_ERR_NCCL, DSLASH_ERR_OOM, \
    DSLASH_ERR_UNSUPPORTED, DSLASH_ERR_NOT_CONVERGED = range(8)
STATUS_NAMES = {0: "DSLASH_OK", 1: "DSLASH_ERR_ARG", 2: "DSLASH_ERR_STATE", 3: "DSLASH_ERR_CUDA",
                4: "DSLASH_ERR_NCCL", 5: "DSLASH_ERR_OOM", 6: "DSLASH_ERR_UNSUPPORTED",
                7: "DSLASH_ERR_NOT_CONVERGED"}
DSLASH_EVEN, DSLASH_ODD, DSLASH_BOTH = 0, 1, 2
DSLASH_F64, DSLASH_F32, DSLASH_MIXED = 0, 1, 2
PRECISIONS = {"f64": DSLASH_F64, "f32": DSLASH_F32, "mixed": DSLASH_MIXED}
DSLASH_KERNEL_SITE, DSLASH_KERNEL_DIR4, DSLASH_KERNEL_DIR2 = 0, 1, 2
# option keys (the values 7 and 12 belonged to options that were removed)
DSLASH_OPT_KERNEL, DSLASH_OPT_BLOCK, DSLASH_OPT_FORCE_HALO, DSLASH_OPT_OVERLAP, DSLASH_OPT_TIMING, \
    DSLASH_OPT_MIN_BLOCKS, DSLASH_OPT_LONG_RECON = range(7)
DSLASH_OPT_TRANSPORT, DSLASH_OPT_PDL, DSLASH_OPT_SELF_NCCL, DSLASH_OPT_STAGE = range(8, 12)
DSLASH_OPT_HALO_DRYRUN, DSLASH_OPT_PUSH = 13, 14
DSLASH_TRANSPORT_NCCL, DSLASH_TRANSPORT_P2P = 0, 1
DSLASH_OVERLAP_NONE, DSLASH_OVERLAP_SITES, DSLASH_OVERLAP_DIRS = 0, 1, 2
OVERLAPS = {"none": DSLASH_OVERLAP_NONE, "sites": DSLASH_OVERLAP_SITES, "dirs": DSLASH_OVERLAP_DIRS}
TRANSPORTS = {"nccl": DSLASH_TRANSPORT_NCCL, "p2p": DSLASH_TRANSPORT_P2P}
DSLASH_TIMING_INTERIOR, DSLASH_TIMING_BOUNDARY, DSLASH_TIMING_ALL, DSLASH_TIMING_SPAN, DSLASH_TIMING_EXCHANGE = range(5)
TIMING_KINDS = {0: "interior", 1: "boundary", 2: "all", 3: "span", 4: "exchange"}
KERNELS = {"site": DSLASH_KERNEL_SITE, "dir4": DSLASH_KERNEL_DIR4, "dir2": DSLASH_KERNEL_DIR2}


class dslash_box_t(ctypes.Structure):
    _fields_ = [("lo", ctypes.c_int32 * 4), ("hi", ctypes.c_int32 * 4)]


class dslash_plan_t(ctypes.Structure):
    _fields_ = [
        ("global_dims", ctypes.c_int32 * 4),
        ("proc_grid", ctypes.c_int32 * 4),
        ("proc_coords", ctypes.c_int32 * 4),
        ("local_dims", ctypes.c_int32 * 4),
        ("origin", ctypes.c_int32 * 4),
        ("halo", ctypes.c_int32 * 4),
        ("nbr_rank", (ctypes.c_int32 * 2) * 4),
        ("rank", ctypes.c_int32),
        ("nranks", ctypes.c_int32),
        ("vh_local", ctypes.c_int64),
        ("face_vh", ctypes.c_int64 * 4),
        ("n_interior", ctypes.c_int32),
        ("n_boundary", ctypes.c_int32),
        ("interior", dslash_box_t * 1),
        ("boundary", dslash_box_t * 4),
        ("interior_sites", ctypes.c_int64),
        ("boundary_sites", ctypes.c_int64),
    ]


class DslashError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS_NAMES.get(status, status)}: {msg}")
        self.status = status


if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is not built: run `python -c 'import __graft_entry__ as g; g.build()'` "
                      "(no CPU fallback exists)")

lib = ctypes.CDLL(LIB_PATH)

_i4 = ctypes.POINTER(ctypes.c_int32)
_h = ctypes.c_void_p
_vp = ctypes.c_void_p

_SIGS = {
    "dslash_plan": ([_i4, _i4, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, ctypes.POINTER(dslash_plan_t)],
                    ctypes.c_int),
    "dslash_create": ([_i4, _i4, ctypes.c_int32, ctypes.c_int32, _vp, ctypes.c_int32, ctypes.c_int32,
                       ctypes.POINTER(_h)], ctypes.c_int),
    "dslash_get_unique_id": ([_vp], ctypes.c_int),
    "dslash_set_device": ([ctypes.c_int32], ctypes.c_int),
    "dslash_device_count": ([], ctypes.c_int32),
    "dslash_ipc_blob_size": ([], ctypes.c_int64),
    "dslash_get_ipc_blob": ([_h, _vp], ctypes.c_int),
    "dslash_open_ipc_blobs": ([_h, _vp], ctypes.c_int),
    "dslash_get_links": ([_h, ctypes.c_int32, _vp], ctypes.c_int),
    "dslash_load_links_halo": ([_h, _vp, _vp, ctypes.POINTER(_vp), ctypes.POINTER(_vp), ctypes.c_int32, _vp],
                               ctypes.c_int),
    "dslash_set_option": ([_h, ctypes.c_int32, ctypes.c_int64], ctypes.c_int),
    "dslash_load_links": ([_h, _vp, _vp, ctypes.c_int32, _vp], ctypes.c_int),
    "dslash_apply": ([_h, _vp, _vp, ctypes.c_int32, _vp], ctypes.c_int),
    "dslash_apply_push": ([_h, _vp, _vp, ctypes.c_int32, _vp], ctypes.c_int),
    "dslash_apply_multi": ([_h, ctypes.c_int32, _vp, _vp, ctypes.c_int32, _vp], ctypes.c_int),
    "dslash_apply_multi_blocked": ([_h, ctypes.c_int32, _vp, _vp, ctypes.c_int32, _vp], ctypes.c_int),
    "dslash_vectors_to_blocked": ([_h, ctypes.c_int32, _vp, _vp, _vp], ctypes.c_int),
    "dslash_vectors_from_blocked": ([_h, ctypes.c_int32, _vp, _vp, _vp], ctypes.c_int),
    "dslash_apply_host": ([_h, _vp, _vp, ctypes.c_int32, _vp], ctypes.c_int),
    "dslash_apply_host_batch": ([_h, ctypes.c_int32, ctypes.POINTER(_vp), ctypes.POINTER(_vp), ctypes.c_int32,
                                 _vp], ctypes.c_int),
    "dslash_normal_apply": ([_h, _vp, _vp, ctypes.c_int32, ctypes.c_double, _vp], ctypes.c_int),
    "dslash_cg": ([_h, _vp, _vp, ctypes.c_int32, ctypes.c_double, ctypes.c_double, ctypes.c_int32,
                   ctypes.POINTER(ctypes.c_int32), ctypes.POINTER(ctypes.c_double), _vp], ctypes.c_int),
    "dslash_cg_mixed": ([_h, _vp, _vp, ctypes.c_int32, ctypes.c_double, ctypes.c_double, ctypes.c_double,
                         ctypes.c_int32, ctypes.POINTER(ctypes.c_int32), ctypes.POINTER(ctypes.c_int32),
                         ctypes.POINTER(ctypes.c_double), _vp], ctypes.c_int),
    "dslash_cg_multi_blocked": ([_h, ctypes.c_int32, _vp, _vp, ctypes.c_int32, ctypes.c_double, ctypes.c_double,
                                 ctypes.c_int32, ctypes.POINTER(ctypes.c_int32), ctypes.POINTER(ctypes.c_double), _vp],
                                ctypes.c_int),
    "dslash_halo_start": ([_h, _vp, ctypes.c_int32, _vp], ctypes.c_int),
    "dslash_halo_wait": ([_h, _vp], ctypes.c_int),
    "dslash_sync": ([_h], ctypes.c_int),
    "dslash_kernel_timing": ([_h, ctypes.c_int32, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_int64)],
                             ctypes.c_int),
    "dslash_kernel_timing_reset": ([_h], ctypes.c_int),
    "dslash_timeline": ([_h, ctypes.c_int64, ctypes.POINTER(ctypes.c_int32), ctypes.POINTER(ctypes.c_double),
                         ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_int64)], ctypes.c_int),
    "dslash_get_plan": ([_h, ctypes.POINTER(dslash_plan_t)], ctypes.c_int),
    "dslash_local_half_volume": ([_h], ctypes.c_int64),
    "dslash_destroy": ([_h], ctypes.c_int),
    "dslash_error_string": ([_h], ctypes.c_char_p),
}
for _name, (_args, _res) in _SIGS.items():
    _f = getattr(lib, _name)
    _f.argtypes = _args
    _f.restype = _res

EXPORTED = tuple(_SIGS)


def error_string(h=None) -> str:
    s = lib.dslash_error_string(h)
    return s.decode() if s else ""


def check(status, h=None):
    if status != DSLASH_OK:
        raise DslashError(status, error_string(h))
    return status


def i4(v):
    return (ctypes.c_int32 * 4)(*[int(a) for a in v])


# ---- the C ABI under its own names (argument marshalling only) ----

def dslash_plan(global_dims, proc_grid=(1, 1, 1, 1), rank=0, nranks=1, force_halo_mask=0) -> dslash_plan_t:
    p = dslash_plan_t()
    check(lib.dslash_plan(i4(global_dims), i4(proc_grid), rank, nranks, force_halo_mask, ctypes.byref(p)))
    return p


def dslash_set_device(device: int) -> None:
    check(lib.dslash_set_device(int(device)))


def dslash_device_count() -> int:
    return int(lib.dslash_device_count())


def dslash_get_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    check(lib.dslash_get_unique_id(buf))
    return buf.raw


def dslash_create(global_dims, proc_grid=(1, 1, 1, 1), parity_mask=DSLASH_BOTH, precision=DSLASH_F64,
                  nccl_unique_id: bytes | None = None, nranks=1, rank=0):
    h = ctypes.c_void_p()
    uid = ctypes.create_string_buffer(nccl_unique_id, 128) if nccl_unique_id is not None else None
    check(lib.dslash_create(i4(global_dims), i4(proc_grid), parity_mask, precision, uid, nranks, rank,
                            ctypes.byref(h)))
    return h


def dslash_ipc_blob_size() -> int:
    return int(lib.dslash_ipc_blob_size())


def dslash_get_ipc_blob(h) -> bytes:
    buf = ctypes.create_string_buffer(dslash_ipc_blob_size())
    check(lib.dslash_get_ipc_blob(h, buf), h)
    return buf.raw


def dslash_open_ipc_blobs(h, blobs: bytes):
    buf = ctypes.create_string_buffer(blobs, len(blobs))
    return check(lib.dslash_open_ipc_blobs(h, buf), h)


def dslash_load_links_halo(h, fat_ptr, lng_ptr, slab_fat_ptrs, slab_lng_ptrs, on_device, stream=0):
    sf = (ctypes.c_void_p * 4)(*[p or None for p in slab_fat_ptrs])
    sl = (ctypes.c_void_p * 4)(*[p or None for p in slab_lng_ptrs])
    return check(lib.dslash_load_links_halo(h, fat_ptr, lng_ptr, sf, sl, on_device, stream), h)


def dslash_get_links(h, parity, out_ptr):
    return check(lib.dslash_get_links(h, parity, out_ptr), h)


def dslash_set_option(h, key, value):
    return check(lib.dslash_set_option(h, key, value), h)


def dslash_load_links(h, fat_ptr, lng_ptr, on_device, stream=0):
    return check(lib.dslash_load_links(h, fat_ptr, lng_ptr, on_device, stream), h)


def dslash_apply(h, out_ptr, in_ptr, parity, stream=0):
    return check(lib.dslash_apply(h, out_ptr, in_ptr, parity, stream), h)


def dslash_apply_push(h, out_ptr, in_ptr, parity, stream=0):
    return check(lib.dslash_apply_push(h, out_ptr, in_ptr, parity, stream), h)


def dslash_apply_multi(h, nrhs, out_ptr, in_ptr, parity, stream=0):
    return check(lib.dslash_apply_multi(h, nrhs, out_ptr, in_ptr, parity, stream), h)


def dslash_apply_multi_blocked(h, nrhs, out_ptr, in_ptr, parity, stream=0):
    return check(lib.dslash_apply_multi_blocked(h, nrhs, out_ptr, in_ptr, parity, stream), h)


def dslash_vectors_to_blocked(h, nrhs, blocked_ptr, planar_ptr, stream=0):
    return check(lib.dslash_vectors_to_blocked(h, nrhs, blocked_ptr, planar_ptr, stream), h)


def dslash_vectors_from_blocked(h, nrhs, planar_ptr, blocked_ptr, stream=0):
    return check(lib.dslash_vectors_from_blocked(h, nrhs, planar_ptr, blocked_ptr, stream), h)


def dslash_apply_host(h, out_ptr, in_ptr, parity, stream=0):
    return check(lib.dslash_apply_host(h, out_ptr, in_ptr, parity, stream), h)


def dslash_apply_host_batch(h, out_ptrs, in_ptrs, parity, stream=0):
    n = len(out_ptrs)
    if len(in_ptrs) != n:
        raise ValueError("out_ptrs and in_ptrs differ in length")
    outs = (ctypes.c_void_p * max(n, 1))(*out_ptrs)
    ins = (ctypes.c_void_p * max(n, 1))(*in_ptrs)
    return check(lib.dslash_apply_host_batch(h, n, outs, ins, parity, stream), h)


def dslash_normal_apply(h, out_ptr, in_ptr, parity, mass, stream=0):
    return check(lib.dslash_normal_apply(h, out_ptr, in_ptr, parity, mass, stream), h)


def dslash_cg(h, x_ptr, b_ptr, parity, mass, rel_tol, max_iter, stream=0):
    """Returns (status, iterations, true relative residual); status is DSLASH_OK or
    DSLASH_ERR_NOT_CONVERGED, anything else raises."""
    it = ctypes.c_int32()
    res = ctypes.c_double()
    st = lib.dslash_cg(h, x_ptr, b_ptr, parity, mass, rel_tol, max_iter, ctypes.byref(it), ctypes.byref(res), stream)
    if st not in (DSLASH_OK, DSLASH_ERR_NOT_CONVERGED):
        check(st, h)
    return st, it.value, res.value


def dslash_cg_multi_blocked(h, nrhs, x_ptr, b_ptr, parity, mass, rel_tol, max_iter, stream=0):
    """Returns (status, [iterations per system], [true relative residual per system])."""
    its = (ctypes.c_int32 * nrhs)()
    res = (ctypes.c_double * nrhs)()
    st = lib.dslash_cg_multi_blocked(h, nrhs, x_ptr, b_ptr, parity, mass, rel_tol, max_iter, its, res, stream)
    if st not in (DSLASH_OK, DSLASH_ERR_NOT_CONVERGED):
        check(st, h)
    return st, list(its), list(res)


def dslash_cg_mixed(h, x_ptr, b_ptr, parity, mass, rel_tol, inner_tol, max_iter, stream=0):
    """Returns (status, inner iterations, outer corrections, true relative residual)."""
    it, outer = ctypes.c_int32(), ctypes.c_int32()
    res = ctypes.c_double()
    st = lib.dslash_cg_mixed(h, x_ptr, b_ptr, parity, mass, rel_tol, inner_tol, max_iter, ctypes.byref(it),
                             ctypes.byref(outer), ctypes.byref(res), stream)
    if st not in (DSLASH_OK, DSLASH_ERR_NOT_CONVERGED):
        check(st, h)
    return st, it.value, outer.value, res.value


def dslash_halo_start(h, in_ptr, src_parity, stream=0):
    return check(lib.dslash_halo_start(h, in_ptr, src_parity, stream), h)


def dslash_halo_wait(h, stream=0):
    return check(lib.dslash_halo_wait(h, stream), h)


def dslash_sync(h):
    return check(lib.dslash_sync(h), h)


def dslash_kernel_timing(h, which=DSLASH_TIMING_ALL):
    ms = ctypes.c_double()
    n = ctypes.c_int64()
    check(lib.dslash_kernel_timing(h, which, ctypes.byref(ms), ctypes.byref(n)), h)
    return ms.value, n.value


def dslash_kernel_timing_reset(h):
    return check(lib.dslash_kernel_timing_reset(h), h)


def dslash_timeline(h, max_entries=4096):
    """[(kind, start_ms, end_ms)] of the recorded intervals (kernels, spans, exchanges)."""
    n = ctypes.c_int64(0)
    kinds = (ctypes.c_int32 * max_entries)()
    a = (ctypes.c_double * max_entries)()
    b = (ctypes.c_double * max_entries)()
    check(lib.dslash_timeline(h, max_entries, kinds, a, b, ctypes.byref(n)), h)
    return [(kinds[i], a[i], b[i]) for i in range(min(n.value, max_entries))]


def dslash_get_plan(h) -> dslash_plan_t:
    p = dslash_plan_t()
    check(lib.dslash_get_plan(h, ctypes.byref(p)), h)
    return p


def dslash_local_half_volume(h) -> int:
    return int(lib.dslash_local_half_volume(h))


def dslash_destroy(h):
    return check(lib.dslash_destroy(h))


def dslash_error_string(h=None) -> str:
    return error_string(h)
